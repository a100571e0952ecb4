"""Top CUDA source lines of one launch by instructions and by stall samples,
plus per-function totals (function = nearest preceding __device__/__global__
definition).  usage: python tools/ncu_lines2.py report.ncu-rep launch_index [N]"""
import collections, csv, io, re, subprocess, sys
rep, idx = sys.argv[1], int(sys.argv[2])
N = int(sys.argv[3]) if len(sys.argv) > 3 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-skip", str(idx), "--launch-count", "1"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
cur = None; hdr = None; src = collections.defaultdict(dict); data = []
for r in rows:
    if len(r) == 2 and r[0] in ("File Name", "File Path"):
        cur = r[1].split("/")[-1]; hdr = None; continue
    if r and r[0] == "Line No":
        hdr = r; continue
    if hdr and len(r) == len(hdr) and r[2] == "-":
        try:
            s = float(r[4] or 0); ie = float(r[7] or 0)
        except ValueError:
            continue
        ln = int(r[0]); src[cur][ln] = r[1]
        data.append((cur, ln, s, ie, r[1].strip()))
    elif hdr is None and len(r) == 2 and r[0].isdigit() and cur:
        src[cur][int(r[0])] = r[1]
fre = re.compile(r"(__global__|__device__).*?(\w+)\s*\(")
def func_of(f, ln):
    lines = src[f]
    for l in range(ln, 0, -1):
        t = lines.get(l, "")
        m = fre.search(t)
        if m and "(" in t and not t.strip().startswith("//"):
            return m.group(2)
    return "?"
ts = sum(d[2] for d in data) or 1; ti = sum(d[3] for d in data) or 1
print(f"stall samples {ts:.0f}, warp inst {ti:.4g}")
agg = collections.defaultdict(lambda: [0.0, 0.0])
for f, ln, s, ie, t in data:
    k = f + ":" + func_of(f, ln); agg[k][0] += s; agg[k][1] += ie
print("-- by function")
for k, v in sorted(agg.items(), key=lambda x: -x[1][1])[:25]:
    print(f"  {k:45s} inst {100*v[1]/ti:5.1f}%  stall {100*v[0]/ts:5.1f}%")
print("-- top lines by instructions")
for f, ln, s, ie, t in sorted(data, key=lambda d: -d[3])[:N]:
    print(f"  {100*ie/ti:5.1f}% ins {100*s/ts:5.1f}% smp  {f}:{ln}  {t[:90]}")
print("-- top lines by stall")
for f, ln, s, ie, t in sorted(data, key=lambda d: -d[2])[:N]:
    print(f"  {100*s/ts:5.1f}% smp {100*ie/ti:5.1f}% ins  {f}:{ln}  {t[:90]}")
