"""Top CUDA source lines by L2 sectors requested by global accesses (ncu source page).
usage: python tools/ncu_sectors.py report.ncu-rep [launch_index] [topn]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
idx = int(sys.argv[2]) if len(sys.argv) > 2 else 0
topn = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-skip", str(idx), "--launch-count", "1"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
cur, hdr, recs = None, None, []
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        cur = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr and len(r) == len(hdr) and r[2] == "-":
        def gi(k):
            try:
                return int(float(r[hdr.index(k)] or 0))
            except ValueError:
                return 0
        recs.append((gi("L2 Theoretical Sectors Global"), gi("L2 Theoretical Sectors Global Ideal"),
                     cur, r[0], r[1][:90]))
tot = sum(x[0] for x in recs) or 1
print(f"total L2 sectors (global ld/st) {tot} = {tot * 32 / 1e6:.1f} MB")
for s, ideal, f, ln, src in sorted(recs, reverse=True)[:topn]:
    print(f"{100 * s / tot:5.1f}%  {s * 32 / 1e6:8.1f} MB (ideal {ideal * 32 / 1e6:7.1f})  {f}:{ln}  {src}")
