"""Aggregate an ncu report's cuda,sass source page by CUDA source line.
usage: python tools/ncu_lines.py report.ncu-rep [launch_index] [topn]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
idx = int(sys.argv[2]) if len(sys.argv) > 2 else 0
topn = int(sys.argv[3]) if len(sys.argv) > 3 else 40
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
        recs.append((gi("Warp Stall Sampling (All Samples)"), gi("Instructions Executed"), cur, r[0], r[1][:100]))
tot_s = sum(x[0] for x in recs) or 1
tot_i = sum(x[1] for x in recs) or 1
print(f"total stall samples {tot_s}, warp instructions executed {tot_i}")
key = (lambda r: (r[1], r[0])) if "--by-inst" in sys.argv else None
for s, i, f, ln, src in sorted(recs, key=key, reverse=True)[:topn]:
    print(f"{100*s/tot_s:5.1f}% smp {100*i/tot_i:5.1f}% ins  {f}:{ln}  {src}")
