"""Per-region stall samples, instructions and average active threads of one
launch in an ncu report (cuda,sass source page), regions = source line ranges.
usage: python tools/ncu_regions.py report.ncu-rep launch_index"""
import collections
import csv
import io
import subprocess
import sys

rep, idx = sys.argv[1], int(sys.argv[2])
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-skip", str(idx), "--launch-count", "1"], capture_output=True,
                     text=True).stdout
REG = {'merge_loop': ('query.cu', 1216, 1265), 'fine_split': ('griffin_dev.cuh', 515, 535),
       'emit_lanes': ('query.cu', 432, 500), 'emit_unit': ('query.cu', 360, 431),
       'tf/bm25': ('griffin_dev.cuh', 460, 480), 'decoders': ('griffin_dev.cuh', 143, 420),
       'nextgeq': ('griffin_dev.cuh', 421, 459),
       'staging': ('query.cu', 250, 359), 'arena_probe': ('query.cu', 739, 826),
       'skip_search': ('query.cu', 641, 738), 'probe_unit': ('query.cu', 827, 999),
       'gallop_unit': ('query.cu', 1266, 1468), 'merge_unit_setup': ('query.cu', 1079, 1215),
       'unit_head': ('query.cu', 1000, 1078), 'lower_bound_s': ('griffin_dev.cuh', 481, 514),
       'carve': ('query.cu', 200, 249), 'scan82': ('griffin_dev.cuh', 76, 86)}
rows = list(csv.reader(io.StringIO(out)))
cur, hdr = None, None
agg = collections.defaultdict(lambda: [0, 0, 0, 0])
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        cur = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr and len(r) == len(hdr) and r[2] == "-":
        try:
            s = float(r[hdr.index("Warp Stall Sampling (All Samples)")] or 0)
            ie = float(r[hdr.index("Instructions Executed")] or 0)
            te = float(r[hdr.index("Thread Instructions Executed")] or 0)
            ni = float(r[hdr.index("stall_no_inst")] or 0) if "stall_no_inst" in hdr else 0.0
        except ValueError:
            continue
        ln = int(r[0])
        name = "other:" + str(cur)
        for k, (f, a, b) in REG.items():
            if f == cur and a <= ln <= b:
                name = k
                break
        agg[name][0] += s
        agg[name][1] += ie
        agg[name][2] += te
        agg[name][3] += ni
ts = sum(v[0] for v in agg.values()) or 1
ti = sum(v[1] for v in agg.values()) or 1
tn = sum(v[3] for v in agg.values()) or 1
print(f"total stall samples {ts:.0f}, warp instructions {ti:.3g}, no_inst samples {tn:.0f}")
for k, v in sorted(agg.items(), key=lambda x: -x[1][0]):
    print(f"{k:18s} stall {100*v[0]/ts:5.1f}%  inst {100*v[1]/ti:5.1f}%  avg thr {v[2]/max(v[1],1):5.1f}  no_inst {100*v[3]/tn:5.1f}%")
