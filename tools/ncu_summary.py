"""Summarise an `ncu --set full` report of the bench into profiles/ (committed).

usage: python tools/ncu_summary.py gpurun_out/prof_X.ncu-rep <tag> [config]

Writes profiles/<tag>_ncu_kernels.txt (per-launch duration, DRAM bytes, issue %,
occupancy, stall mix, top source lines) and profiles/ncu_summary_<config>.json
(mean DRAM read+write bytes per launch per kernel; bench.py reports it as
roofline.traffic).
"""
import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
rep, tag = sys.argv[1], sys.argv[2]
config = sys.argv[3] if len(sys.argv) > 3 else "c2"

out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr, units = rows[0], rows[1]
U = dict(zip(hdr, units))


def val(d, k, scale_to=None):
    v = d.get(k)
    try:
        v = float(v)
    except (TypeError, ValueError):
        return None
    u = U.get(k, "")
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ms": 1e-3, "us": 1e-6,
            "ns": 1e-9, "s": 1.0}.get(u, 1)
    return v * mult


lines = [f"# ncu --set full summary ({os.path.basename(rep)})", ""]
per_kernel = defaultdict(list)
for r in rows[2:]:
    d = dict(zip(hdr, r))
    name = d["Kernel Name"].split("(")[0].replace("void ", "").replace("griffin::", "")
    t = val(d, "gpu__time_duration.sum")
    rd = val(d, "dram__bytes_read.sum") or 0.0
    wr = val(d, "dram__bytes_write.sum") or 0.0
    per_kernel[name].append(rd + wr)
    stalls = []
    for h, v in d.items():
        if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("_not_issued"):
            try:
                stalls.append((float(v), h.replace("smsp__pcsamp_warps_issue_stalled_", "")))
            except ValueError:
                pass
    tot = sum(x for x, _ in stalls) or 1.0
    # warp-execution efficiency = active threads per executed warp instruction / 32;
    # divergence = branch targets reached by a divergent subset of a warp's threads
    r = val(d, "smsp__thread_inst_executed_per_inst_executed.ratio")
    wee = f"{100 * r / 32:.1f}%" if r is not None else "n/a"
    dv = val(d, "smsp__sass_branch_targets_threads_divergent.sum")
    br = val(d, "smsp__inst_executed_op_branch.sum")
    div = (f"{dv:.3g} ({100 * dv / br:.1f}% of {br:.3g} branch instr)" if dv is not None and br
           else "n/a")
    top = ", ".join(f"{h} {100 * x / tot:.0f}%" for x, h in sorted(stalls, reverse=True)[:4])
    lines.append(f"{name}: {t * 1e3:.3f} ms, DRAM read {rd / 1e6:.1f} MB write {wr / 1e6:.1f} MB "
                 f"({(rd + wr) / t / 1e9:.0f} GB/s), inst {val(d, 'smsp__inst_executed.sum'):.3g}, "
                 f"issue {d.get('smsp__issue_active.avg.pct_of_peak_sustained_active')}%, "
                 f"warps active {d.get('sm__warps_active.avg.pct_of_peak_sustained_active')}%, "
                 f"warp-exec efficiency {wee}, divergent branch targets {div}, "
                 f"stalls: {top}")
lines.append("")
for idx in range(len(rows) - 2):
    name = rows[2 + idx][hdr.index("Kernel Name")]
    if "intersect" in name or "decode" in name or "probe" in name:
        src = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "ncu_lines2.py"), rep,
                              str(idx), "12"], capture_output=True, text=True).stdout
        lines.append(f"## top source lines, launch {idx}: {name.split('(')[0]}")
        lines += src.strip().splitlines()
        lines.append("")
os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
with open(os.path.join(ROOT, "profiles", f"{tag}_ncu_kernels.txt"), "w") as f:
    f.write("\n".join(lines) + "\n")
summ = {"source": os.path.basename(rep), "config": config,
        "dram_bytes_per_launch": {k: sum(v) / len(v) for k, v in per_kernel.items()}}
# bench.py keys
# the intersect stage = round 1 (intersect_kernel<1, 1> merge units followed by
# intersect_kernel<1, 2> gallop/single-term units: ONE timed stage section) + the
# later rounds (the probe pass probe_kernel, or intersect_kernel<0, 0> without
# it). Per stage section, like bench.py's launch count (launches_intersect).
_stage = [k for k in per_kernel if k.startswith("intersect_kernel") or k == "probe_kernel"]
_bytes = sum(sum(per_kernel[k]) for k in _stage)
_sections = sum(len(per_kernel[k]) for k in _stage if not k.replace(" ", "").endswith(",2>"))
summ["dram_bytes_per_launch"]["intersect_kernel"] = _bytes / max(1, _sections)
with open(os.path.join(ROOT, "profiles", f"ncu_summary_{config}.json"), "w") as f:
    json.dump(summ, f, indent=1)
print("\n".join(lines))
