"""Per-kernel summary of an ncu --csv metrics log (one line per launch).
usage: python tools/ncu_brief.py log.csv"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, out = None, collections.OrderedDict()
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        out.setdefault((d["ID"], d["Kernel Name"][:42]), {})[d["Metric Name"]] = d["Metric Value"]


def f(v, k, s=1.0):
    try:
        return float(v.get(k, "nan").replace(",", "")) / s
    except ValueError:
        return float("nan")


for (i, n), v in out.items():
    print("%3s %-42s ms=%.3f rd=%.2fGB wr=%.2fGB l2hit=%.1f inst=%.3g warps=%.1f issue=%.1f" % (
        i, n, f(v, "gpu__time_duration.sum", 1e6), f(v, "dram__bytes_read.sum", 1e9),
        f(v, "dram__bytes_write.sum", 1e9), f(v, "lts__t_sector_hit_rate.pct"),
        f(v, "smsp__inst_executed.sum"), f(v, "sm__warps_active.avg.pct_of_peak_sustained_active"),
        f(v, "smsp__issue_active.avg.pct_of_peak_sustained_active")))
