"""Print the key numbers of a bench JSON line.  usage: python tools/bench_brief.py file.json"""
import json
import sys

d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value %.0f  ms/step %.3f  e2e %s  sync %s" % (d["value"], d["ms_per_step"],
      (d.get("e2e") or {}).get("value"), (d.get("sync_qps") or {}).get("value")))
print("stages", {k: round(v, 3) for k, v in d["stage_ms_per_step_isolated"].items()})
r = d["roofline"]
print("roofline frac %.3f  achieved %.0f GB/s  ms/launch %.3f  frac_all %.3f" %
      (r["frac"], r["achieved"], r["ms_per_launch"], r.get("frac_all_bytes", 0)))
print("units", {k: int(v) for k, v in d["kernels"]["intersect_kernel"]["units_per_step"].items()})
if d.get("parity"):
    print("parity", d["parity"])
