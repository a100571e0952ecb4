"""Decode-only sweep (SURVEY §8(d) C5 sweep row) over a named config's index."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_0044ws18_b200 as g
from synth import make_workload
cfg_name = sys.argv[1] if len(sys.argv) > 1 else "c2"
blocks = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [128]
iters = int(sys.argv[3]) if len(sys.argv) > 3 else 5
c, ql, cfg = make_workload(cfg_name, num_queries=1)
for B in blocks:
    ix = g.GriffinIndex(c, block_size=B)
    r = ix.griffin_debug_decode_all(iters=iters)
    r["B"] = B
    r["gbs"] = r["bytes"] / (r["ms"] / 1e3) / 1e9
    r["gpostings_per_s"] = r["postings"] / (r["ms"] / 1e3) / 1e9
    print(json.dumps(r), flush=True)
    ix.close()
