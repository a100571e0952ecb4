"""Per-stage device time of one batch (1 stream, CUDA events per stage), median
over repeats — a low-variance A/B probe for kernel changes (GPU box)."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_0044ws18_b200 as g  # noqa: E402
from synth import batch_of, make_workload  # noqa: E402

cfg_name = sys.argv[1] if len(sys.argv) > 1 else "c2"
c, ql, cfg = make_workload(cfg_name)
ql = batch_of(ql, cfg, 0)
k = cfg["k"]
nq = ql.num_queries
ix = g.GriffinIndex(c, block_size=int(os.environ.get("PROBE_B", cfg["block"])))
ix.griffin_reserve(ql.offsets, ql.terms, k)
mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
keys = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
cnt = torch.zeros(nq, dtype=torch.int32, device="cuda")
st = torch.cuda.current_stream()
stages = ("ms_plan", "ms_decode", "ms_intersect", "ms_compact", "ms_topk")
variants = [("default", lambda: None)]
for extra in sys.argv[2:]:
    name, val = extra.split("=")
    variants.append((extra, lambda n=name, v=int(val): (getattr(ix, "griffin_set_" + n)(v),
                                                        ix.griffin_reserve(ql.offsets, ql.terms, k))))
for name, setup in variants:
    setup()
    for _ in range(5):
        ix.griffin_query_batch_device(d_off, d_t, mt, k, keys, cnt, st)
    torch.cuda.synchronize()
    per = {s: [] for s in stages}
    tot = []
    for rep in range(7):
        ix.griffin_reset_profile()
        ix.griffin_set_profiling(2)   # stage events only
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        for _ in range(10):
            ix.griffin_query_batch_device(d_off, d_t, mt, k, keys, cnt, st)
        b.record(st)
        torch.cuda.synchronize()
        ix.griffin_set_profiling(False)
        p = ix.griffin_get_profile()
        for s in stages:
            per[s].append(p[s] / 10)
        tot.append(a.elapsed_time(b) / 10)
    print(json.dumps({"config": cfg_name, "variant": name,
                      "ms_per_batch": statistics.median(tot),
                      **{s: round(statistics.median(v), 4) for s, v in per.items()}}), flush=True)
sw = ix.griffin_debug_decode_all(iters=5)
print(json.dumps({"config": cfg_name, "decode_sweep_ms": sw["ms"],
                  "gpostings_per_s": sw["postings"] / (sw["ms"] / 1e3) / 1e9,
                  "gbs": sw["bytes"] / (sw["ms"] / 1e3) / 1e9}), flush=True)
