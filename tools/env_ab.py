"""A/B of build-time env knobs on one generated workload (GPU box): for each
VAR=value spec, build the index with that env, time batches (1 stream, 5 x 3
batches, median) and print per-stage ms.  usage: python tools/env_ab.py c5 GRIFFIN_SORDER=0 GRIFFIN_SORDER=4"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_0044ws18_b200 as g  # noqa: E402
from synth import make_workload  # noqa: E402

cfg_name = sys.argv[1]
c, ql, cfg = make_workload(cfg_name)
k, nq = cfg["k"], ql.num_queries
mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
keys = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
cnt = torch.zeros(nq, dtype=torch.int32, device="cuda")
st = torch.cuda.current_stream()
stages = ("ms_plan", "ms_decode", "ms_intersect", "ms_compact", "ms_topk")
reps, per = (5, 3) if nq > 2000 else (7, 10)
for spec in sys.argv[2:] * 2:
    var, val = spec.split("=")
    os.environ[var] = val
    ix = g.GriffinIndex(c, block_size=cfg["block"])
    ix.griffin_reserve(ql.offsets, ql.terms, k)
    for _ in range(3):
        ix.griffin_query_batch_device(d_off, d_t, mt, k, keys, cnt, st)
    torch.cuda.synchronize()
    tot, agg = [], {s: [] for s in stages}
    for rep in range(reps):
        ix.griffin_reset_profile()
        ix.griffin_set_profiling(True)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        for _ in range(per):
            ix.griffin_query_batch_device(d_off, d_t, mt, k, keys, cnt, st)
        b.record(st)
        torch.cuda.synchronize()
        ix.griffin_set_profiling(False)
        p = ix.griffin_get_profile()
        tot.append(a.elapsed_time(b) / per)
        for s in stages:
            agg[s].append(p[s] / per)
    print(json.dumps({"config": cfg_name, "spec": spec, "ms_per_batch": round(statistics.median(tot), 4),
                      **{s: round(statistics.median(v), 4) for s, v in agg.items()}}), flush=True)
    del ix
    torch.cuda.empty_cache()
