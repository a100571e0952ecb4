"""Batch-scale crossover sweep on a config's query log (GPU box): C2 batch time
per (T, Tdec) = (gallop_ratio, gallop_ratio_decoded) build option pair.
usage: python tools/t_sweep.py [config] [T:Tdec ...]"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_0044ws18_b200 as g  # noqa: E402
from synth import make_workload  # noqa: E402

cfg_name = sys.argv[1] if len(sys.argv) > 1 else "c2"
pairs = [tuple(int(x) for x in a.split(":")) for a in sys.argv[2:]] or [(16, 16)]
c, ql, cfg = make_workload(cfg_name)
k, nq = cfg["k"], ql.num_queries
mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
keys = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
cnt = torch.zeros(nq, dtype=torch.int32, device="cuda")
st = torch.cuda.current_stream()
for T, Td in pairs:
    ix = g.GriffinIndex(c, block_size=cfg["block"], gallop_ratio=T, gallop_ratio_decoded=Td)
    ix.griffin_reserve(ql.offsets, ql.terms, k)
    for _ in range(5):
        ix.griffin_query_batch_device(d_off, d_t, mt, k, keys, cnt, st)
    torch.cuda.synchronize()
    tot, xs = [], []
    for rep in range(7):
        ix.griffin_reset_profile()
        ix.griffin_set_profiling(True)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        for _ in range(10):
            ix.griffin_query_batch_device(d_off, d_t, mt, k, keys, cnt, st)
        b.record(st)
        torch.cuda.synchronize()
        ix.griffin_set_profiling(False)
        p = ix.griffin_get_profile()
        tot.append(a.elapsed_time(b) / 10)
        xs.append(p["ms_intersect"] / 10)
    print(json.dumps({"config": cfg_name, "T": T, "Tdec": Td, "ms_per_batch": statistics.median(tot),
                      "ms_intersect": statistics.median(xs)}), flush=True)
    del ix
    torch.cuda.empty_cache()
