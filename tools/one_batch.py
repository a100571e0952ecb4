"""Run batch 0 of a workload a few times through the device API (ncu target).
usage: python tools/one_batch.py <config> [reuse 0/1/2] [repeats]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_0044ws18_b200 as g  # noqa: E402
from synth import batch_of, make_workload  # noqa: E402

cfg_name = sys.argv[1] if len(sys.argv) > 1 else "c2"
reuse = int(sys.argv[2]) if len(sys.argv) > 2 else 2
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
c, ql, cfg = make_workload(cfg_name)
ql = batch_of(ql, cfg, 0)
k, nq = cfg["k"], ql.num_queries
ix = g.GriffinIndex(c, block_size=cfg["block"])
ix.griffin_set_reuse(reuse)
ix.griffin_reserve(ql.offsets, ql.terms, k)
mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
keys = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
cnt = torch.zeros(nq, dtype=torch.int32, device="cuda")
for _ in range(reps):
    ix.griffin_query_batch_device(d_off, d_t, mt, k, keys, cnt, torch.cuda.current_stream())
    torch.cuda.synchronize()
ix.griffin_sync_status()
print("ok", cfg_name, nq, int(cnt.sum()))
