"""Where does a C2 batch's time go beyond its kernels?  Times the batch loop
(1 and 2 streams, profiling off/on), the host enqueue cost per batch, and the
sum of kernel durations (profiling events) — run on the GPU box."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_0044ws18_b200 as g  # noqa: E402
from synth import make_workload  # noqa: E402

c, ql, cfg = make_workload(sys.argv[1] if len(sys.argv) > 1 else "c2")
k = cfg["k"]
nq = ql.num_queries
ix = g.GriffinIndex(c, block_size=cfg["block"])
ix.griffin_reserve(ql.offsets, ql.terms, k)
ws = ix.griffin_workspace_create()
ws.griffin_workspace_reserve(ql.offsets, ql.terms, k)
mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
outs = [(torch.zeros(nq * k, dtype=torch.int64, device="cuda"),
         torch.zeros(nq, dtype=torch.int32, device="cuda")) for _ in range(2)]
streams = [torch.cuda.current_stream(), torch.cuda.Stream()]


def launch(i):
    kk, cc = outs[i]
    if i == 0:
        ix.griffin_query_batch_device(d_off, d_t, mt, k, kk, cc, streams[0])
    else:
        ws.griffin_query_batch_device_ws(d_off, d_t, mt, k, kk, cc, streams[1])


for prof in (False, True):
    ix.griffin_set_profiling(prof)
    for S in (1, 2):
        for i in range(6):
            launch(i % S)
        torch.cuda.synchronize()
        ix.griffin_reset_profile()
        K = 40
        enq = 0.0
        t0 = time.perf_counter()
        for step in range(K):
            a = time.perf_counter()
            launch(step % S)
            enq += time.perf_counter() - a
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        line = {"profiling": prof, "streams": S, "ms_per_batch": 1e3 * dt / K,
                "enqueue_ms_per_batch": 1e3 * enq / K, "qps": nq * K / dt}
        if prof:
            p = ix.griffin_get_profile()
            line["stage_ms_sum_per_batch"] = sum(p[x] for x in (
                "ms_plan", "ms_decode", "ms_intersect", "ms_compact", "ms_topk")) / K
            line["launches_per_batch"] = p["launches_total"] / K
        print(json.dumps(line), flush=True)
