import sys, time, json
sys.path.insert(0, '/root/repo')
import numpy as np, torch
import paper_conf_ppopp_0044ws18_b200 as g
from synth import make_workload
c, ql, cfg = make_workload('c2')
k = 10; nq = ql.num_queries
ixs = [g.GriffinIndex(c, block_size=128) for _ in range(3)]
mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
for ix in ixs: ix.griffin_reserve(ql.offsets, ql.terms, k)
outs = [(torch.zeros(nq*k, dtype=torch.int64, device='cuda'), torch.zeros(nq, dtype=torch.int32, device='cuda')) for _ in ixs]
streams = [torch.cuda.Stream() for _ in ixs]
for S in (1, 2, 3):
    for it in range(3):
        for i in range(S):
            ixs[i].griffin_query_batch_device(d_off, d_t, mt, k, outs[i][0], outs[i][1], streams[i])
    torch.cuda.synchronize()
    K = 60
    t0 = time.perf_counter()
    for step in range(K):
        i = step % S
        ixs[i].griffin_query_batch_device(d_off, d_t, mt, k, outs[i][0], outs[i][1], streams[i])
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    print(json.dumps({"streams": S, "ms_per_batch": 1e3*dt/K, "qps": nq*K/dt}), flush=True)
