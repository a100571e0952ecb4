"""Multi-process (gloo, world size 2, CPU) tests of the N>1 plumbing: docID
range shards, the g-major all-gather layout the merge kernel consumes, and the
exactness of merging per-shard top-k.  The per-shard ranking
comes from the (never sharded) oracle's global ranking restricted to the
shard's docID range; the merge here is a plain sorted-merge reference, the
device merge kernel itself is covered by tests/test_gpu_parity.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_q, exchange="allgather"):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import paper_conf_ppopp_0044ws18_b200 as g
        from paper_conf_ppopp_0044ws18_b200.sharded import (exchange_sliced, gather_runs,
                                                            query_slices)
        from synth import make_workload
        c, ql, cfg = make_workload("tiny")
        ox = oracle.OracleIndex(c)
        k = 7
        nq = ql.num_queries
        # global ranking (all results) from the oracle, then this shard's top-k
        D, S, C = ox.query_batch(ql, 4096)
        base, end = g.griffin_shard_range(c.num_docs, world, rank)
        keys = np.zeros((nq, k), np.uint64)
        cnts = np.zeros(nq, np.int32)
        for q in range(nq):
            sel = [(int(S[q, i].view(np.uint32)), int(D[q, i])) for i in range(C[q])
                   if base <= D[q, i] < end]
            sel = sel[:k]
            cnts[q] = len(sel)
            for i, (sb, d) in enumerate(sel):
                keys[q, i] = (np.uint64(sb) << np.uint64(32)) | np.uint64(0xFFFFFFFF - d)
        kt = torch.from_numpy(keys.view(np.int64).reshape(-1).copy())
        ct = torch.from_numpy(cnts)
        if exchange == "allgather":
            all_k, all_c = gather_runs(kt, ct)
            lo, hi = 0, nq
        else:
            all_k, all_c, (lo, hi) = exchange_sliced(kt, ct, k)
            assert (lo, hi) == query_slices(nq, world)[rank]
        m = hi - lo
        assert all_k.shape == (world, m * k) and all_c.shape == (world, m)
        # reference k-way merge over the g-major runs
        ok = True
        for q in range(lo, hi):
            runs = []
            for r in range(world):
                n = int(all_c[r, q - lo])
                runs += [int(x) & 0xFFFFFFFFFFFFFFFF
                         for x in all_k[r, (q - lo) * k:(q - lo) * k + n].tolist()]
            top = sorted(runs, reverse=True)[:k]
            want = [(int(S[q, i].view(np.uint32)) << 32) | (0xFFFFFFFF - int(D[q, i]))
                    for i in range(min(k, C[q]))]
            ok &= top == want
        out_q.put((rank, ok))
    finally:
        dist.destroy_process_group()


def _run(world, exchange):
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, exchange))
             for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(ok for _, ok in res), res


def test_gloo_world2_shard_exchange_and_merge_exact():
    _run(2, "allgather")


def test_gloo_world3_query_sliced_exchange_exact():
    """NEXT-2: all-to-all of per-shard runs by query slice (uneven slices at G=3)."""
    _run(3, "sliced")


def test_query_slices_cover():
    from paper_conf_ppopp_0044ws18_b200.sharded import query_slices
    for nq in (0, 1, 2, 7, 1000):
        for w in (1, 2, 3, 8):
            sl = query_slices(nq, w)
            assert len(sl) == w and sl[0][0] == 0 and sl[-1][1] == nq
            assert all(a <= b for a, b in sl)
            assert all(sl[i][1] == sl[i + 1][0] for i in range(w - 1))
