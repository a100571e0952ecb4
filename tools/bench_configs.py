"""Measurements for the BASELINE.json configs beyond bench.py's headline C2 line.

  python tools/bench_configs.py c1        single-query closed-loop latency (p50/p99), C1
  python tools/bench_configs.py c3        merge-vs-gallop crossover over the paper's ratio
                                          groups (Fig. 8 / Fig. 13 analog, GPU only)
  python tools/bench_configs.py c5 [nq]   10K-query top-1000 batch on the 50M-doc index +
                                          decode-only sweep over block sizes 64..512
  python tools/bench_configs.py codecs [cfg]  EF vs PforDelta (NEXT-3): bits/posting and
                                          decode-only sweep on the same lists (Table 1 /
                                          Fig. 12 shape)

Each prints JSON lines (one per measurement).  Timing: CUDA events on the
launching stream for device-side numbers, perf_counter for host-API latency.
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_0044ws18_b200 as g  # noqa: E402
from synth import batch_of, make_pair_workload, make_workload  # noqa: E402


def dev_batch(ix, ql, k):
    nq = ql.num_queries
    ix.griffin_reserve(ql.offsets, ql.terms, k)
    d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
    d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
    keys = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
    cnt = torch.zeros(nq, dtype=torch.int32, device="cuda")
    mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
    st = torch.cuda.current_stream()

    def run():
        ix.griffin_query_batch_device(d_off, d_t, mt, k, keys, cnt, st)
    return run


def time_dev(run, iters=10, warmup=3):
    for _ in range(warmup):
        run()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(iters):
        run()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / iters


def c1():
    c, ql, cfg = make_workload("c1")
    ix = g.GriffinIndex(c, block_size=128)
    terms = ql.query(0)
    for _ in range(200):
        ix.griffin_query(terms, 10)
    lat = []
    for _ in range(10_000):
        t0 = time.perf_counter()
        ix.griffin_query(terms, 10)
        lat.append((time.perf_counter() - t0) * 1e3)
    lat.sort()
    run = dev_batch(ix, ql, 10)
    ms = time_dev(run, iters=200)
    prof = None
    print(json.dumps({"config": "c1", "metric": "single-query latency (griffin_query, host buffers)",
                      "p50_ms": lat[len(lat) // 2], "p99_ms": lat[int(0.99 * len(lat)) - 1],
                      "closed_loop_qps": 1e3 / (sum(lat) / len(lat)),
                      "device_ms_per_query": ms, "df": [int(c.df()[t]) for t in terms]}),
          flush=True)


def c3():
    """Merge vs gallop per ratio group (P:858-859 groups + lambda = 1000), at batch
    scale: 64 pairs per group share one |S| = 1.5M list (fused decode, reuse off,
    as in the paper's per-pair measurement; and with the batch arena, reuse on)."""
    from synth import make_ratio_groups
    groups = [(1, 16), (16, 32), (32, 64), (64, 128), (128, 256), (256, 512), (512, 1024),
              (1000, 1001)]
    c, ql, gid = make_ratio_groups(25_000_000, 1_500_000, groups, 64, seed=0x4752494646494E03)
    ix = g.GriffinIndex(c, block_size=128)
    for gi, (lo, hi) in enumerate(groups):
        qs = np.nonzero(gid == gi)[0]
        sub = ql.slice(int(qs[0]), int(qs[-1]) + 1)
        res = {"config": "c3", "group": [lo, hi], "pairs": len(qs),
               "R_len_mean": float(np.mean([c.df()[sub.query(i)[0]] for i in range(sub.num_queries)])),
               "S_len": int(c.df()[sub.query(0)[1]])}
        for reuse in (0, 1):
            ix.griffin_set_reuse(reuse)
            for name, mode, ngeq in (("merge", g.MODE_MERGE, 1), ("gallop", g.MODE_GALLOP, 1),
                                     ("gallop_blockdec", g.MODE_GALLOP, 0),
                                     ("auto", g.MODE_AUTO, 1)):
                if reuse and ngeq == 0:
                    continue
                ix.griffin_set_mode(mode)
                ix.griffin_set_nextgeq(ngeq)
                run = dev_batch(ix, sub, 10)
                ix.griffin_reset_profile()
                ix.griffin_set_profiling(True)
                ms = time_dev(run, iters=5, warmup=2)
                ix.griffin_set_profiling(False)
                p = ix.griffin_get_profile()
                res[f"{name}{'_reuse' if reuse else ''}"] = {
                    "us_per_pair": 1e3 * ms / len(qs),
                    "intersect_us_per_pair": 1e3 * p["ms_intersect"] / 7 / len(qs),
                    "payload_KB_per_pair": p["payload_bytes"] / 7 / len(qs) / 1e3,
                    "decoded_postings_per_pair": p["decoded_postings"] / 7 / len(qs)}
        res["winner_fused"] = ("merge" if res["merge"]["intersect_us_per_pair"] <=
                               res["gallop"]["intersect_us_per_pair"] else "gallop")
        res["winner_reuse"] = ("merge" if res["merge_reuse"]["intersect_us_per_pair"] <=
                               res["gallop_reuse"]["intersect_us_per_pair"] else "gallop")
        print(json.dumps(res), flush=True)


def c5(nq=None):
    t0 = time.time()
    c, ql, cfg = make_workload("c5")
    ql = batch_of(ql, cfg, 0)
    if nq:
        ql = ql.slice(0, nq)
    gen_s = time.time() - t0
    k = cfg["k"]
    for B in (128, 64, 256, 512):
        t0 = time.time()
        ix = g.GriffinIndex(c, block_size=B)
        build_s = time.time() - t0
        st = ix.griffin_index_stats()
        sw = ix.griffin_debug_decode_all(iters=3)
        line = {"config": "c5", "block_size": B, "num_postings": c.num_postings,
                "gen_s": gen_s, "build_s": build_s, "index_bytes": st["payload_bytes"] +
                st["skip_bytes"] + st["tf_bytes"],
                "decode_sweep": {"ms": sw["ms"], "gbs": sw["bytes"] / (sw["ms"] / 1e3) / 1e9,
                                 "gpostings_per_s": sw["postings"] / (sw["ms"] / 1e3) / 1e9}}
        if B == 128:
            for kq in (k, 10):   # C5 (top-1000) and the C4 per-shard workload at G = 1 (top-10)
                run = dev_batch(ix, ql, kq)
                ix.griffin_reset_profile()
                ix.griffin_set_profiling(1)
                ms = time_dev(run, iters=3, warmup=2)
                ix.griffin_set_profiling(False)
                p = ix.griffin_get_profile()
                line[f"k{kq}"] = {"queries": ql.num_queries, "k": kq, "ms_per_batch": ms,
                                  "qps": ql.num_queries / (ms / 1e3),
                                  "intersect_alg_gbs": p["alg_bytes"] / (p["ms_intersect"] / 1e3) / 1e9,
                                  "stage_ms": {kk: p[kk] / 5 for kk in (
                                      "ms_plan", "ms_decode", "ms_intersect", "ms_compact",
                                      "ms_topk")}}
        print(json.dumps(line), flush=True)
        ix.close()


def codecs(cfg_name="c2"):
    c, _, cfg = make_workload(cfg_name, num_queries=1)
    for B in (128, 64, 256):
        ix = g.GriffinIndex(c, block_size=B)
        st = ix.griffin_index_stats()
        ef_bytes = st["payload_bytes"] + st["skip_bytes"]
        sw = ix.griffin_debug_decode_all(iters=5)
        ix.close()
        px = g.GriffinPfd(c, block_size=B)
        ps = px.griffin_pfd_stats()
        pf_bytes = ps["payload_bytes"] + ps["skip_bytes"]
        pw = px.griffin_pfd_decode_all(iters=5)
        px.close()
        P = c.num_postings
        line = {"config": cfg_name, "block_size": B, "postings": P,
                "ef": {"bits_per_posting": 8 * ef_bytes / P, "compression_ratio": 32 * P / (8 * ef_bytes),
                       "decode_ms": sw["ms"], "decode_gbs": sw["bytes"] / (sw["ms"] / 1e3) / 1e9,
                       "gpostings_per_s": sw["postings"] / (sw["ms"] / 1e3) / 1e9},
                "pfd": {"bits_per_posting": 8 * pf_bytes / P, "compression_ratio": 32 * P / (8 * pf_bytes),
                        "exception_frac": ps["exceptions"] / max(1, P - ps["num_blocks"]),
                        "decode_ms": pw["ms"], "decode_gbs": pw["bytes"] / (pw["ms"] / 1e3) / 1e9,
                        "gpostings_per_s": pw["postings"] / (pw["ms"] / 1e3) / 1e9},
                "paper_table1": {"pfd_ratio": 3.3, "ef_ratio": 4.6, "note": "ClueWeb12, CPU PforDelta"}}
        line["ef_vs_pfd_size"] = pf_bytes / ef_bytes
        line["ef_vs_pfd_decode_speed"] = pw["ms"] / sw["ms"]
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    which = sys.argv[1]
    if which == "c1":
        c1()
    elif which == "c3":
        c3()
    elif which == "c5":
        c5(int(sys.argv[2]) if len(sys.argv) > 2 else None)
    elif which == "codecs":
        codecs(sys.argv[2] if len(sys.argv) > 2 else "c2")
