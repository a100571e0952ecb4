#!/usr/bin/env python
"""Benchmark of the B200 Griffin-GPU conjunctive query path.

One "step" = one pass of the whole hot path (plus a8 for
N > 1) over one batch: the BASELINE.json configs[1] workload — a 10M-doc
synthetic Zipfian index (EF blocks of 128) and its 1000-query 2-5 term log,
BM25 top-10 — with the query log already resident in HBM.  Prints ONE JSON line.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2] [--impl reference]

N > 1 is launched by torchrun (one process per GPU): each rank holds one
docID-range shard of the same corpus, runs the batch, and the per-shard top-k
keys are all-gathered over NCCL and merged by the library's k-way merge kernel.
The reference arm (--impl reference) times the CPU oracle (the test oracle,
as it stands) on the same workload; there is no installable reference code.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

WORKLOAD_DESC = {
    "c1": "C1: single 2-term AND query, 100K-doc synthetic Zipf index (lists ~10K and ~1K), EF block 128, BM25 top-10",
    "c2": "C2: 10M-doc synthetic Zipf index (alpha 0.8, df 1K..5M, 42K terms, 0.19B postings), replayed 1000-query 2-5 term log, EF block 128, BM25 top-10",
    "c3": "C3: GOV2-shaped 25M-doc synthetic Zipf index (df up to 10M), 1000-query log, BM25 top-10",
    "c4": "C4: ClueWeb-shaped 50M-doc synthetic Zipf index (df up to 30M), 10K-query log, BM25 top-10",
    "c5": "C5: 50M-doc index, 10K concurrent queries, BM25 top-1000",
}


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """SM clock + throttle reasons sampled during the timed region: NVML in a
    background thread every 2 ms (the timed region can be tens of ms), with
    nvidia-smi as a fallback."""

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.samples = []
        self.max_mhz = 0.0
        self.reasons = set()
        self._stop = None
        self._th = None
        self._nvml = None

    def start(self):
        import threading
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.gpu)
            self.max_mhz = float(nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM))
            self._nvml = (nv, h)
        except Exception:
            self._nvml = None
        self._stop = threading.Event()
        self._th = threading.Thread(target=self._run, daemon=True)
        self._th.start()

    def _run(self):
        names = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
                 "sw_power_cap": 0x4}
        while not self._stop.is_set():
            if self._nvml:
                nv, h = self._nvml
                try:
                    self.samples.append(float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)))
                    fn = getattr(nv, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                        nv.nvmlDeviceGetCurrentClocksThrottleReasons
                    r = fn(h)
                    for nm, bit in names.items():
                        if r & bit:
                            self.reasons.add(nm)
                except Exception:
                    pass
                self._stop.wait(0.002)
            else:
                try:
                    out = subprocess.run(["nvidia-smi", "-i", str(self.gpu),
                                          "--query-gpu=clocks.sm,clocks.max.sm",
                                          "--format=csv,noheader,nounits"],
                                         capture_output=True, text=True, timeout=5).stdout
                    a, b = out.strip().split(",")[:2]
                    self.samples.append(float(a))
                    self.max_mhz = max(self.max_mhz, float(b))
                except Exception:
                    pass
                self._stop.wait(0.05)

    def stop(self):
        if self._th is None:
            return None
        self._stop.set()
        self._th.join(timeout=5)
        if not self.samples:
            return None
        mx = self.max_mhz or max(self.samples)
        loaded = [x for x in self.samples if x > 0.5 * mx] or self.samples
        return {"sm_mhz": statistics.median(loaded), "sm_max_mhz": mx,
                "reasons": sorted(self.reasons), "samples": len(self.samples),
                "source": "nvml" if self._nvml else "nvidia-smi"}


def _cpu_info():
    model = ""
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True).stdout
        for line in out.splitlines():
            if line.startswith("Model name"):
                model = line.split(":", 1)[1].strip()
    except OSError:
        pass
    return os.cpu_count() or 1, model


def oracle_baseline(corpus, ql, k, block, budget_s=12.0, threads=None):
    """Time the oracle (as it stands) on a bounded prefix of the query log."""
    import oracle
    cores, model = _cpu_info()
    threads = threads or cores
    t0 = time.time()
    ox = oracle.OracleIndex(corpus, block_size=block)
    build_s = time.time() - t0
    m = min(ql.num_queries, max(threads, 16))
    while True:
        sub = ql.slice(0, m)
        t0 = time.perf_counter()
        ox.query_batch(sub, k, nthreads=threads)
        dt = time.perf_counter() - t0
        if dt >= budget_s / 3 or m >= ql.num_queries:
            break
        m = min(ql.num_queries, int(m * max(2.0, budget_s / 3 / max(dt, 1e-3))))
    return {"value": m / dt, "unit": "queries/s", "cores": threads, "kind": "oracle",
            "sample": f"first {m} of the {ql.num_queries}-query log, {threads} std::threads, "
                      f"round-robin; oracle index build {build_s:.1f}s not timed",
            "cpu_model": model, "seconds": dt}, ox, m


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from synth import make_workload
    corpus, ql, cfg = make_workload(args.config)
    k = cfg["k"]
    base, ox, m = oracle_baseline(corpus, ql, k, cfg["block"], budget_s=6.0)
    sub = ql.slice(0, m)
    threads = base["cores"]
    for _ in range(args.warmup):
        ox.query_batch(sub, k, nthreads=threads)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        ox.query_batch(sub, k, nthreads=threads)
        times.append(time.perf_counter() - t0)
    ms = 1e3 * statistics.mean(times)
    qps = m / (ms / 1e3)
    base["value"] = qps
    line = {"impl": "reference", "metric": "queries/sec", "value": qps, "unit": "queries/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32/f32",
            "data": "synthetic",
            "config": {"workload": WORKLOAD_DESC[args.config], "num_docs": corpus.num_docs,
                       "queries_per_step": m, "k": k, "block_size": cfg["block"]},
            "cpu_baseline": base,
            "e2e": {"value": qps, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_gpu(args):
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_0044ws18_b200 as g
    from paper_conf_ppopp_0044ws18_b200.sharded import (ShardedSearcher, exchange_sliced,
                                                        gather_runs)
    from synth import make_workload

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    dev = torch.cuda.current_device()
    corpus, ql, cfg = make_workload(args.config)
    k, B = cfg["k"], cfg["block"]
    nq = ql.num_queries
    # docid: rank r holds docID-range shard r and the per-shard top-k are exchanged
    # (all-gather, or the query-sliced all-to-all); replicate: every rank holds the
    # whole index and runs its own batch, no exchange
    replicate = world > 1 and args.shard_mode == "replicate"
    sharded = world > 1 and not replicate
    t0 = time.time()
    if replicate:
        ix = g.GriffinIndex(corpus, block_size=B, device=dev)
    else:
        ix = g.GriffinIndex(corpus, block_size=B, device=dev, shard_index=rank, num_shards=world)
    build_s = time.time() - t0
    st = ix.griffin_index_stats()
    ix.griffin_reserve(ql.offsets, ql.terms, k)
    max_terms = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
    stream = torch.cuda.current_stream()
    d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
    d_terms = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
    keys = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
    cnts = torch.zeros(nq, dtype=torch.int32, device="cuda")
    # batches in flight: slot 0 = the index's own workspace on the current
    # stream, slots 1.. = extra workspaces on their own streams (serving engine
    # overlapping consecutive batches); each slot has its own outputs
    nstreams = max(1, args.streams) if not sharded else 1
    slots = [(None, stream, keys, cnts)]
    for _ in range(nstreams - 1):
        w = ix.griffin_workspace_create()
        w.griffin_workspace_reserve(ql.offsets, ql.terms, k)
        slots.append((w, torch.cuda.Stream(), torch.zeros(nq * k, dtype=torch.int64, device="cuda"),
                      torch.zeros(nq, dtype=torch.int32, device="cuda")))
    if sharded:
        out_keys = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
        out_cnts = torch.zeros(nq, dtype=torch.int32, device="cuda")
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device="cuda")  # 256 MB > L2

    def step_on(i):
        w, st_, kk_, cc_ = slots[i % len(slots)]
        if w is None:
            ix.griffin_query_batch_device(d_off, d_terms, max_terms, k, kk_, cc_, st_)
        else:
            w.griffin_query_batch_device_ws(d_off, d_terms, max_terms, k, kk_, cc_, st_)

    def step():
        ix.griffin_query_batch_device(d_off, d_terms, max_terms, k, keys, cnts, stream)
        if sharded and args.exchange == "allgather":
            ak, ac = gather_runs(keys, cnts)
            ix.griffin_merge_topk_device(world, nq, k, ak, ac, out_keys, out_cnts, stream)
        elif sharded:
            ak, ac, (lo, hi) = exchange_sliced(keys, cnts, k)
            if hi > lo:
                ix.griffin_merge_topk_device(world, hi - lo, k, ak, ac, out_keys, out_cnts, stream)

    for i in range(args.warmup):
        step_on(i)
    torch.cuda.synchronize()
    ix.griffin_sync_status()
    ix.griffin_reset_profile()
    ix.griffin_set_profiling(True)
    clocks = ClockSampler(dev)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    if len(slots) == 1:
        for i in range(args.steps):
            flush.fill_(i)                   # L2 flush between timed steps (outside events)
            ev[i][0].record(stream)
            step()
            ev[i][1].record(stream)
    else:
        # overlapped batches: one event pair around the whole region (start on the
        # first stream, end after every stream's last batch); no per-step flush —
        # the inputs (index >> L2) are larger than L2
        for _, st_, _, _ in slots[1:]:
            st_.wait_stream(stream)
        ev[0][0].record(stream)
        for i in range(args.steps):
            step_on(i)
        for _, st_, _, _ in slots[1:]:
            stream.wait_stream(st_)
        ev[0][1].record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    ix.griffin_set_profiling(False)
    prof = ix.griffin_get_profile()
    ix.griffin_sync_status()
    if len(slots) == 1:
        step_ms = [a.elapsed_time(b) for a, b in ev]
        total_ms = sum(step_ms)
    else:
        total_ms = ev[0][0].elapsed_time(ev[0][1])
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    # replicate: every rank answered its own full batch (weak scaling)
    qps = (world if replicate else 1) * nq * args.steps / (total_ms / 1e3)
    peak, peak_kind = _peaks()
    ms_x = prof["ms_intersect"]
    achieved = prof["alg_bytes"] / (ms_x / 1e3) / 1e9 if ms_x > 0 else 0.0
    ms_d = prof["ms_decode"]
    achieved_d = prof["dec_alg_bytes"] / (ms_d / 1e3) / 1e9 if ms_d > 0 else 0.0
    kernels = {
        "intersect_kernel": {
            "what": "fused EF decode + merge-path/gallop intersection + BM25 (all SvS rounds)",
            "ms_per_step": ms_x / args.steps, "launches": prof["launches_intersect"],
            "alg_bytes_per_launch": prof["alg_bytes"] / max(1, prof["launches_intersect"]),
            "achieved_gbs": achieved, "share_of_step": ms_x / total_ms if total_ms else None,
            "decoded_postings_per_step": prof["decoded_postings"] / args.steps},
        "decode_once_kernel": {
            "what": "batch decode-once: Para-EF decode of hot lists into the HBM arena",
            "ms_per_step": ms_d / args.steps, "launches": prof["launches_decode"],
            "alg_bytes_per_launch": prof["dec_alg_bytes"] / max(1, prof["launches_decode"]),
            "achieved_gbs": achieved_d, "share_of_step": ms_d / total_ms if total_ms else None,
            "decoded_postings_per_step": prof["dec_postings"] / args.steps},
    }
    dom = "intersect_kernel" if ms_x >= ms_d else "decode_once_kernel"
    kd = kernels[dom]
    roof = {"bound": "hbm", "kernel": dom, "achieved": kd["achieved_gbs"], "peak": peak,
            "unit": "GB/s", "frac": kd["achieved_gbs"] / peak if peak else None, "traffic": None,
            "peak_kind": peak_kind, "alg_bytes_per_launch": kd["alg_bytes_per_launch"],
            "ms_per_launch": kd["ms_per_step"] * args.steps / max(1, kd["launches"]),
            "share_of_step": kd["share_of_step"]}
    # per-GPU figures of this rank; the job aggregate for N ranks is N x (max-time) based
    decoded_ps = ((prof["decoded_postings"] + prof["dec_postings"]) / (total_ms / 1e3)
                  if total_ms > 0 else 0.0)

    # ---- e2e: the public host-buffer C-ABI call, H2D of the step's queries and
    # D2H of its results inside every timed step (wall clock, max over ranks)
    e2e_times = []
    if sharded:
        searcher = ShardedSearcher.from_index(ix)
    if world > 1:
        h_off = torch.from_numpy(ql.offsets.astype(np.int32)).pin_memory()
        h_terms = torch.from_numpy(ql.terms.astype(np.int32)).pin_memory()
    if not sharded:
        # griffin_query_batch split into submit/collect over the slots'
        # workspaces: the same host-buffer call with len(slots) batches in
        # flight (H2D of the queries, the path, D2H of the results per batch)
        # (slot 0 = the index's own workspace; no extra device memory)
        e2e_ws = [ix] + [sl[0] for sl in slots[1:]]
        e2e_st = [sl[1] for sl in slots]

        # results read in place from each slot's pinned staging (zero-copy views,
        # griffin_query_batch_results), valid until that slot's next submit
        e2e_out = ["view"] * len(e2e_ws)

        def e2e_run(n):
            nw = len(e2e_ws)
            for i in range(n):
                w = e2e_ws[i % nw]
                if i >= nw:
                    w.griffin_query_batch_collect(e2e_out[i % nw])
                w.griffin_query_batch_submit(ql.offsets, ql.terms, k, e2e_st[i % nw])
            for i in range(max(0, n - nw), n):
                e2e_ws[i % nw].griffin_query_batch_collect(e2e_out[i % nw])

        e2e_run(args.warmup)
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        e2e_run(args.steps)
        e2e_times.append(time.perf_counter() - t0)
    for i in range(args.warmup + args.steps if sharded else 0):
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        e_off = h_off.to("cuda", non_blocking=True)
        e_terms = h_terms.to("cuda", non_blocking=True)
        if args.exchange == "allgather":
            dd, ss, cc = searcher.search(e_off, e_terms, max_terms, k, stream)
        else:
            _, _, dd, ss, cc = searcher.search_sliced(e_off, e_terms, max_terms, k, stream)
        dd, ss, cc = dd.cpu(), ss.cpu(), cc.cpu()
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            e2e_times.append(dt)
    e2e_s = sum(e2e_times)
    if world > 1:
        t = torch.tensor([e2e_s], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_s = float(t.item())
    h2d = (nq + 1) * 4 + len(ql.terms) * 4
    d2h = nq * k * 8 + nq * 4
    if sharded and args.exchange == "sliced":   # each rank reads back its own slice
        d2h = -(-nq // world) * (k * 8 + 4)

    # ---- closed-loop single-query latency (griffin_query, one in flight)
    lat = []
    nlat = min(nq, args.latency_queries)
    for q in range(min(nlat, 64)):          # warm-up: capture the per-term-count graphs
        ix.griffin_query(ql.query(q), k)
    for q in range(nlat):
        t0 = time.perf_counter()
        ix.griffin_query(ql.query(q), k)
        lat.append((time.perf_counter() - t0) * 1e3)
    lat.sort()

    def pct(p):
        return lat[min(len(lat) - 1, int(np.ceil(p / 100 * len(lat))) - 1)] if lat else None

    line = {
        "metric": "queries/sec", "value": qps, "unit": "queries/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step,
        "higher_is_better": True, "scaling": "weak" if replicate else "strong",
        "vs_baseline": None, "dtype": "u32/f32", "data": "synthetic",
        "config": {"workload": WORKLOAD_DESC[args.config], "num_docs": corpus.num_docs,
                   "num_terms": corpus.num_terms, "num_postings": corpus.num_postings,
                   "queries_per_step": nq, "k": k, "block_size": B,
                   "l2": ("flushed between timed steps (256 MB write)" if len(slots) == 1 else
                          "inputs larger than L2 (index %.0f MB, L2 126 MB); not flushed" %
                          ((st["payload_bytes"] + st["skip_bytes"] + st["tf_bytes"]) / 1e6)),
                   "batches_in_flight": len(slots),
                   "parallelism": (f"docid-range shards x{world}, {args.exchange} exchange"
                                   if sharded else f"replicated index x{world}, no exchange"
                                   if replicate else "1 shard"),
                   "index_bytes_per_shard": st["payload_bytes"] + st["skip_bytes"] + st["tf_bytes"],
                   "index_build_s": build_s},
        "decoded_postings_per_s": decoded_ps * world,
        "reuse": "auto (decode-once of hot lists per batch)",
        "hbm_gbs": achieved,
        "latency_ms": {"p50": pct(50), "p99": pct(99), "queries": nlat,
                       "mode": "closed-loop griffin_query (host buffers), one in flight"},
        "roofline": roof,
        "kernels": kernels,
        "stage_ms_note": ("CUDA-event durations per stage summed over all launches; with "
                          "batches_in_flight > 1 the stages of different batches overlap"),
        "stage_ms_per_step": {kk: prof[kk] / args.steps for kk in
                              ("ms_plan", "ms_decode", "ms_intersect", "ms_compact", "ms_topk",
                               "ms_merge")},
        "gpu_launches": int(prof["launches_total"]),
        "e2e": {"value": (world if replicate else 1) * nq * args.steps / e2e_s,
                "unit": "queries/s", "h2d_bytes_per_step": h2d,
                "d2h_bytes_per_step": d2h,
                "how": ("griffin_query_batch_submit/collect (host buffers; pinned staging, H2D queries, "
                        "D2H results), batches_in_flight workspaces" if not sharded else
                        "ShardedSearcher.search (pinned H2D queries, D2H results)")},
        "clocks": clk,
    }
    # decode-only sweep over every block of the shard (SURVEY §8(d) C5 sweep row)
    sw = ix.griffin_debug_decode_all(iters=3)
    line["decode_sweep"] = {"ms": sw["ms"], "postings": sw["postings"], "bytes": sw["bytes"],
                            "gbs": sw["bytes"] / (sw["ms"] / 1e3) / 1e9,
                            "postings_per_s": sw["postings"] / (sw["ms"] / 1e3),
                            "frac_of_hbm_peak": sw["bytes"] / (sw["ms"] / 1e3) / 1e9 / peak}
    traffic = _ncu_traffic(args.config, dom)
    if traffic is not None:
        line["roofline"]["traffic"] = traffic
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        base, _, _ = oracle_baseline(corpus, ql, k, B, budget_s=args.cpu_budget)
        line["cpu_baseline"] = base
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def _ncu_traffic(config, kernel):
    """dram read+write bytes per launch of `kernel` from the committed ncu summary."""
    p = os.path.join(ROOT, "profiles", f"ncu_summary_{config}.json")
    if not os.path.exists(p):
        return None
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get("dram_bytes_per_launch", {}).get(kernel)
    except (OSError, ValueError):
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c2", choices=sorted(WORKLOAD_DESC))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--latency-queries", type=int, default=1000)
    ap.add_argument("--streams", type=int, default=None,
                    help="batches in flight on separate streams/workspaces (N=1 only); default "
                         "3 for the 1K-query configs, 2 for the 10K-query top-1000 batches "
                         "(three workspaces of those exceed HBM)")
    ap.add_argument("--shard-mode", default="docid", choices=["docid", "replicate"],
                    help="N>1: docID-range shards + exchange, or a replicated index per rank")
    ap.add_argument("--exchange", default="allgather", choices=["allgather", "sliced"],
                    help="docid shards: all-gather of per-shard top-k, or query-sliced all-to-all")
    ap.add_argument("--cpu-budget", type=float, default=12.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.streams is None:
        args.streams = 2 if args.config in ("c4", "c5") else 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_gpu(args)


if __name__ == "__main__":
    main()
