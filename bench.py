#!/usr/bin/env python
"""Benchmark of the B200 Griffin-GPU conjunctive query path.

One "step" = one pass of the whole hot path (plus a8 for
N > 1) over one batch of queries with the query log resident in HBM.  Default
workload: BASELINE.json configs[4] (C5) — the 50M-doc ClueWeb-shaped synthetic
index (EF blocks of 128, ~1.9 B postings) and a batch of 10K concurrent 2-5
term queries, BM25 top-1000 — the largest single-GPU configuration.  The timed
loop rotates through the config's distinct query batches (3 by default).
Prints ONE JSON line.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c5] [--impl reference]

Measurements on the same line:
  value       queries/s, batches pipelined over --streams workspaces (device API)
  roofline    the dominant kernel's §8(d) algorithmic bytes per launch / its
              ISOLATED launch duration (one batch in flight, profiling pass,
              CUDA events on the launching stream), vs the measured HBM peak;
              traffic = ncu DRAM bytes per launch from profiles/
  sync_qps    §8(d)'s definition: batch / median wall time of one synchronous
              griffin_query_batch call (host buffers, H2D + D2H inside)
  e2e         the same metric through the host-buffer C ABI, pipelined
  parity      the last timed batch vs the CPU oracle on the cpu_baseline sample
N > 1 is launched by torchrun (one process per GPU): each rank holds one
docID-range shard; per-shard top-k keys are all-gathered over NCCL and merged by
the library's k-way merge kernel.  The reference arm (--impl reference) times
the CPU oracle (the test oracle, as it stands) on a bounded sample of the same
workload; there is no installable reference code (PAPER.md only).
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
    "c2": "C2: 10M-doc synthetic Zipf index (alpha 0.8, df 1K..5M, 42K terms, 0.19B postings), 1000-query 2-5 term batches, EF block 128, BM25 top-10",
    "c3": "C3: GOV2-shaped 25M-doc synthetic Zipf index (df up to 10M), 1000-query log, BM25 top-10",
    "c4": "C4: ClueWeb-shaped 50M-doc synthetic Zipf index (alpha 0.8, df 1K..30M, 395K terms, 1.9B postings), 10K-query batches, EF block 128, BM25 top-10",
    "c5": "C5: ClueWeb-shaped 50M-doc synthetic Zipf index (alpha 0.8, df 1K..30M, 395K terms, 1.9B postings), 10K concurrent 2-5 term queries per batch, EF block 128, BM25 top-1000",
}


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, STREAM copy)"
    return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """SM clock + throttle reasons sampled during the timed region: NVML in a
    background thread every 2 ms, with nvidia-smi as a fallback."""

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


def load_workload(name):
    """(corpus, [batch query logs], cfg); large corpora come from the
    on-disk synth cache (generated once, memory-mapped by every rank)."""
    from synth import batch_of, make_workload
    corpus, ql, cfg = make_workload(name)
    batches = [batch_of(ql, cfg, i) for i in range(cfg.get("batches", 1))]
    return corpus, batches, cfg


def _parallelism(args):
    if args.gpus <= 1:
        return "1 shard"
    if args.shard_mode == "replicate":
        return f"replicated index x{args.gpus}, no exchange"
    return f"docid-range shards x{args.gpus}, {args.exchange} exchange ({args.dist_backend})"


def config_dict(args, corpus, cfg, nq, extra=None):
    """The `config` object, identical on both arms (ours and --impl reference)."""
    d = {"workload": WORKLOAD_DESC[args.config], "num_docs": corpus.num_docs,
         "num_terms": corpus.num_terms, "num_postings": corpus.num_postings,
         "queries_per_step": nq, "k": cfg["k"], "block_size": cfg["block"],
         "batches_rotated": cfg.get("batches", 1),
         "l2": "inputs larger than L2 (index > 126 MB L2, rotating query batches)",
         "parallelism": _parallelism(args)}
    if extra:
        d.update(extra)
    return d


class OracleSample:
    """The CPU oracle (tests' checker, as it stands) over the lists of a bounded
    sample of one batch: timed as the cpu_baseline / reference arm, and its
    answers are the parity reference for the same queries on the GPU."""

    def __init__(self, corpus, batch, k, block, budget_s, threads=None):
        import oracle
        from synth import sub_corpus
        self.cores, self.model = _cpu_info()
        self.threads = threads or self.cores
        self.k = k
        # grow the sample until one pass costs ~budget/3 (bounded CPU work)
        m = min(batch.num_queries, max(self.threads, 16))
        while True:
            sub = batch.slice(0, m)
            t0 = time.time()
            ox = oracle.OracleIndex(sub_corpus(corpus, sub.terms), block_size=block)
            self.build_s = time.time() - t0
            t0 = time.perf_counter()
            res = ox.query_batch(sub, k, nthreads=self.threads)
            dt = time.perf_counter() - t0
            if dt >= budget_s / 3 or m >= batch.num_queries:
                break
            m = min(batch.num_queries, int(m * max(2.0, budget_s / 3 / max(dt, 1e-3))))
        self.ox, self.sub, self.m, self.res, self.dt = ox, sub, m, res, dt

    def run(self):
        t0 = time.perf_counter()
        self.res = self.ox.query_batch(self.sub, self.k, nthreads=self.threads)
        return time.perf_counter() - t0

    def baseline(self, value, nq_batch):
        return {"value": value, "unit": "queries/s", "cores": self.threads, "kind": "oracle",
                "sample": f"first {self.m} of a {nq_batch}-query batch, {self.threads} std::threads "
                          f"round-robin; oracle indexes only the sample's lists (same N, dl, df) "
                          f"in {self.build_s:.1f}s, not timed",
                "cpu_model": self.model}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    corpus, batches, cfg = load_workload(args.config)
    k = cfg["k"]
    last = batches[(args.steps - 1) % len(batches)]
    osm = OracleSample(corpus, last, k, cfg["block"], budget_s=args.cpu_budget)
    for _ in range(args.warmup):
        osm.run()
    times = [osm.run() for _ in range(args.steps)]
    ms = 1e3 * statistics.mean(times)
    qps = osm.m / (ms / 1e3)
    line = {"impl": "reference", "metric": "queries/sec", "value": qps, "unit": "queries/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "u32/f32", "data": "synthetic",
            "config": config_dict(args, corpus, cfg, last.num_queries),
            "cpu_baseline": osm.baseline(qps, last.num_queries),
            "e2e": {"value": qps, "unit": "queries/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    line["cpu_baseline"]["queries_per_step_timed"] = osm.m
    print(json.dumps(line), flush=True)


def _keys_to_rows(keys, counts, nq, k):
    """(score desc, docID asc) rows from the library's u64 keys (host, for the
    parity check): key = f32 score bits << 32 | (0xFFFFFFFF - docID)."""
    kk = keys.view(np.uint64).reshape(nq, k)
    d = (np.uint64(0xFFFFFFFF) - (kk & np.uint64(0xFFFFFFFF))).astype(np.uint32)
    s = (kk >> np.uint64(32)).astype(np.uint32).view(np.float32)
    c = counts.view(np.uint32)[:nq]
    valid = np.arange(k)[None, :] < c[:, None]
    d = np.where(valid, d, np.uint32(0xFFFFFFFF))
    s = np.where(valid, s, np.float32(-np.inf))
    return d, s, c


def run_gpu(args):
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_0044ws18_b200 as g
    from paper_conf_ppopp_0044ws18_b200.sharded import exchange_sliced, gather_runs

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        # gloo (a dry run of the N>1 path on fewer GPUs than ranks): ranks share devices
        local = local % torch.cuda.device_count() if args.dist_backend == "gloo" else local
        torch.cuda.set_device(local)
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group("gloo")
    else:
        torch.cuda.set_device(0)
    dev = torch.cuda.current_device()
    t0 = time.time()
    corpus, batches, cfg = load_workload(args.config)
    gen_s = time.time() - t0
    k, B = cfg["k"], cfg["block"]
    NB = len(batches)
    nq = batches[0].num_queries
    # docid: rank r holds docID-range shard r, per-shard top-k exchanged (all-gather
    # or query-sliced all-to-all) and merged; replicate: every
    # rank holds the whole index and answers its own batches, no exchange
    replicate = world > 1 and args.shard_mode == "replicate"
    sharded = world > 1 and not replicate
    t0 = time.time()
    ix = g.GriffinIndex(corpus, block_size=B, device=dev, shard_index=rank if sharded else 0,
                        num_shards=world if sharded else 1)
    build_s = time.time() - t0
    st = ix.griffin_index_stats()
    ix.griffin_set_reuse({"auto": 2, "on": 1, "off": 0}[args.reuse])
    ix.griffin_set_bitmap(args.bitmap)
    if args.probe_chunk:
        ix.griffin_set_probe_chunk(args.probe_chunk)
    # intermediate capacity per workspace buffer: packed by actual survivors, so a
    # budget well under the sum of per-query bounds holds a batch (C5: ~1e9 bound)
    budget = args.entry_budget if args.entry_budget is not None else \
        (400_000_000 if args.config in ("c4", "c5") else 0)
    ix.griffin_set_entry_budget(budget)
    stream = torch.cuda.current_stream()
    dq = []   # per batch: (d_off, d_terms, max_terms)
    for b in batches:
        ix.griffin_reserve(b.offsets, b.terms, k)
        mt = int(max(len(set(b.query(q).tolist())) for q in range(b.num_queries)))
        dq.append((torch.from_numpy(b.offsets.astype(np.int32)).cuda(),
                   torch.from_numpy(b.terms.astype(np.int32)).cuda(), mt))
    nstreams = max(1, args.streams) if not sharded else 1
    slots = [(None, stream, torch.zeros(nq * k, dtype=torch.int64, device="cuda"),
              torch.zeros(nq, dtype=torch.int32, device="cuda"))]
    for _ in range(nstreams - 1):
        w = ix.griffin_workspace_create()
        for b in batches:
            w.griffin_workspace_reserve(b.offsets, b.terms, k)
        slots.append((w, torch.cuda.Stream(), torch.zeros(nq * k, dtype=torch.int64, device="cuda"),
                      torch.zeros(nq, dtype=torch.int32, device="cuda")))
    if sharded:
        out_keys = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
        out_cnts = torch.zeros(nq, dtype=torch.int32, device="cuda")
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device="cuda")  # 256 MB > L2

    def step_on(i):
        w, st_, kk_, cc_ = slots[i % len(slots)]
        d_off, d_t, mt = dq[i % NB]
        if w is None:
            ix.griffin_query_batch_device(d_off, d_t, mt, k, kk_, cc_, st_)
        else:
            w.griffin_query_batch_device_ws(d_off, d_t, mt, k, kk_, cc_, st_)
        if sharded and args.exchange == "allgather":   # a8: all-gather + k-way merge (NCCL)
            ak, ac = gather_runs(kk_, cc_)
            ix.griffin_merge_topk_device(world, nq, k, ak, ac, out_keys, out_cnts, st_)
        elif sharded:   # NEXT-2: query-sliced all-to-all, this rank merges its slice
            ak, ac, (lo, hi) = exchange_sliced(kk_, cc_, k)
            if hi > lo:
                ix.griffin_merge_topk_device(world, hi - lo, k, ak, ac, out_keys, out_cnts, st_)

    for i in range(args.warmup):
        step_on(i)
    torch.cuda.synchronize()
    ix.griffin_sync_status()
    for w, _, _, _ in slots[1:]:
        w.griffin_workspace_sync_status()
    ix.griffin_reset_profile()

    # ---- timed region: batches pipelined over the slots (rotating batches) ----
    clocks = ClockSampler(dev)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    for _, st_, _, _ in slots[1:]:
        st_.wait_stream(stream)
    ev0.record(stream)
    for i in range(args.steps):
        step_on(i)
    for _, st_, _, _ in slots[1:]:
        stream.wait_stream(st_)
    ev1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    total_ms = ev0.elapsed_time(ev1)
    launches = int(ix.griffin_get_profile()["launches_total"])
    ix.griffin_sync_status()
    for w, _, _, _ in slots[1:]:
        w.griffin_workspace_sync_status()
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    qps = (world if replicate else 1) * nq * args.steps / (total_ms / 1e3)
    # results of the last timed step (its slot's outputs are untouched since)
    last_i = args.steps - 1
    _, _, lk, lc = slots[last_i % len(slots)]
    if sharded and args.exchange == "allgather":
        lk, lc = out_keys, out_cnts
    last_keys, last_cnts = lk.cpu().numpy(), lc.cpu().numpy()
    last_batch = batches[last_i % NB]

    # ---- isolated pass: one batch at a time, L2 flushed between, per-stage
    # CUDA events on the launching stream -> per-kernel durations ----
    n_iso = max(NB, min(args.steps, 2 * NB))
    ix.griffin_reset_profile()
    ix.griffin_set_profiling(2)            # stage events only (no counting work)
    iso = []
    for i in range(n_iso):
        flush.fill_(i)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        d_off, d_t, mt = dq[i % NB]
        ix.griffin_query_batch_device(d_off, d_t, mt, k, slots[0][2], slots[0][3], stream)
        e1.record(stream)
        torch.cuda.synchronize()
        iso.append(e0.elapsed_time(e1))
    ix.griffin_set_profiling(False)
    prof = ix.griffin_get_profile()
    # counting pass (algorithmic bytes, postings, survivors), not timed
    ix.griffin_reset_profile()
    ix.griffin_set_profiling(3)
    for i in range(n_iso):
        d_off, d_t, mt = dq[i % NB]
        ix.griffin_query_batch_device(d_off, d_t, mt, k, slots[0][2], slots[0][3], stream)
    torch.cuda.synchronize()
    ix.griffin_set_profiling(False)
    cnt = ix.griffin_get_profile()
    for kk in ("alg_bytes", "c8d_bytes", "payload_bytes", "decoded_postings", "survivors",
               "dec_alg_bytes", "dec_c8d_bytes", "dec_postings", "arena_postings", "merge_units",
               "merge_elems", "gallop_units", "gallop_elems", "bitmap_units", "bitmap_elems", "bitand_units", "bitand_words"):
        prof[kk] = cnt[kk]
    ix.griffin_sync_status()
    iso_ms = sum(iso)
    peak, peak_kind = _peaks()

    def kern(ms, alg, c8d, launches_, post, what):
        per = max(1, launches_)
        return {"what": what, "ms_per_step": ms / n_iso, "launches_per_step": launches_ / n_iso,
                "ms_per_launch": ms / per, "share_of_step": ms / iso_ms if iso_ms else None,
                "alg_bytes_per_launch": c8d / per, "all_bytes_per_launch": alg / per,
                "achieved_gbs": (c8d / per) / (ms / per / 1e3) / 1e9 if ms > 0 else 0.0,
                "achieved_all_bytes_gbs": (alg / per) / (ms / per / 1e3) / 1e9 if ms > 0 else 0.0,
                "decoded_postings_per_step": post / n_iso,
                "survivors_per_step": None}

    kernels = {
        "intersect_kernel": kern(prof["ms_intersect"], prof["alg_bytes"], prof["c8d_bytes"],
                                 prof["launches_intersect"], prof["decoded_postings"],
                                 "SvS rounds: intersect_kernel (round 1: fused EF decode / arena tiles + "
                                 "merge-path, gallop or bitvector-lookup intersection + BM25) and probe_kernel (rounds "
                                 "2..m-1 as one multi-list probe pass)"),
        "decode_once_kernel": kern(prof["ms_decode"], prof["dec_alg_bytes"],
                                   prof["dec_c8d_bytes"], prof["launches_decode"],
                                   prof["dec_postings"],
                                   "batch decode-once: Para-EF decode of hot lists into the HBM arena "
                                   "(dense lists into a bitvector + rank)"),
    }
    kernels["intersect_kernel"]["survivors_per_step"] = prof["survivors"] / n_iso
    kernels["intersect_kernel"]["arena_postings_per_step"] = prof["arena_postings"] / n_iso
    kernels["intersect_kernel"]["units_per_step"] = {
        kk: prof[kk] / n_iso for kk in ("merge_units", "merge_elems", "gallop_units", "gallop_elems",
                                        "bitmap_units", "bitmap_elems", "bitand_units",
                                        "bitand_words")}
    stage_ms = {kk: prof[kk] / n_iso for kk in
                ("ms_plan", "ms_decode", "ms_intersect", "ms_compact", "ms_topk", "ms_merge")}
    dom = max(kernels, key=lambda n: kernels[n]["ms_per_step"])
    kd = kernels[dom]
    traffic = _ncu_traffic(args.config, dom)
    roof = {"bound": "hbm", "kernel": dom, "achieved": kd["achieved_gbs"], "peak": peak,
            "unit": "GB/s", "frac": kd["achieved_gbs"] / peak, "traffic": traffic,
            "peak_kind": peak_kind,
            "numerator": ("SURVEY §8(d) algorithmic bytes per launch (compressed payload + 8 B skip/meta "
                          "of every block the method reads, decoded-arena postings charged at their "
                          "compressed size, 8 B per intermediate entry, tf sector + norm per survivor)"),
            "alg_bytes_per_launch": kd["alg_bytes_per_launch"],
            "achieved_all_bytes": kd["achieved_all_bytes_gbs"],
            "frac_all_bytes": kd["achieved_all_bytes_gbs"] / peak,
            "all_bytes_per_launch": kd["all_bytes_per_launch"],
            "ms_per_launch": kd["ms_per_launch"], "share_of_step": kd["share_of_step"],
            "timing": (f"isolated: {n_iso} batches one at a time, 256 MB L2 flush between, "
                       "per-stage CUDA events on the launching stream (no counting work); bytes "
                       "from a separate counting pass over the same batches")}
    decoded_ps = (prof["decoded_postings"] + prof["dec_postings"]) / (iso_ms / 1e3) if iso_ms else 0.0

    # ---- §8(d) QPS: median wall time of one synchronous griffin_query_batch ----
    sync_ms = []
    if world == 1:
        sync_out = (np.zeros(nq * k, np.uint32), np.zeros(nq * k, np.float32), np.zeros(nq, np.uint32))
        for i in range(2 + max(5, NB)):
            b = batches[i % NB]
            t0 = time.perf_counter()
            ix.griffin_query_batch(b.offsets, b.terms, k, out=sync_out)
            if i >= 2:
                sync_ms.append((time.perf_counter() - t0) * 1e3)

    # ---- e2e: host-buffer C ABI, pipelined submit/collect over the slots ----
    e2e_s = None
    h2d = (nq + 1) * 4 + int(np.mean([len(b.terms) for b in batches])) * 4
    d2h = nq * k * 8 + nq * 4
    if sharded and args.exchange == "sliced":   # each rank reads back its own slice
        d2h = -(-nq // world) * (k * 8 + 4)
    if not sharded:
        e2e_ws = [ix] + [sl[0] for sl in slots[1:]]
        e2e_st = [sl[1] for sl in slots]

        def e2e_run(n):
            nw = len(e2e_ws)
            for i in range(n):
                w = e2e_ws[i % nw]
                if i >= nw:
                    w.griffin_query_batch_collect("view")
                b = batches[i % NB]
                w.griffin_query_batch_submit(b.offsets, b.terms, k, e2e_st[i % nw])
            for i in range(max(0, n - nw), n):
                e2e_ws[i % nw].griffin_query_batch_collect("view")

        e2e_run(args.warmup)
        t0 = time.perf_counter()
        e2e_run(args.steps)
        e2e_s = time.perf_counter() - t0
    else:
        from paper_conf_ppopp_0044ws18_b200.sharded import ShardedSearcher
        searcher = ShardedSearcher.from_index(ix)
        times = []
        for i in range(args.warmup + args.steps):
            b = batches[i % NB]
            h_off = torch.from_numpy(b.offsets.astype(np.int32)).pin_memory()
            h_t = torch.from_numpy(b.terms.astype(np.int32)).pin_memory()
            dist.barrier()
            t0 = time.perf_counter()
            if args.exchange == "allgather":
                dd, ss, cc = searcher.search(h_off.to("cuda", non_blocking=True),
                                             h_t.to("cuda", non_blocking=True), dq[i % NB][2], k,
                                             stream)
            else:
                _, _, dd, ss, cc = searcher.search_sliced(h_off.to("cuda", non_blocking=True),
                                                          h_t.to("cuda", non_blocking=True),
                                                          dq[i % NB][2], k, stream)
            dd, ss, cc = dd.cpu(), ss.cpu(), cc.cpu()
            if i >= args.warmup:
                times.append(time.perf_counter() - t0)
        e2e_s = sum(times)
    if world > 1:
        t = torch.tensor([e2e_s], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_s = float(t.item())

    # ---- closed-loop single-query latency (griffin_query, one in flight) ----
    lat = []
    if world == 1:
        b0 = batches[0]
        nlat = min(b0.num_queries, args.latency_queries)
        for q in range(min(nlat, 64)):          # warm-up: capture the per-term-count graphs
            ix.griffin_query(b0.query(q), k)
        for q in range(nlat):
            t0 = time.perf_counter()
            ix.griffin_query(b0.query(q), k)
            lat.append((time.perf_counter() - t0) * 1e3)
        lat.sort()

    def pct(p):
        return lat[min(len(lat) - 1, int(np.ceil(p / 100 * len(lat))) - 1)] if lat else None

    sw = ix.griffin_debug_decode_all(iters=3)
    line = {
        "metric": "queries/sec", "value": qps, "unit": "queries/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step,
        "higher_is_better": True, "scaling": "weak" if replicate else "strong", "vs_baseline": None,
        "dtype": "u32/f32", "data": "synthetic",
        "config": config_dict(args, corpus, cfg, nq),
        "batches_in_flight": len(slots),
        "index": {"bytes_per_shard": st["payload_bytes"] + st["skip_bytes"] + st["tf_bytes"],
                  "payload_bytes": st["payload_bytes"], "build_s": build_s,
                  "corpus_load_s": gen_s, "reuse": args.reuse, "bitmap_inv": args.bitmap,
                  "entry_budget": budget},
        "decoded_postings_per_s": decoded_ps * world,
        "sync_qps": {"value": nq / (statistics.median(sync_ms) / 1e3) if sync_ms else None,
                     "unit": "queries/s", "median_ms": statistics.median(sync_ms) if sync_ms else None,
                     "calls": len(sync_ms),
                     "how": "SURVEY §8(d): batch size / median wall time of one synchronous "
                            "griffin_query_batch (host buffers, H2D + D2H inside; the caller's "
                            "output arrays reused across calls), rotating batches"},
        "latency_ms": {"p50": pct(50), "p99": pct(99), "queries": len(lat),
                       "mode": "closed-loop griffin_query (host buffers), one in flight"},
        "roofline": roof,
        "kernels": kernels,
        "stage_ms_per_step_isolated": stage_ms,
        "isolated_ms_per_step": iso_ms / n_iso,
        "gpu_launches": launches,
        "e2e": {"value": nq * args.steps / e2e_s if e2e_s else None, "unit": "queries/s",
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "how": ("griffin_query_batch_submit/collect (host buffers; pinned staging, H2D queries, "
                        "D2H results read in place), batches_in_flight workspaces, rotating batches"
                        if not sharded else "ShardedSearcher.search (pinned H2D queries, D2H results)")},
        "clocks": clk,
        "decode_sweep": {"ms": sw["ms"], "postings": sw["postings"], "bytes": sw["bytes"],
                         "gbs": sw["bytes"] / (sw["ms"] / 1e3) / 1e9,
                         "postings_per_s": sw["postings"] / (sw["ms"] / 1e3),
                         "frac_of_hbm_peak": sw["bytes"] / (sw["ms"] / 1e3) / 1e9 / peak,
                         "alu_roofline": _sweep_alu(sw["postings"] / (sw["ms"] / 1e3)),
                         "note": "every block of the shard decoded once per launch; the index "
                                 "(> L2) is streamed from HBM"},
    }
    if rank == 0 and not args.no_cpu_baseline and not (sharded and args.exchange == "sliced"):
        # oracle on a bounded sample of the LAST timed batch: the cpu_baseline,
        # and the parity reference for the same queries of the GPU's results
        osm = OracleSample(corpus, last_batch, k, B, budget_s=args.cpu_budget)
        dt = osm.run()
        line["cpu_baseline"] = osm.baseline(osm.m / dt, nq)
        gd, gs, gc = _keys_to_rows(last_keys, last_cnts, nq, k)
        od, os_, oc = osm.res
        m = osm.m
        ok_c = np.array_equal(gc[:m], oc)
        ok_d = np.array_equal(gd[:m], od)
        ok_s = np.array_equal(gs[:m].view(np.uint32), os_.view(np.uint32))
        line["parity"] = {"queries_checked": m, "of": nq, "batch": last_i % NB,
                          "bit_exact": bool(ok_c and ok_d and ok_s),
                          "what": "last timed step's top-k (docIDs, order, score bits, counts) "
                                  "vs the CPU oracle on the same queries"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


# Warp instructions the run decoder issues per posting: ncu --set full of the
# decode-only sweep (C2 index, B = 128): 1.48e8 warp instructions for 192,979,545
# postings (profiles/r02s11_decode_sweep_ncu_kernels.txt).
SWEEP_WARP_INST_PER_POSTING = 1.48e8 / 192979545


def _sweep_alu(postings_per_s):
    """The decode sweep against its issue roofline (it is integer-ALU / issue
    bound, not HBM bound): achieved warp-instruction rate = postings/s x the
    ncu-measured instructions per posting; peak = SMs x 4 schedulers x the max
    SM clock (one warp instruction per scheduler per cycle)."""
    try:
        import torch
        sms = torch.cuda.get_device_properties(0).multi_processor_count
    except Exception:   # no device visible: the B200's count
        sms = 148
    mhz = 1965.0
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            mhz = float(json.load(f).get("sm_max_mhz", mhz))
    except (OSError, ValueError):
        pass
    peak = sms * 4 * mhz * 1e6
    ach = postings_per_s * SWEEP_WARP_INST_PER_POSTING
    return {"bound": "alu", "unit": "warp instructions/s", "achieved": ach, "peak": peak,
            "frac": ach / peak, "warp_inst_per_posting": SWEEP_WARP_INST_PER_POSTING,
            "peak_how": f"{sms} SMs x 4 schedulers x {mhz:.0f} MHz"}


def _ncu_traffic(config, kernel):
    """ncu dram read+write bytes per launch of `kernel` from the committed summary."""
    p = os.path.join(ROOT, "profiles", f"ncu_summary_{config}.json")
    if not os.path.exists(p):
        return None
    try:
        with open(p) as f:
            d = json.load(f)
        v = d.get("dram_bytes_per_launch", {}).get(kernel)
        return v if v else None
    except (OSError, ValueError):
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c5", choices=sorted(WORKLOAD_DESC))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--latency-queries", type=int, default=1000)
    ap.add_argument("--streams", type=int, default=None,
                    help="batches in flight on separate streams/workspaces (N=1 only); default 3")
    ap.add_argument("--reuse", default="auto", choices=["auto", "on", "off"],
                    help="batch decode-once of hot lists into an HBM arena")
    ap.add_argument("--bitmap", type=int, default=32,
                    help="dense lists (density >= 1/INV) decoded once per batch into a bitvector; 0 = off")
    ap.add_argument("--probe-chunk", type=int, default=0,
                    help="probe-pass survivors per unit (0 = library default)")
    ap.add_argument("--shard-mode", default="docid", choices=["docid", "replicate"],
                    help="N>1: docID-range shards + exchange, or a replicated index per rank")
    ap.add_argument("--exchange", default="allgather", choices=["allgather", "sliced"],
                    help="docid shards: all-gather of per-shard top-k, or query-sliced all-to-all")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="N>1 process group; gloo lets ranks share a GPU (dry runs)")
    ap.add_argument("--entry-budget", type=int, default=None,
                    help="intermediate entries per workspace buffer (0 = exact bound); "
                         "default 4e8 for c4/c5, else 0")
    ap.add_argument("--cpu-budget", type=float, default=12.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.streams is None:
        args.streams = 3
    args.gpus = int(os.environ.get("WORLD_SIZE", args.gpus))
    if args.impl == "reference":
        run_reference(args)
    else:
        run_gpu(args)


if __name__ == "__main__":
    main()
