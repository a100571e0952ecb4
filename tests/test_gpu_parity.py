"""Parity of the CUDA path (through the C ABI) against the CPU oracle.

Bar (BASELINE.json north_star): docID sets and top-k ordering bit-exact with ties
by docID; BM25 scores within 1e-5 relative — in practice bit-identical, which is
what these tests require (same f32 op order on both sides)."""
import os

import numpy as np
import pytest

import oracle
import paper_conf_ppopp_0044ws18_b200 as g
from helpers import corpus_from_lists, random_corpus, random_queries
from synth import QueryLog, batch_of, make_pair_workload, make_workload, sub_corpus

pytestmark = pytest.mark.gpu


def _bits(a):
    return np.asarray(a, np.float32).view(np.uint32)


def assert_topk_equal(gd, gs, gc, od, os_, oc, rel=1e-5):
    assert np.array_equal(np.asarray(gc), np.asarray(oc)), "counts differ"
    assert np.array_equal(gd, od), "docIDs / order differ"
    fin = np.isfinite(os_)
    assert np.array_equal(np.isfinite(gs), fin)
    assert np.all(np.abs(gs[fin] - os_[fin]) <= rel * np.abs(os_[fin]))
    # the f32 op order is identical on both sides: expect identical bits
    assert np.array_equal(_bits(gs), _bits(os_)), "scores not bit-identical"


@pytest.fixture(scope="module")
def tiny():
    c, ql, cfg = make_workload("tiny")
    return c, ql, oracle.OracleIndex(c, block_size=128)


@pytest.fixture(scope="module")
def tiny_gpu(tiny):
    return g.GriffinIndex(tiny[0], block_size=128)


# ---------------------------------------------------------------- codec

@pytest.mark.parametrize("B", [64, 128, 256, 512])
def test_encoder_logical_streams_match_oracle(B):
    c, ql, _ = make_workload("tiny")
    ox = oracle.OracleIndex(c, block_size=B)
    gx = g.GriffinIndex(c, block_size=B)
    rng = np.random.default_rng(B)
    terms = list(range(0, 12)) + rng.integers(0, c.num_terms, 40).tolist()
    for t in terms:
        nb = ox.num_blocks(t)
        for blk in range(nb):
            o = ox.block_streams(t, blk)
            gg = gx.griffin_debug_block_streams(t, blk)
            assert o[0] == gg[0] and o[1] == gg[1] and o[2] == gg[2]
            assert o[4] == gg[4] and np.array_equal(o[3], gg[3])
            assert o[6] == gg[6] and np.array_equal(o[5], gg[5])


@pytest.mark.parametrize("B", [64, 96, 128, 256, 512])
def test_decode_list_roundtrip(B):
    c, ql, _ = make_workload("tiny")
    gx = g.GriffinIndex(c, block_size=B)
    for t in range(c.num_terms):
        assert np.array_equal(gx.griffin_debug_decode_list(t), c.list(t)), t


def test_decode_edge_lists():
    N = 5_000_000
    lists = [np.array([0]), np.array([N - 1]), np.array([0, N - 1]), np.arange(1000, 1000 + 777),
             np.arange(0, N, 4999), np.array([3, 4, 5, 1 << 20, (1 << 20) + 1])]
    c = corpus_from_lists(N, lists, doc_lengths=np.full(N, 7, np.uint32))
    for B in (64, 512):
        gx = g.GriffinIndex(c, block_size=B)
        for t in range(len(lists)):
            assert np.array_equal(gx.griffin_debug_decode_list(t), c.list(t))


def test_decode_all_checksum(tiny, tiny_gpu):
    c = tiny[0]
    r = tiny_gpu.griffin_debug_decode_all(iters=2)
    assert r["postings"] == c.num_postings
    assert r["checksum"] == int(np.bitwise_xor.reduce(c.docids.astype(np.uint64)))


# ---------------------------------------------------------------- intersection

@pytest.mark.parametrize("mode", [g.MODE_AUTO, g.MODE_MERGE, g.MODE_GALLOP])
def test_intersect_sets_match_oracle(tiny, tiny_gpu, mode):
    c, ql, ox = tiny
    for q in range(ql.num_queries):
        terms = ql.query(q)
        want = ox.intersect(terms)
        got = tiny_gpu.griffin_debug_intersect(terms, mode)
        assert np.array_equal(got, want), (q, terms, len(got), len(want))


@pytest.mark.parametrize("mode", [g.MODE_MERGE, g.MODE_GALLOP])
def test_intersect_random_small_corpora(mode):
    rng = np.random.default_rng(11 + mode)
    for trial in range(6):
        c = random_corpus(rng, num_docs=int(rng.integers(500, 60_000)), num_terms=8, max_df=20_000)
        ox = oracle.OracleIndex(c, block_size=128)
        gx = g.GriffinIndex(c, block_size=int(rng.choice([64, 128, 256])))
        for _ in range(12):
            terms = rng.integers(0, c.num_terms, size=int(rng.integers(1, 6)))
            assert np.array_equal(gx.griffin_debug_intersect(terms, mode), ox.intersect(terms))


def test_ratio_pairs_all_modes_agree():
    """Skewed pairs (G6): merge, gallop and auto give the oracle's set."""
    c, ql = make_pair_workload(3_000_000, 200_000, [1, 3, 16, 100, 300, 1000, 5000], seed=77)
    ox = oracle.OracleIndex(c)
    gx = g.GriffinIndex(c)
    for q in range(ql.num_queries):
        want = ox.intersect(ql.query(q))
        for mode in (g.MODE_AUTO, g.MODE_MERGE, g.MODE_GALLOP):
            assert np.array_equal(gx.griffin_debug_intersect(ql.query(q), mode), want)


# ---------------------------------------------------------------- end to end

@pytest.mark.parametrize("k", [1, 10, 1000])
def test_query_batch_bit_exact(tiny, tiny_gpu, k):
    c, ql, ox = tiny
    od, os_, oc = ox.query_batch(ql, k)
    gd, gs, gc = tiny_gpu.griffin_query_batch(ql.offsets, ql.terms, k)
    assert_topk_equal(gd, gs, gc, od, os_, oc)


@pytest.mark.parametrize("mode", [g.MODE_MERGE, g.MODE_GALLOP])
def test_query_batch_forced_modes(tiny, mode):
    c, ql, ox = tiny
    gx = g.GriffinIndex(c, block_size=128)
    gx.griffin_set_mode(mode)
    od, os_, oc = ox.query_batch(ql, 10)
    gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, 10)
    assert_topk_equal(gd, gs, gc, od, os_, oc)


@pytest.mark.parametrize("chunk", [32, 64, 96])
def test_probe_chunk_sizes(tiny, chunk):
    """Probe-pass units of `chunk` survivors give the same results (incl. the
    single-query graph path, whose capture bakes the option in)."""
    c, ql, ox = tiny
    gx = g.GriffinIndex(c, block_size=128)
    gx.griffin_set_probe_chunk(chunk)
    od, os_, oc = ox.query_batch(ql, 10)
    gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, 10)
    assert_topk_equal(gd, gs, gc, od, os_, oc)
    for q in range(min(ql.num_queries, 8)):
        d1, s1, c1 = ox.query(ql.query(q), 10)
        d2, s2, c2 = gx.griffin_query(ql.query(q), 10)
        assert_topk_equal(d2, s2, c2, d1, s1, c1)
    with pytest.raises(Exception):
        gx.griffin_set_probe_chunk(48)


def test_c1_single_query():
    c, ql, cfg = make_workload("c1")
    ox = oracle.OracleIndex(c, block_size=128)
    gx = g.GriffinIndex(c, block_size=128)
    od, os_, oc = ox.query(ql.query(0), 10)
    gd, gs, gc = gx.griffin_query(ql.query(0), 10)
    assert oc > 0
    assert_topk_equal(gd, gs, gc, od, os_, oc)


def test_large_result_radix_select_path():
    """> 4096 survivors per query exercises the radix-select top-k."""
    rng = np.random.default_rng(21)
    N = 200_000
    lists = [np.sort(rng.choice(N, size=n, replace=False)) for n in (120_000, 150_000, 90_000, 5)]
    tfs = [rng.integers(1, 30, size=len(l)) for l in lists]
    c = corpus_from_lists(N, lists, tfs, rng.integers(1, 3000, size=N))
    ox = oracle.OracleIndex(c)
    gx = g.GriffinIndex(c)
    qs = [[0, 1], [0, 1, 2], [2], [0], [3, 0]]
    ql = QueryLog(offsets=np.cumsum([0] + [len(q) for q in qs]).astype(np.uint32),
                  terms=np.concatenate(qs).astype(np.uint32))
    for k in (10, 4096):
        od, os_, oc = ox.query_batch(ql, k)
        gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
        assert_topk_equal(gd, gs, gc, od, os_, oc)


def test_edge_queries():
    c = corpus_from_lists(1000, [[1, 2, 3, 999], [], [2, 3, 4, 999], [0]],
                          [[1, 2, 3, 4], [], [5, 6, 7, 8], [9]], np.arange(1, 1001))
    ox = oracle.OracleIndex(c)
    gx = g.GriffinIndex(c)
    for terms in ([0, 0, 2], [2, 0], [0, 1], [1], [3], [3, 0], [0]):
        od, os_, oc = ox.query(terms, 5)
        gd, gs, gc = gx.griffin_query(terms, 5)
        assert_topk_equal(gd, gs, gc, od, os_, oc)
    for bad in ([7], []):
        with pytest.raises(g.GriffinError):
            gx.griffin_query(bad, 5)
    with pytest.raises(g.GriffinError):
        gx.griffin_query([0], 4097)


def test_random_batches_bit_exact():
    rng = np.random.default_rng(123)
    for trial in range(4):
        c = random_corpus(rng, num_docs=int(rng.integers(1000, 100_000)), num_terms=12,
                          max_df=40_000)
        ox = oracle.OracleIndex(c)
        gx = g.GriffinIndex(c, block_size=int(rng.choice([64, 128, 256, 512])),
                            gallop_ratio=int(rng.choice([0, 4, 1000])))
        ql = random_queries(rng, c.num_terms, 50)
        k = int(rng.choice([5, 100, 2000]))
        od, os_, oc = ox.query_batch(ql, k)
        gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
        assert_topk_equal(gd, gs, gc, od, os_, oc)


def test_device_api_matches_host_api(tiny, tiny_gpu):
    import torch
    c, ql, ox = tiny
    k = 10
    nq = ql.num_queries
    tiny_gpu.griffin_reserve(ql.offsets, ql.terms, k)
    d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
    d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
    keys = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
    cnt = torch.zeros(nq, dtype=torch.int32, device="cuda")
    dd = torch.zeros(nq * k, dtype=torch.int32, device="cuda")
    ds = torch.zeros(nq * k, dtype=torch.float32, device="cuda")
    s = torch.cuda.current_stream()
    mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
    tiny_gpu.griffin_query_batch_device(d_off, d_t, mt, k, keys, cnt, s)
    tiny_gpu.griffin_keys_to_results_device(nq, k, keys, cnt, dd, ds, s)
    torch.cuda.synchronize()
    tiny_gpu.griffin_sync_status()
    od, os_, oc = ox.query_batch(ql, k)
    gd = dd.cpu().numpy().view(np.uint32).reshape(nq, k)
    gs = ds.cpu().numpy().reshape(nq, k)
    assert_topk_equal(gd, gs, cnt.cpu().numpy().view(np.uint32), od, os_, oc)


@pytest.mark.parametrize("G", [2, 3, 8])
def test_docid_sharding_merge_equals_unsharded(tiny, G):
    """G docID-range shards on one device (same code path as one shard per GPU,
    minus NCCL): per-shard top-k keys merged by the device k-way merge equal the
    unsharded oracle bit for bit (SURVEY §8(e) exactness argument)."""
    import torch
    c, ql, ox = tiny
    k = 20
    nq = ql.num_queries
    mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
    d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
    d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
    keys = torch.zeros(G, nq * k, dtype=torch.int64, device="cuda")
    cnts = torch.zeros(G, nq, dtype=torch.int32, device="cuda")
    shards = []
    for s in range(G):
        sx = g.GriffinIndex(c, shard_index=s, num_shards=G)
        sx.griffin_reserve(ql.offsets, ql.terms, k)
        sx.griffin_query_batch_device(d_off, d_t, mt, k, keys[s], cnts[s],
                                      torch.cuda.current_stream())
        shards.append(sx)
    torch.cuda.synchronize()
    out_k = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
    out_c = torch.zeros(nq, dtype=torch.int32, device="cuda")
    shards[0].griffin_merge_topk_device(G, nq, k, keys, cnts, out_k, out_c)
    dd = torch.zeros(nq * k, dtype=torch.int32, device="cuda")
    ds = torch.zeros(nq * k, dtype=torch.float32, device="cuda")
    shards[0].griffin_keys_to_results_device(nq, k, out_k, out_c, dd, ds)
    torch.cuda.synchronize()
    od, os_, oc = ox.query_batch(ql, k)
    assert_topk_equal(dd.cpu().numpy().view(np.uint32).reshape(nq, k),
                      ds.cpu().numpy().reshape(nq, k), out_c.cpu().numpy().view(np.uint32),
                      od, os_, oc)


# ---------------------------------------------------------------- full size (bench config)

def _timed_config_run(c, batches, k, slots, steps):
    """Run `steps` batches exactly as bench.py times them: device API, `slots`
    workspaces (the index's own + extra ones) each on its own stream, batch i
    on slot i % slots, rotating through `batches`; returns the host results of
    every step's batch (keys -> rows) plus the index (for further checks)."""
    import torch
    gx = g.GriffinIndex(c, block_size=128)
    dq = []
    for b in batches:
        gx.griffin_reserve(b.offsets, b.terms, k)
        mt = int(max(len(set(b.query(q).tolist())) for q in range(b.num_queries)))
        dq.append((torch.from_numpy(b.offsets.astype(np.int32)).cuda(),
                   torch.from_numpy(b.terms.astype(np.int32)).cuda(), mt))
    nq = batches[0].num_queries
    sl = [(None, torch.cuda.current_stream())]
    for _ in range(slots - 1):
        w = gx.griffin_workspace_create()
        for b in batches:
            w.griffin_workspace_reserve(b.offsets, b.terms, k)
        sl.append((w, torch.cuda.Stream()))
    outs = [(torch.zeros(nq * k, dtype=torch.int64, device="cuda"),
             torch.zeros(nq, dtype=torch.int32, device="cuda")) for _ in range(steps)]
    for i in range(steps):
        w, st = sl[i % slots]
        d_off, d_t, mt = dq[i % len(batches)]
        kk, cc = outs[i]
        if w is None:
            gx.griffin_query_batch_device(d_off, d_t, mt, k, kk, cc, st)
        else:
            w.griffin_query_batch_device_ws(d_off, d_t, mt, k, kk, cc, st)
    torch.cuda.synchronize()
    gx.griffin_sync_status()
    for w, _ in sl[1:]:
        w.griffin_workspace_sync_status()
    res = []
    for kk, cc in outs:
        keys = kk.cpu().numpy().view(np.uint64).reshape(nq, k)
        cnt = cc.cpu().numpy().view(np.uint32)
        d = (np.uint64(0xFFFFFFFF) - (keys & np.uint64(0xFFFFFFFF))).astype(np.uint32)
        sc = (keys >> np.uint64(32)).astype(np.uint32).view(np.float32)
        valid = np.arange(k)[None, :] < cnt[:, None]
        res.append((np.where(valid, d, np.uint32(0xFFFFFFFF)),
                    np.where(valid, sc, np.float32(-np.inf)), cnt))
    return gx, res


@pytest.mark.slow
def test_c2_full_size_all_queries_timed_config():
    """BASELINE configs[1] at full size in the launch configuration bench.py
    times for it (3 workspaces on 3 streams, rotating the config's 3 batches of
    1000 queries): EVERY query of every batch bit-exact against the oracle."""
    c, ql, cfg = make_workload("c2")
    batches = [batch_of(ql, cfg, i) for i in range(cfg["batches"])]
    k = cfg["k"]
    gx, res = _timed_config_run(c, batches, k, slots=3, steps=6)
    del gx
    ox = oracle.OracleIndex(c, block_size=128)
    for i, b in enumerate(batches):
        od, os_, oc = ox.query_batch(b, k, nthreads=os.cpu_count() or 4)
        for step in (i, i + 3):   # each batch ran twice, on different slots
            gd, gs, gc = res[step]
            assert_topk_equal(gd, gs, gc, od, os_, oc)


@pytest.mark.parametrize("inv", [0, 32, 1 << 24])
def test_large_batch_s_locality_order(inv):
    """Batches of >= 4096 queries hand out merge units (and bitvector units, by
    S slot and R docID) in S-locality order (sorder_scatter_kernel); the results
    must not depend on it."""
    import torch
    c, ql, cfg = make_workload("small", num_queries=5000)
    gx = g.GriffinIndex(c, block_size=128)
    gx.griffin_set_bitmap(inv)
    gx.griffin_set_profiling(3)
    ox = oracle.OracleIndex(c, block_size=128)
    k, nq = 10, ql.num_queries
    # device API: one batch of all 5000 queries (the host API would slice it)
    gx.griffin_reserve(ql.offsets, ql.terms, k)
    mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
    d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
    d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
    keys = torch.zeros(nq * k, dtype=torch.int64, device="cuda")
    cnt = torch.zeros(nq, dtype=torch.int32, device="cuda")
    gx.griffin_query_batch_device(d_off, d_t, mt, k, keys, cnt, torch.cuda.current_stream())
    dd = torch.zeros(nq * k, dtype=torch.int32, device="cuda")
    ds = torch.zeros(nq * k, dtype=torch.float32, device="cuda")
    gx.griffin_keys_to_results_device(nq, k, keys, cnt, dd, ds)
    torch.cuda.synchronize()
    gx.griffin_sync_status()
    od, os_, oc = ox.query_batch(ql, k, nthreads=4)
    assert_topk_equal(dd.cpu().numpy().view(np.uint32).reshape(nq, k), ds.cpu().numpy().reshape(nq, k),
                      cnt.cpu().numpy().view(np.uint32), od, os_, oc)
    prof = gx.griffin_get_profile()
    if inv == 0:
        assert prof["bitmap_units"] == 0
    if inv == 1 << 24:
        assert prof["bitmap_units"] > 0


def test_large_host_batch_bit_exact():
    """A host-buffer griffin_query_batch of 9000 queries (word-AND units, the
    S-locality order and the subset top-k threshold all engaged) equals the
    oracle, with bitvectors on and off."""
    c, ql, cfg = make_workload("small", num_queries=9000)
    ox = oracle.OracleIndex(c, block_size=128)
    # k = 1000: 72 MB of results through the pinned staging
    for inv, k in ((32, 10), (0, 10), (32, 1000)):
        od, os_, oc = ox.query_batch(ql, k, nthreads=4)
        gx = g.GriffinIndex(c, block_size=128)
        gx.griffin_set_bitmap(inv)
        gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
        assert_topk_equal(gd, gs, gc, od, os_, oc)
        gx.close()


@pytest.mark.slow
def test_c5_full_size_timed_config():
    """BASELINE configs[4] at full size (50M docs, ~1.9 B postings, 10K queries
    per batch, top-1000) in bench.py's launch configuration (2 workspaces on 2
    streams, rotating batches, decode-once reuse on): invariants on every query
    of two batches and the first 1000 queries of batch 0 plus 200 of batch 1
    bit-exact against the oracle (built over those queries' complete lists with
    the full corpus' N and doc lengths, synth.sub_corpus)."""
    c, ql, cfg = make_workload("c5")
    batches = [batch_of(ql, cfg, i) for i in range(2)]
    k = cfg["k"]
    gx, res = _timed_config_run(c, batches, k, slots=2, steps=2)
    del gx
    for (gd, gs, gc), b in zip(res, batches):
        nq = b.num_queries
        assert gc.max() > 100, "the planted co-occurrences should give large results"
        for q in range(nq):
            n = gc[q]
            s_, d_ = gs[q, :n], gd[q, :n]
            assert np.all((s_[1:] < s_[:-1]) | ((s_[1:] == s_[:-1]) & (d_[1:] > d_[:-1])))
            assert np.all(gd[q, n:] == 0xFFFFFFFF) and np.all(np.isneginf(gs[q, n:]))
    for (gd, gs, gc), b, m in zip(res, batches, (1000, 200)):
        sub = b.slice(0, m)
        ox = oracle.OracleIndex(sub_corpus(c, sub.terms), block_size=128)
        od, os_, oc = ox.query_batch(sub, k, nthreads=os.cpu_count() or 4)
        assert_topk_equal(gd[:m], gs[:m], gc[:m], od, os_, oc)
        del ox


@pytest.mark.parametrize("B", [64, 128])
def test_large_tf_values_lossless(B):
    """tf is stored losslessly: tf in {65535, 65536, 2^20, 2^32-1}
    scores exactly as the oracle (no 16-bit clamp)."""
    rng = np.random.default_rng(7)
    N = 300_000
    big = np.array([65535, 65536, 1 << 20, 0xFFFFFFFF, 1, 2], np.uint32)
    lists, tfs = [], []
    for t in range(6):
        df = [500, 3000, 20000, 150, 80000, 7][t]
        lst = np.sort(rng.choice(N, size=df, replace=False)).astype(np.uint32)
        tf = rng.choice(big, size=df).astype(np.uint32)
        lists.append(lst)
        tfs.append(tf)
    # shared docs so every query has results
    common = np.sort(rng.choice(N, size=300, replace=False)).astype(np.uint32)
    lists = [np.union1d(l, common).astype(np.uint32) for l in lists]
    tfs = [rng.choice(big, size=len(l)).astype(np.uint32) for l in lists]
    c = corpus_from_lists(N, lists, tfs, rng.integers(1, 5000, size=N).astype(np.uint32))
    qs = [[0, 1], [1, 2], [0, 4], [2, 3, 4], [0, 1, 2, 3, 4], [5, 4], [4]]
    ql = QueryLog(offsets=np.cumsum([0] + [len(q) for q in qs]).astype(np.uint32),
                  terms=np.concatenate([np.array(q, np.uint32) for q in qs]))
    gx = g.GriffinIndex(c, block_size=B)
    ox = oracle.OracleIndex(c, block_size=B)
    for k in (10, 400):
        gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
        od, os_, oc = ox.query_batch(ql, k)
        assert_topk_equal(gd, gs, gc, od, os_, oc)


@pytest.mark.slow
def test_c3_full_size_ratio_pairs():
    """BASELINE configs[2] shape at full size: 25M docs, |S| = 10M (G6 extended),
    |R| = |S|/lambda for lambda from 1 to 1000: merge, gallop and
    auto give the oracle's docID set, and the scored top-10 / top-1000 are
    bit-exact (one batch of all pairs)."""
    ratios = [1, 4, 16, 64, 128, 512, 1000]
    c, ql = make_pair_workload(25_000_000, 10_000_000, ratios, seed=0x4752494646494E03)
    ox = oracle.OracleIndex(c, block_size=128)
    gx = g.GriffinIndex(c, block_size=128)
    for q in range(ql.num_queries):
        want = ox.intersect(ql.query(q))
        assert len(want) > 0
        for mode in (g.MODE_AUTO, g.MODE_MERGE, g.MODE_GALLOP):
            assert np.array_equal(gx.griffin_debug_intersect(ql.query(q), mode), want)
    for k in (10, 1000):
        d, s, cn = gx.griffin_query_batch(ql.offsets, ql.terms, k)
        od, os_, oc = ox.query_batch(ql, k)
        assert_topk_equal(d, s, cn, od, os_, oc)


# ---------------------------------------------------------------- batch list reuse

@pytest.mark.parametrize("reuse", [0, 1])
@pytest.mark.parametrize("mode", [g.MODE_AUTO, g.MODE_MERGE, g.MODE_GALLOP])
def test_reuse_and_modes_bit_exact(tiny, reuse, mode):
    """Decode-once arena (reuse=1) and fused decode (reuse=0), every intersection
    mode: identical to the oracle."""
    c, ql, ox = tiny
    gx = g.GriffinIndex(c, block_size=128)
    gx.griffin_set_reuse(reuse)
    gx.griffin_set_mode(mode)
    for k in (10, 300):
        od, os_, oc = ox.query_batch(ql, k)
        gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
        assert_topk_equal(gd, gs, gc, od, os_, oc)


def test_reuse_random_batches_and_single_terms():
    rng = np.random.default_rng(321)
    for trial in range(4):
        c = random_corpus(rng, num_docs=int(rng.integers(2000, 80_000)), num_terms=10,
                          max_df=30_000)
        ox = oracle.OracleIndex(c)
        B = int(rng.choice([64, 128, 256, 512]))
        gx = g.GriffinIndex(c, block_size=B, gallop_ratio=int(rng.choice([0, 3, 500])))
        gx.griffin_set_reuse(1)
        ql = random_queries(rng, c.num_terms, 60, max_terms=4)
        od, os_, oc = ox.query_batch(ql, 50)
        gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, 50)
        assert_topk_equal(gd, gs, gc, od, os_, oc)


@pytest.mark.parametrize("inv", [0, 32, 1 << 24])
def test_bitmap_decode_once_bit_exact(tiny, inv):
    """Dense lists decoded once into a bitvector + rank (griffin_set_bitmap):
    off, the default density threshold, and every decoded list — identical to
    the oracle, and the bitvector units really ran when enabled."""
    c, ql, ox = tiny
    gx = g.GriffinIndex(c, block_size=128)
    gx.griffin_set_reuse(1)
    gx.griffin_set_bitmap(inv)
    gx.griffin_set_profiling(3)
    for k in (10, 300):
        od, os_, oc = ox.query_batch(ql, k)
        gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
        assert_topk_equal(gd, gs, gc, od, os_, oc)
    prof = gx.griffin_get_profile()
    if inv == 1 << 24:
        assert prof["bitmap_units"] > 0 and prof["bitmap_elems"] > 0
    if inv == 0:
        assert prof["bitmap_units"] == 0
    gx.close()


@pytest.mark.parametrize("tau", [True, False])
@pytest.mark.parametrize("B", [64, 96, 128, 256, 512])
def test_bitmap_dense_runs_and_edges(B, tau, monkeypatch):
    """Bitvector construction and word-AND edge cases: lists of consecutive docIDs (whole
    words owned by one lane: plain stores), near-complete lists, docID 0 and
    N-1, word boundaries shared by lanes and blocks, multi-term queries (probe
    pass / later SvS rounds against bitvectors), every block size."""
    rng = np.random.default_rng(B)
    N = 70_003
    lists = [
        np.arange(0, N, dtype=np.uint32),                                   # every doc
        np.arange(5, N - 3, dtype=np.uint32)[rng.random(N - 8) < 0.97],     # near complete
        np.nonzero(rng.random(N) < 0.5)[0].astype(np.uint32),
        np.nonzero(rng.random(N) < 0.06)[0].astype(np.uint32),
        np.unique(np.concatenate([[0, 31, 32, 63, 64, N - 33, N - 32, N - 1],
                                  rng.integers(0, N, 3000)])).astype(np.uint32),
        np.arange(1000, 9000, dtype=np.uint32),                             # one run
        np.nonzero(rng.random(N) < 0.002)[0].astype(np.uint32),
    ]
    tfs = [rng.integers(1, 9, size=len(l)).astype(np.uint32) for l in lists]
    dl = rng.integers(1, 3000, size=N).astype(np.uint32)
    c = corpus_from_lists(N, lists, tfs, dl)
    ox = oracle.OracleIndex(c, block_size=B)
    # tau: the subset top-k threshold of 2-term word-AND queries (DESIGN R7)
    # at this small batch size too (the library applies it from 4096 queries)
    monkeypatch.setenv("GRIFFIN_TAU_MIN_QUERIES", "8" if tau else "1000000")
    gx = g.GriffinIndex(c, block_size=B)
    gx.griffin_set_reuse(1)
    gx.griffin_set_bitmap(1 << 24)
    gx.griffin_set_profiling(3)
    V = len(lists)
    offs, terms = [0], []
    for _ in range(3):
        for a in range(V):
            for b in range(V):
                terms.extend([a, b])
                offs.append(len(terms))
    for _ in range(40):
        m = int(rng.integers(3, 7))
        terms.extend(int(t) for t in rng.choice(V, size=m, replace=False))
        offs.append(len(terms))
    ql = QueryLog(offsets=np.array(offs, np.uint32), terms=np.array(terms, np.uint32))
    for k in (7, 1000):
        od, os_, oc = ox.query_batch(ql, k)
        gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
        assert_topk_equal(gd, gs, gc, od, os_, oc)
    prof = gx.griffin_get_profile()
    # every decoded list is a bitvector here: pairs of two of them are ANDed
    assert prof["bitand_units"] > 0
    gx.close()


@pytest.mark.parametrize("k", [64, 65, 1000, 2048])
def test_multilevel_topk_large_results(k):
    """Survivor sets of 10^4..10^5 per query force several chunked selection
    levels (zero-padded candidate arrays) before the final sort."""
    rng = np.random.default_rng(700 + k)
    N = 400_000
    lists = [np.sort(rng.choice(N, size=n, replace=False))
             for n in (300_000, 250_000, 200_000, 60_000, 9_000)]
    tfs = [rng.integers(1, 40, size=len(l)) for l in lists]
    c = corpus_from_lists(N, lists, tfs, rng.integers(1, 5000, size=N))
    ox = oracle.OracleIndex(c)
    gx = g.GriffinIndex(c)
    qs = [[0, 1], [0, 1, 2], [0], [1, 3], [2, 4], [0, 2], [1]]
    ql = QueryLog(offsets=np.cumsum([0] + [len(q) for q in qs]).astype(np.uint32),
                  terms=np.concatenate(qs).astype(np.uint32))
    od, os_, oc = ox.query_batch(ql, k)
    gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
    assert_topk_equal(gd, gs, gc, od, os_, oc)


@pytest.mark.parametrize("k", [100, 1000])
def test_topk_prefilter_on_off_identical(k, monkeypatch):
    """Queries with > 65536 candidates go through the sampled-threshold
    pre-filter (topk_sample/filter kernels, k > 64); with it disabled
    (GRIFFIN_TOPK_FILTER=0 at build) the results are the same and equal the
    oracle's.  Scores concentrated in a narrow docID band (long docs elsewhere)
    make the systematic sample unrepresentative on purpose."""
    rng = np.random.default_rng(900 + k)
    N = 600_000
    lists = [np.sort(rng.choice(N, size=n, replace=False)) for n in (500_000, 450_000, 200_000)]
    tfs = [rng.integers(1, 40, size=len(l)) for l in lists]
    dl = rng.integers(2000, 5000, size=N)
    dl[300_000:300_050] = 1      # a band of very short docs: the top scores
    c = corpus_from_lists(N, lists, tfs, dl)
    qs = [[0, 1], [0], [1, 2], [0, 1, 2], [2]]
    ql = QueryLog(offsets=np.cumsum([0] + [len(q) for q in qs]).astype(np.uint32),
                  terms=np.concatenate(qs).astype(np.uint32))
    od, os_, oc = oracle.OracleIndex(c).query_batch(ql, k)
    res = []
    for flag in ("1", "0"):
        monkeypatch.setenv("GRIFFIN_TOPK_FILTER", flag)
        gx = g.GriffinIndex(c)
        res.append(gx.griffin_query_batch(ql.offsets, ql.terms, k))
        del gx
    for gd, gs, gc in res:
        assert_topk_equal(gd, gs, gc, od, os_, oc)


def test_single_query_graph_path_reuse_and_recapture(tiny):
    """griffin_query replays cached CUDA graphs keyed by (distinct terms, k): many
    different queries, repeated, interleaved with a batch call that grows the
    workspace (forcing re-capture), all bit-exact."""
    c, ql, ox = tiny
    gx = g.GriffinIndex(c, block_size=128)
    for rep in range(2):
        for q in range(ql.num_queries):
            for k in (1, 10):
                od, os_, oc = ox.query(ql.query(q), k)
                gd, gs, gc = gx.griffin_query(ql.query(q), k)
                assert_topk_equal(gd, gs, gc, od, os_, oc)
        # a batch grows buffers -> the next single queries must re-capture
        gx.griffin_query_batch(ql.offsets, ql.terms, 3000)


def test_concurrent_workspaces_on_two_streams(tiny):
    """Two batches in flight on two streams (default + extra workspace) give the
    same, oracle-exact results as one at a time."""
    import torch
    c, ql, ox = tiny
    gx = g.GriffinIndex(c, block_size=128)
    ws = gx.griffin_workspace_create()
    k = 25
    nq = ql.num_queries
    mt = int(max(len(set(ql.query(q).tolist())) for q in range(nq)))
    gx.griffin_reserve(ql.offsets, ql.terms, k)
    ws.griffin_workspace_reserve(ql.offsets, ql.terms, k)
    d_off = torch.from_numpy(ql.offsets.astype(np.int32)).cuda()
    d_t = torch.from_numpy(ql.terms.astype(np.int32)).cuda()
    outs = [(torch.zeros(nq * k, dtype=torch.int64, device="cuda"),
             torch.zeros(nq, dtype=torch.int32, device="cuda")) for _ in range(2)]
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    for _ in range(3):
        gx.griffin_query_batch_device(d_off, d_t, mt, k, outs[0][0], outs[0][1], s1)
        ws.griffin_query_batch_device_ws(d_off, d_t, mt, k, outs[1][0], outs[1][1], s2)
    torch.cuda.synchronize()
    gx.griffin_sync_status()
    ws.griffin_workspace_sync_status()
    assert torch.equal(outs[0][0], outs[1][0]) and torch.equal(outs[0][1], outs[1][1])
    dd = torch.zeros(nq * k, dtype=torch.int32, device="cuda")
    ds = torch.zeros(nq * k, dtype=torch.float32, device="cuda")
    gx.griffin_keys_to_results_device(nq, k, outs[1][0], outs[1][1], dd, ds)
    torch.cuda.synchronize()
    od, os_, oc = ox.query_batch(ql, k)
    assert_topk_equal(dd.cpu().numpy().view(np.uint32).reshape(nq, k), ds.cpu().numpy().reshape(nq, k),
                      outs[1][1].cpu().numpy().view(np.uint32), od, os_, oc)
    ws.close()


def test_submit_collect_pipelined_workspaces(tiny):
    """griffin_query_batch_submit/collect with three workspaces in flight on
    three streams (bench.py's e2e loop): every collected batch is oracle-exact;
    different batches (varying k and query subsets) do not mix; misuse and a bad
    term are reported, and the workspace stays usable afterwards."""
    import torch
    c, ql, ox = tiny
    gx = g.GriffinIndex(c, block_size=128)
    wss = [gx.griffin_workspace_create() for _ in range(3)]
    sts = [torch.cuda.Stream() for _ in range(3)]
    nq = ql.num_queries
    subsets = [(0, nq, 10), (0, nq // 2, 25), (nq // 3, nq, 7), (1, 5, 1), (0, nq, 100)]
    expect = []
    for lo, hi, k in subsets:
        sub = ql.slice(lo, hi)
        expect.append((sub, k, ox.query_batch(sub, k)))
    got = [None] * len(expect)
    for i, (sub, k, _) in enumerate(expect * 2):
        w = wss[i % 3]
        if i >= 3:
            got[(i - 3) % len(expect)] = w.griffin_query_batch_collect()
        w.griffin_query_batch_submit(sub.offsets, sub.terms, k, sts[i % 3])
    for i in range(2 * len(expect) - 3, 2 * len(expect)):
        got[i % len(expect)] = wss[i % 3].griffin_query_batch_collect()
    for (sub, k, (od, os_, oc)), (gd, gs, gc) in zip(expect, got):
        assert_topk_equal(gd, gs, gc, od, os_, oc)
    w = wss[0]
    with pytest.raises(g.GriffinError):
        w.griffin_query_batch_collect()             # nothing submitted
    sub, k, (od, os_, oc) = expect[0]
    w.griffin_query_batch_submit(sub.offsets, sub.terms, k)
    with pytest.raises(g.GriffinError):
        w.griffin_query_batch_submit(sub.offsets, sub.terms, k)   # not yet collected
    assert_topk_equal(*w.griffin_query_batch_collect(), od, os_, oc)
    with pytest.raises(g.GriffinError):
        w.griffin_query_batch_submit(np.array([0, 1], np.uint32),
                                     np.array([c.num_terms], np.uint32), 10)
    w.griffin_query_batch_submit(sub.offsets, sub.terms, k)
    assert_topk_equal(*w.griffin_query_batch_collect(), od, os_, oc)
    # the index's own workspace (ws = NULL) blocks the synchronous calls while
    # it holds a batch
    gx.griffin_query_batch_submit(sub.offsets, sub.terms, k)
    with pytest.raises(g.GriffinError):
        gx.griffin_query_batch(sub.offsets, sub.terms, k)
    nqs = sub.num_queries
    out = (np.full(nqs * k, 7, np.uint32), np.zeros(nqs * k, np.float32), np.zeros(nqs, np.uint32))
    gd, gs, gc = gx.griffin_query_batch_collect(out)
    assert gd.base is out[0] or gd is out[0] or np.shares_memory(gd, out[0])
    assert_topk_equal(gd, gs, gc, od, os_, oc)
    assert_topk_equal(*gx.griffin_query_batch(sub.offsets, sub.terms, k), od, os_, oc)
    # zero-copy views of a workspace's pinned staging
    w = wss[1]
    w.griffin_query_batch_submit(sub.offsets, sub.terms, k)
    vd, vs, vc = w.griffin_query_batch_collect("view")
    assert not vd.flags.writeable
    assert_topk_equal(vd, vs, vc, od, os_, oc)
    for w in wss:
        w.close()


# ---------------------------------------------------------------- EF NextGEQ gallop

def _nextgeq_corpus(rng, N=3_000_000):
    """Lists that stress the bucket search: a consecutive run (b = 0), a very
    sparse list (large b, many empty buckets), a clustered list (bursts of
    consecutive docIDs: full buckets next to long zero runs), and random lists
    of several densities to probe them with."""
    run = np.arange(1_000_000, 1_006_000)
    sparse = np.sort(rng.choice(N, size=900, replace=False))
    starts = np.sort(rng.choice(N - 64, size=400, replace=False))
    clustered = np.unique(np.concatenate([s + np.arange(int(rng.integers(1, 60))) for s in starts]))
    lists = [run, sparse, clustered] + [np.sort(rng.choice(N, size=n, replace=False))
                                        for n in (300, 3_000, 30_000, 300_000, 1_500_000)]
    tfs = [rng.integers(1, 9, size=len(x)) for x in lists]
    return corpus_from_lists(N, lists, tfs, rng.integers(1, 3000, size=N))


def test_merge_tile_tail_no_false_matches():
    """Regression: the uniform-trip merge loop can step the S side past the
    tile's valid elements; stale shared memory there once matched an R element
    of an earlier unit (~1 in 400 calls at B = 512, D = 2; fixed by a sentinel).
    Repeats the triggering merges (a consecutive-run S list, a short random R)
    many times so stale tiles from earlier calls are around."""
    rng = np.random.default_rng(900 + 512)
    c = _nextgeq_corpus(rng)
    ox = oracle.OracleIndex(c)
    gx = g.GriffinIndex(c, block_size=512)
    gx.griffin_set_reuse(0)
    qs = ([0, 4], [4, 0], [0, 3], [0, 5], [0, 6], [0, 7])
    want = [ox.intersect(q) for q in qs]
    for _ in range(150):
        for q, w in zip(qs, want):
            for mode in (g.MODE_AUTO, g.MODE_MERGE):
                assert np.array_equal(gx.griffin_debug_intersect(q, mode), w), (q, mode)


@pytest.mark.parametrize("B", [64, 128, 256, 512])
def test_nextgeq_gallop_matches_block_decode_and_oracle(B):
    """Galloping into compressed lists by EF NextGEQ (select0 on the unary stream,
    only the probe's bucket decoded) gives the oracle's sets and bit-exact top-k;
    so does the block-decode gallop it replaces (griffin_set_nextgeq(0))."""
    rng = np.random.default_rng(900 + B)
    c = _nextgeq_corpus(rng)
    ox = oracle.OracleIndex(c)
    gx = g.GriffinIndex(c, block_size=B)
    gx.griffin_set_reuse(0)           # S stays compressed: the NextGEQ path
    pairs = [[a, b] for a in range(8) for b in range(8) if a != b]
    triples = [list(rng.choice(8, size=3, replace=False)) for _ in range(20)]
    qs = pairs + triples
    ql = QueryLog(offsets=np.cumsum([0] + [len(q) for q in qs]).astype(np.uint32),
                  terms=np.concatenate(qs).astype(np.uint32))
    for ng in (1, 0):
        gx.griffin_set_nextgeq(ng)
        for q in qs:
            want = ox.intersect(q)
            for mode in (g.MODE_GALLOP, g.MODE_AUTO):
                assert np.array_equal(gx.griffin_debug_intersect(q, mode), want), (ng, q, mode)
        for mode in (g.MODE_GALLOP, g.MODE_AUTO):
            gx.griffin_set_mode(mode)
            od, os_, oc = ox.query_batch(ql, 100)
            gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, 100)
            assert_topk_equal(gd, gs, gc, od, os_, oc)
        gx.griffin_set_mode(g.MODE_AUTO)


def test_entry_budget_packed_intermediates(tiny):
    """griffin_set_entry_budget: intermediates packed by actual survivors; a
    budget that holds them gives identical results, one that does not reports
    GRIFFIN_ERR_OOM, and the workspace recovers after the budget is raised."""
    c, ql, ox = tiny
    k = 10
    od, os_, oc = ox.query_batch(ql, k)
    # survivors of round 1 are at most the batch's results' superset; the exact
    # bound (sum of min(df0, df1)) is far larger than what is produced
    gx = g.GriffinIndex(c, block_size=128)
    gx.griffin_set_entry_budget(200_000)
    gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
    assert_topk_equal(gd, gs, gc, od, os_, oc)
    for mode in (g.MODE_MERGE, g.MODE_GALLOP):   # multi-round SvS (no probe pass): packed tops
        gx.griffin_set_mode(mode)
        gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
        assert_topk_equal(gd, gs, gc, od, os_, oc)
    gy = g.GriffinIndex(c, block_size=128)
    gy.griffin_set_entry_budget(64)
    with pytest.raises(g.GriffinError) as e:
        gy.griffin_query_batch(ql.offsets, ql.terms, k)
    assert e.value.status == 3
    gy.griffin_set_entry_budget(0)
    gd, gs, gc = gy.griffin_query_batch(ql.offsets, ql.terms, k)
    assert_topk_equal(gd, gs, gc, od, os_, oc)
