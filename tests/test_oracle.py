"""Pins for the CPU oracle against what the paper and the mathematics fix.

Every test here checks the oracle against something other than itself: the
paper's worked examples (tests/golden/*, each citing PAPER.md), closed forms, the
EF size bound, brute-force set intersection and exact double-precision BM25.
"""
import math

import numpy as np
import pytest

import oracle
from conftest import read_golden
from helpers import (bits_lsb_first, corpus_from_lists, f32_bits, f32_from_hex,
                     random_corpus, random_queries)


# ---------------------------------------------------------------- EF codec (O3/O4)

def test_fig4_encoding_example():
    """Fig. 4: b, low bits, unary-coded high bits."""
    g = read_golden("fig4_ef_example.txt")
    vals = [int(x) for x in g["values"][0]]
    U = int(g["U"][0][0])
    b, low, low_bits, high, high_bits = oracle.ef_encode(vals, U)
    assert b == int(g["b"][0][0])
    assert low_bits == len(vals) * b
    low_vals = [(int(low[(i * b) // 32]) >> ((i * b) % 32)) & ((1 << b) - 1) for i in range(len(vals))]
    assert low_vals == [int(x) for x in g["low_values"][0]]
    assert bits_lsb_first(high, high_bits) == g["unary_stream"][0][0]
    # reading A3 (LSB-first 32-bit words): the words SURVEY T1 states
    assert int(high[0]) == 0x2156 and int(low[0]) == 0x6C9
    # decode gives the sequence back
    assert oracle.ef_decode(low, high, len(vals), b).tolist() == vals


def test_high_parts_are_unary_gaps():
    """The accumulated number of zeros before the k-th one is h_k."""
    g = read_golden("fig4_ef_example.txt")
    vals = [int(x) for x in g["values"][0]]
    b, _, _, high, high_bits = oracle.ef_encode(vals, int(g["U"][0][0]))
    s = bits_lsb_first(high, high_bits)
    zeros, hs = 0, []
    for ch in s:
        if ch == "0":
            zeros += 1
        else:
            hs.append(zeros)
    assert hs == [int(x) for x in g["high_values"][0]] == [v >> b for v in vals]


def _ceil_log2_ratio(u, n):
    """smallest c >= 0 with n * 2^c >= u (exact integers)."""
    c = 0
    while n * (1 << c) < u:
        c += 1
    return c


@pytest.mark.parametrize("B", [64, 128, 256, 512])
def test_roundtrip_and_size_bound(B):
    rng = np.random.default_rng(1000 + B)
    N = 300_000
    lists = []
    for df in [1, 2, B - 1, B, B + 1, 3 * B + 7, 5000, 40_000, 200_000]:
        lists.append(np.sort(rng.choice(N, size=df, replace=False)))
    lists.append(np.arange(10, 10 + 2 * B + 3))            # consecutive run: u = n, b = 0
    lists.append(np.array([0]))                             # docID 0 alone
    lists.append(np.array([0, N - 1]))                      # extremes
    c = corpus_from_lists(N, lists)
    ix = oracle.OracleIndex(c, block_size=B)
    for t in range(c.num_terms):
        ref = c.list(t)
        assert np.array_equal(ix.decode_list(t), ref)
        nb = ix.num_blocks(t)
        assert nb == (len(ref) + B - 1) // B
        for blk in range(nb):
            first, n, b, low, lb, high, hb = ix.block_streams(t, blk)
            x = ref[blk * B: blk * B + n].astype(np.int64)
            assert n == len(x) and first == x[0]
            u = int(x[-1] - x[0] + 1)
            assert b == (u // n).bit_length() - 1          # reading A1, b = floor(log2(u/n))
            assert lb == n * b
            assert hb == n + (int(x[-1] - x[0]) >> b)
            # EF size bound (north star): n*b + L <= n*(2 + ceil(log2(u/n)))
            assert lb + hb <= n * (2 + _ceil_log2_ratio(u, n))
            if len(ref) > 1 and (ref[1:] - ref[:-1] == 1).all():
                assert b == 0


def test_max_docid_roundtrip():
    """docIDs up to 2^32 - 2 (reading A18: 0xFFFFFFFF is the sentinel), block
    semantics v_i = x_i - first, U = v_{n-1} + 1 (reading A2)."""
    x = np.array([0, 5, 1 << 31, 0xFFFFFFFE], np.uint64)
    v = (x - x[0]).astype(np.uint32)
    b, low, lb, high, hb = oracle.ef_encode(v, int(v[-1]) + 1)
    assert b == ((int(v[-1]) + 1) // 4).bit_length() - 1
    assert np.array_equal(oracle.ef_decode(low, high, 4, b), v)


def test_fig2_skip_pointer_lookup():
    """Fig. 2: the block holding x is upper_bound(first, x) - 1;
    block firsts of an index built from those ranges equal the figure's."""
    g = read_golden("skip_fig2.txt")
    firsts = [int(x) for x in g["firsts"][0]]
    lasts = [int(x) for x in g["lasts"][0]]
    B = 64
    lst = []
    rng = np.random.default_rng(7)
    for f, l in zip(firsts, lasts):
        mid = np.sort(rng.choice(np.arange(f + 1, l), size=B - 2, replace=False))
        lst.extend([f, *mid.tolist(), l])
    c = corpus_from_lists(9000, [np.array(lst)])
    ix = oracle.OracleIndex(c, block_size=B)
    got = [ix.block_streams(0, k)[0] for k in range(ix.num_blocks(0))]
    assert got == firsts
    for x, blk in g["lookup"]:
        k = int(np.searchsorted(np.array(got), int(x), side="right")) - 1
        assert k == int(blk)


# ---------------------------------------------------------------- SvS intersection (O5)

def test_svs_paper_example():
    g = read_golden("svs_example.txt")
    lists = [np.array([int(x) for x in row]) for row in g["list"]]
    c = corpus_from_lists(100, lists)
    ix = oracle.OracleIndex(c)
    want = [int(x) for x in g["result"][0]]
    for perm in ([0, 1, 2], [2, 1, 0], [1, 2, 0]):
        assert ix.intersect(perm).tolist() == want


def test_intersection_matches_bruteforce_hashset():
    rng = np.random.default_rng(42)
    for trial in range(30):
        c = random_corpus(rng, num_docs=int(rng.integers(50, 3000)), num_terms=6, max_df=700)
        ix = oracle.OracleIndex(c, block_size=int(rng.choice([64, 128, 256])))
        for _ in range(8):
            k = int(rng.integers(1, 6))
            terms = rng.integers(0, c.num_terms, size=k)
            s = None
            for t in terms:
                st = set(int(x) for x in c.list(int(t)))
                s = st if s is None else (s & st)
            assert ix.intersect(terms).tolist() == sorted(s)


# ---------------------------------------------------------------- BM25 (O1, O6)

def _bm25_double(c, terms, d, k1=1.2, b=0.75):
    """Exact double-precision textbook BM25 (readings A12-A13), independent of the oracle."""
    N = c.num_docs
    avgdl = float(np.sum(c.doc_lengths, dtype=np.uint64)) / N
    s = 0.0
    for t in sorted(set(int(x) for x in terms)):
        lst = c.list(t)
        pos = int(np.searchsorted(lst, d))
        assert lst[pos] == d
        tf = float(c.tf_list(t)[pos])
        df = float(len(lst))
        idf = math.log(1.0 + (N - df + 0.5) / (df + 0.5))
        s += idf * tf * (k1 + 1.0) / (tf + k1 * ((1 - b) + b * c.doc_lengths[d] / avgdl))
    return s


def _hand_corpus():
    g = read_golden("bm25_hand.txt")
    N = int(g["N"][0][0])
    dl = [int(x) for x in g["doc_lengths"][0]]
    lists, tfs = [], []
    for row in g["term"]:
        lists.append([int(p.split(":")[0]) for p in row])
        tfs.append([int(p.split(":")[1]) for p in row])
    return g, corpus_from_lists(N, lists, tfs, dl)


def test_bm25_hand_example_bits():
    g, c = _hand_corpus()
    ix = oracle.OracleIndex(c, k1=1.2, b=0.75)
    assert [f32_bits(ix.idf(t)) for t in range(2)] == [int(h, 16) for h in g["idf_bits"][0]]
    assert [f32_bits(ix.norm(d)) for d in range(4)] == [int(h, 16) for h in g["norm_bits"][0]]
    assert f32_bits(ix.k1p1()) == int(g["k1p1_bits"][0][0], 16)
    d, s, cnt = ix.query([int(x) for x in g["query"][0]], k=3)
    want = [(int(a), int(h, 16)) for a, h in g["top"]]
    assert cnt == len(want)
    assert [(int(d[i]), f32_bits(s[i])) for i in range(cnt)] == want
    assert d[2] == 0xFFFFFFFF and s[2] == -np.inf


def test_bm25_closed_form():
    """idf/norm are the double closed form rounded once to f32 (A14); scores are
    within the fp32 error bound of the exact double BM25."""
    g, c = _hand_corpus()
    ix = oracle.OracleIndex(c)
    assert ix.idf(0) == np.float32(math.log1p((4 - 2 + 0.5) / (2 + 0.5)))
    assert ix.idf(0) == np.float32(math.log(2.0))
    assert ix.idf(1) == np.float32(math.log(10.0 / 7.0))
    assert ix.norm(0) == np.float32(1.2 * (0.25 + 0.75 * 10 / 25))
    d, s, cnt = ix.query([0, 1], k=2)
    for i in range(cnt):
        ref = _bm25_double(c, [0, 1], int(d[i]))
        assert abs(float(s[i]) - ref) <= 1e-6 * ref


def test_bm25_monotone_and_tie_order():
    # tie case: equal (tf, dl) => equal scores, ordered by docID ascending (A16)
    c = corpus_from_lists(4, [[1, 3]], [[2, 2]], [25, 25, 25, 25])
    ix = oracle.OracleIndex(c)
    d, s, cnt = ix.query([0], k=4)
    assert cnt == 2 and d[:2].tolist() == [1, 3] and s[0] == s[1]
    assert f32_bits(s[0]) == 0x3F73FCE1
    # monotone: w grows with tf, shrinks with dl
    c = corpus_from_lists(4, [[0, 1, 2, 3]], [[1, 2, 2, 2]], [50, 50, 10, 90])
    ix = oracle.OracleIndex(c)
    d, s, cnt = ix.query([0], k=4)
    sc = {int(d[i]): float(s[i]) for i in range(cnt)}
    assert sc[1] > sc[0]            # tf 2 > tf 1 at equal dl
    assert sc[2] > sc[1] > sc[3]    # shorter doc scores higher at equal tf


def test_scores_and_topk_against_double_bruteforce():
    """Full query vs a brute-force double reference on random tiny corpora: the
    docID set of the top-k, the count, the ordering rule and the score values."""
    rng = np.random.default_rng(5)
    for trial in range(20):
        c = random_corpus(rng, num_docs=int(rng.integers(100, 2000)), num_terms=5, max_df=600)
        ix = oracle.OracleIndex(c)
        ql = random_queries(rng, c.num_terms, 10)
        for q in range(ql.num_queries):
            terms = ql.query(q)
            k = int(rng.choice([1, 5, 10, 1000]))
            d, s, cnt = ix.query(terms, k)
            inter = None
            for t in terms:
                st = set(int(x) for x in c.list(int(t)))
                inter = st if inter is None else inter & st
            assert cnt == min(k, len(inter))
            exact = {x: _bm25_double(c, terms, x) for x in inter}
            for i in range(cnt):
                assert int(d[i]) in inter
                assert abs(float(s[i]) - exact[int(d[i])]) <= 2e-6 * exact[int(d[i])]
                if i:
                    assert (s[i] < s[i - 1]) or (s[i] == s[i - 1] and d[i] > d[i - 1])
            # everything left out scores no higher than the last kept (up to fp32 error)
            if cnt and cnt < len(inter):
                kept = set(int(x) for x in d[:cnt])
                worst = min(exact[x] for x in kept)
                assert all(exact[x] <= worst * (1 + 4e-6) for x in inter - kept)
            assert (d[cnt:] == 0xFFFFFFFF).all() and np.isneginf(s[cnt:]).all()


def test_topk_prefix_consistency_and_batch():
    rng = np.random.default_rng(9)
    c = random_corpus(rng, num_docs=5000, num_terms=8, max_df=3000)
    ix = oracle.OracleIndex(c)
    ql = random_queries(rng, c.num_terms, 40)
    D, S, C = ix.query_batch(ql, k=50, nthreads=3)
    for q in range(ql.num_queries):
        d, s, cnt = ix.query(ql.query(q), 50)
        assert cnt == C[q] and np.array_equal(d, D[q]) and np.array_equal(s, S[q])
        d2, s2, c2 = ix.query(ql.query(q), 7)
        assert c2 == min(7, cnt) and np.array_equal(d2[:c2], d[:c2])


def test_dedup_and_empty_terms():
    c = corpus_from_lists(50, [[1, 2, 3], [], [2, 3, 4]])
    ix = oracle.OracleIndex(c)
    d, s, cnt = ix.query([0, 0, 2], 10)
    d2, s2, c2 = ix.query([2, 0], 10)
    assert cnt == c2 == 2 and np.array_equal(d, d2) and np.array_equal(s, s2)
    assert ix.query([0, 1], 10)[2] == 0
    with pytest.raises(ValueError):
        ix.query([7], 10)
