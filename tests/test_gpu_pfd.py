"""Parity of the GPU PforDelta comparator codec (griffin_pfd_*, SURVEY.md §8(f)
NEXT-3) against the oracle's PforDelta (oracle/pfd.cpp): encoded streams word
for word, decoded lists, and the decode sweep's checksum."""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_0044ws18_b200 as g
from helpers import corpus_from_lists, random_corpus

pytestmark = pytest.mark.gpu


def _edge_corpus(rng, N=2_000_000):
    lists = [
        np.array([5], np.uint32),                                   # n = 1: no gaps
        np.array([0, N - 1], np.uint32),                            # one huge gap
        np.arange(700_000, 700_900, dtype=np.uint32),               # all gaps 1 (b = 1)
        np.sort(rng.choice(N, size=3000, replace=False)),           # random
        np.unique(np.concatenate([s + np.arange(40) for s in rng.choice(N - 64, 200)])),  # bursts
        np.sort(np.concatenate([np.arange(0, 1000, 1), [N - 3, N - 2]])).astype(np.uint32),
        np.sort(rng.choice(N, size=200_000, replace=False)),
    ]
    return corpus_from_lists(N, lists)


@pytest.mark.parametrize("B", [64, 128, 256, 512])
def test_pfd_streams_and_decode_match_oracle(B):
    rng = np.random.default_rng(300 + B)
    for c in (_edge_corpus(rng), random_corpus(rng, 100_000, 12, 40_000)):
        px = g.GriffinPfd(c, block_size=B)
        st = px.griffin_pfd_stats()
        pay = 0
        exc = 0
        for t in range(c.num_terms):
            lst = c.docids[c.offsets[t]:c.offsets[t + 1]]
            for k, s in enumerate(range(0, len(lst), B)):
                blk = lst[s:s + B]
                want, _, ne = oracle.pfd_encode(blk)
                f, n, words = px.griffin_pfd_block_stream(t, k)
                assert (f, n) == (int(blk[0]), len(blk))
                assert np.array_equal(words, want), (t, k)
                pay += ((len(want) + 3) // 4) * 16
                exc += ne
            got = px.griffin_pfd_decode_list(t, len(lst))
            assert np.array_equal(got, lst), t
        assert st["payload_bytes"] == pay and st["exceptions"] == exc
        assert st["num_postings"] == len(c.docids)


def test_pfd_decode_sweep_checksum():
    rng = np.random.default_rng(77)
    c = random_corpus(rng, 1_000_000, 40, 300_000)
    px = g.GriffinPfd(c, block_size=128)
    r = px.griffin_pfd_decode_all(iters=2)
    x = np.bitwise_xor.reduce(c.docids.astype(np.uint64)) if len(c.docids) else 0
    assert r["checksum"] == int(x) and r["postings"] == len(c.docids)
    st = px.griffin_pfd_stats()
    assert r["bytes"] == st["payload_bytes"] + st["skip_bytes"]
