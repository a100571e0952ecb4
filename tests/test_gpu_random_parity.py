"""Randomised parity (hypothesis): random small corpora (list lengths from empty
to dense, docIDs near 0 and N-1, tf up to 2^32-1), random block sizes and
batches of 1-8 term queries with repeats and empty-list terms, k from 1 to 600,
each index mode and decode-once representation (docID arena or dense-list
bitvector) — the GPU top-k (docIDs, order, score bits, counts) must equal
the oracle's.  Shapes are kept small so every example runs in well under a
second; the examples together exercise partial blocks, b = 0 runs, single-block
lists, merge and gallop rounds, the probe pass and the top-k levels."""
import numpy as np
import pytest

hypothesis = pytest.importorskip("hypothesis")
from hypothesis import HealthCheck, given, settings, strategies as st  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ppopp_0044ws18_b200 as g  # noqa: E402
from helpers import corpus_from_lists  # noqa: E402
from synth import QueryLog  # noqa: E402

pytestmark = pytest.mark.gpu


@st.composite
def workloads(draw):
    seed = draw(st.integers(0, 2**32 - 1))
    rng = np.random.default_rng(seed)
    N = draw(st.sampled_from([97, 1_000, 40_000, 3_000_000]))
    V = draw(st.integers(2, 12))
    lists, tfs = [], []
    for _ in range(V):
        kind = draw(st.sampled_from(["empty", "tiny", "sparse", "dense", "run", "edges"]))
        if kind == "empty":
            lst = np.zeros(0, np.uint32)
        elif kind == "tiny":
            lst = np.sort(rng.choice(N, size=min(N, int(rng.integers(1, 5))), replace=False))
        elif kind == "sparse":
            lst = np.sort(rng.choice(N, size=min(N, int(rng.integers(5, 3000))), replace=False))
        elif kind == "dense":
            lst = np.nonzero(rng.random(N) < rng.uniform(0.2, 0.9))[0]
        elif kind == "run":   # consecutive docIDs: b = 0 blocks
            a = int(rng.integers(0, N))
            lst = np.arange(a, min(N, a + int(rng.integers(1, 2000))))
        else:
            lst = np.unique(np.concatenate([[0, N - 1], rng.integers(0, N, 50)]))
        lst = lst.astype(np.uint32)
        lists.append(lst)
        tfs.append(rng.choice(np.array([1, 2, 3, 7, 65535, 65536, 2**32 - 1], np.uint32),
                              size=len(lst), p=[.4, .2, .2, .1, .04, .03, .03]).astype(np.uint32))
    dl = rng.integers(1, 3000, size=N).astype(np.uint32)
    nq = draw(st.integers(1, 24))
    offs, terms = [0], []
    for _ in range(nq):
        m = int(rng.integers(1, 9))
        terms.extend(int(t) for t in rng.integers(0, V, size=m))   # repeats allowed
        offs.append(len(terms))
    ql = QueryLog(offsets=np.array(offs, np.uint32), terms=np.array(terms, np.uint32))
    B = draw(st.sampled_from([64, 96, 128, 256, 512]))
    k = draw(st.sampled_from([1, 3, 10, 100, 600]))
    mode = draw(st.sampled_from([g.MODE_AUTO, g.MODE_MERGE, g.MODE_GALLOP]))
    reuse = draw(st.sampled_from([0, 1, 2]))
    bitmap = draw(st.sampled_from([0, 32, 1 << 24]))   # dense-list bitvectors: off / default / every decoded list
    return corpus_from_lists(N, lists, tfs, dl), ql, B, k, mode, reuse, bitmap


@settings(max_examples=150, deadline=None, derandomize=True,
          suppress_health_check=list(HealthCheck))
@given(workloads())
def test_random_workloads_bit_exact(w):
    c, ql, B, k, mode, reuse, bitmap = w
    import os
    os.environ["GRIFFIN_TAU_MIN_QUERIES"] = "8"   # the R7 threshold at these small batches too
    try:
        gx = g.GriffinIndex(c, block_size=B)
    finally:
        del os.environ["GRIFFIN_TAU_MIN_QUERIES"]
    gx.griffin_set_mode(mode)
    gx.griffin_set_reuse(reuse)
    gx.griffin_set_bitmap(bitmap)
    ox = oracle.OracleIndex(c, block_size=B)
    gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
    od, os_, oc = ox.query_batch(ql, k)
    assert np.array_equal(gc, oc)
    assert np.array_equal(gd, od)
    assert np.array_equal(gs.view(np.uint32), os_.view(np.uint32))
    gx.close()
