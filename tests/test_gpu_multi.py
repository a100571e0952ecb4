"""The multi-GPU handle behind the C ABI (SURVEY §8(b) num_gpus, §8(e)):
griffin_query_batch on a handle over G docID-range shards returns the GLOBAL
top-k, bit-exact against the unsharded oracle, for every exchange mode the box
can run.  On a one-GPU box the shards share device 0 (peer exchange: the fused
gather+merge kernel reads each shard's runs in place) and the NCCL exchanges
run as a one-rank communicator; with >= 2 GPUs the NCCL modes run across
distinct devices."""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_0044ws18_b200 as g
from helpers import random_corpus, random_queries
from synth import batch_of, make_workload

pytestmark = pytest.mark.gpu


def _bits(a):
    return np.asarray(a, np.float32).view(np.uint32)


def _check(gx, ox, ql, k):
    gd, gs, gc = gx.griffin_query_batch(ql.offsets, ql.terms, k)
    od, os_, oc = ox.query_batch(ql, k, nthreads=4)
    assert np.array_equal(gc, oc)
    assert np.array_equal(gd, od)
    assert np.array_equal(_bits(gs), _bits(os_))


@pytest.fixture(scope="module")
def small():
    c, ql, cfg = make_workload("small", num_queries=300)
    return c, ql, oracle.OracleIndex(c, block_size=128)


@pytest.mark.parametrize("G", [2, 3, 8])
@pytest.mark.parametrize("k", [10, 1000])
def test_peer_exchange_shards_on_one_device(small, G, k):
    c, ql, ox = small
    gx = g.GriffinIndex(c, block_size=128, num_gpus=G, devices=[0] * G,
                        exchange=g.EXCHANGE_PEER)
    st = gx.griffin_index_stats()
    assert st["num_shards"] == G and st["num_postings"] == c.num_postings
    _check(gx, ox, ql, k)
    # single query through the same handle
    d, s, n = gx.griffin_query(ql.query(3), k)
    od, os_, on = ox.query(ql.query(3), k)
    assert n == on and np.array_equal(d, od) and np.array_equal(_bits(s), _bits(os_))


@pytest.mark.parametrize("exchange", [1, 3])
def test_nccl_exchange_one_rank(small, exchange):
    """The NCCL code path (communicator per device, all-gather or grouped
    send/recv, merge) with one rank — all a one-GPU box can run."""
    c, ql, ox = small
    try:
        gx = g.GriffinIndex(c, block_size=128, num_gpus=1, exchange=exchange)
    except g.GriffinError as e:
        if e.status == 5:
            pytest.skip("NCCL not loadable: " + str(e))
        raise
    _check(gx, ox, ql, 10)


def test_multi_handle_random_corpora_and_edge_queries():
    rng = np.random.default_rng(11)
    c = random_corpus(rng, 50_000, 40, 6000)
    ql = random_queries(rng, 40, 200, max_terms=5)
    ox = oracle.OracleIndex(c, block_size=64)
    gx = g.GriffinIndex(c, block_size=64, num_gpus=4, devices=[0, 0, 0, 0])
    for k in (1, 7, 300):
        _check(gx, ox, ql, k)
    with pytest.raises(g.GriffinError) as e:   # single-shard-only entry points
        gx.griffin_reserve(ql.offsets, ql.terms, 10)
    assert e.value.status == 6


def test_nccl_needs_distinct_devices(small):
    c, ql, ox = small
    with pytest.raises(g.GriffinError) as e:
        g.GriffinIndex(c, num_gpus=2, devices=[0, 0], exchange=g.EXCHANGE_NCCL_ALLGATHER)
    assert e.value.status in (1, 5)


def test_multi_gpu_distinct_devices_all_exchanges(small):
    import torch
    n = torch.cuda.device_count()
    if n < 2:
        pytest.skip("needs >= 2 GPUs")
    c, ql, ox = small
    G = min(n, 8)
    for ex in (1, 2, 3):
        gx = g.GriffinIndex(c, block_size=128, num_gpus=G, exchange=ex)
        _check(gx, ox, ql, 100)
        gx.close()


def test_launch_config_shared_across_threads(small):
    """Shard launcher threads configure kernels for their block size; that must
    never shrink the shared-memory limit a larger configuration on another
    thread relies on (regression: a per-thread cache did)."""
    c, ql, ox = small
    gx = g.GriffinIndex(c, block_size=64, num_gpus=4, devices=[0] * 4)
    _check(gx, ox, ql, 10)   # worker threads configure B = 64
    big = g.GriffinIndex(c, block_size=128)
    _check(big, ox, ql, 10)  # main thread, larger shared memory per CTA
    _check(gx, ox, ql, 10)
