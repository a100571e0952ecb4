"""docID-range sharded search over one process per GPU.

Plumbing only: each rank owns one `griffin_index` shard (docIDs
[g*ceil(N/G), min(N,(g+1)*ceil(N/G)))); the per-shard top-k keys/counts of a
batch are exchanged with `torch.distributed` (NCCL on GPUs) and the global
top-k is produced by the library's k-way merge kernel
(`griffin_merge_topk_device`).  No arithmetic of the method lives here.
"""
from __future__ import annotations

from typing import Optional

import torch
import torch.distributed as dist


def gather_runs(keys: torch.Tensor, counts: torch.Tensor, group=None):
    """All-gather per-shard runs into the g-major layout the merge kernel takes:
    keys [G, nq*k] (int64 bit patterns of u64 keys), counts [G, nq]."""
    world = dist.get_world_size(group)
    if keys.is_cuda and dist.get_backend(group) == "gloo":   # gloo: exchange through host memory
        ak, ac = gather_runs(keys.cpu(), counts.cpu(), group)
        return ak.to(keys.device), ac.to(counts.device)
    all_keys = torch.empty((world,) + tuple(keys.shape), dtype=keys.dtype, device=keys.device)
    all_cnts = torch.empty((world,) + tuple(counts.shape), dtype=counts.dtype, device=counts.device)
    if keys.is_cuda:
        dist.all_gather_into_tensor(all_keys.view(-1), keys.contiguous().view(-1), group=group)
        dist.all_gather_into_tensor(all_cnts.view(-1), counts.contiguous().view(-1), group=group)
    else:  # gloo (CPU tests): list form
        dist.all_gather(list(all_keys.unbind(0)), keys.contiguous(), group=group)
        dist.all_gather(list(all_cnts.unbind(0)), counts.contiguous(), group=group)
    return all_keys, all_cnts


def query_slices(nq: int, world: int):
    """Query slice owned by each rank in the query-sliced exchange: rank r merges
    queries [r*ceil(nq/G), min(nq, (r+1)*ceil(nq/G)))."""
    step = (nq + world - 1) // world if world else 0
    return [(min(nq, r * step), min(nq, (r + 1) * step)) for r in range(world)]


def exchange_sliced(keys: torch.Tensor, counts: torch.Tensor, k: int, group=None):
    """Query-sliced exchange: every rank sends the
    per-shard runs of query slice s to rank s (one all-to-all) and receives the G
    runs of its own slice in the g-major layout the merge kernel takes:
    keys [G, m*k], counts [G, m] with m = its slice length.  Received bytes per
    rank drop from (G-1)*Q*k*8 (all-gather) to about (G-1)/G*Q*k*8.
    Returns (keys, counts, (q_lo, q_hi))."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    if keys.is_cuda and dist.get_backend(group) == "gloo":   # gloo: exchange through host memory
        ak, ac, lh = exchange_sliced(keys.cpu(), counts.cpu(), k, group)
        return ak.to(keys.device), ac.to(counts.device), lh
    nq = counts.numel()
    sl = query_slices(nq, world)
    lo, hi = sl[rank]
    m = hi - lo
    in_k = [(b - a) * k for a, b in sl]
    in_c = [b - a for a, b in sl]
    all_keys = torch.empty((world, m * k), dtype=keys.dtype, device=keys.device)
    all_cnts = torch.empty((world, m), dtype=counts.dtype, device=counts.device)
    dist.all_to_all_single(all_keys.view(-1), keys.contiguous().view(-1),
                           output_split_sizes=[m * k] * world, input_split_sizes=in_k,
                           group=group)
    dist.all_to_all_single(all_cnts.view(-1), counts.contiguous().view(-1),
                           output_split_sizes=[m] * world, input_split_sizes=in_c, group=group)
    return all_keys, all_cnts, (lo, hi)


class ShardedSearcher:
    """One rank's view: its shard index + the exchange + merge."""

    def __init__(self, corpus, block_size: int = 128, device: Optional[int] = None, group=None):
        from . import GriffinIndex
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        dev = torch.cuda.current_device() if device is None else device
        self.ix = GriffinIndex(corpus, block_size=block_size, device=dev,
                               shard_index=self.rank, num_shards=self.world)

    @classmethod
    def from_index(cls, ix, group=None) -> "ShardedSearcher":
        """Wrap an already built shard index (shard_index == this rank)."""
        self = cls.__new__(cls)
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.ix = ix
        return self

    def search(self, d_offsets, d_terms, max_terms: int, k: int, stream=None):
        """Batch search; returns (docids int32 [nq,k] bit-patterns of u32, scores f32 [nq,k],
        counts int32 [nq]) — the global top-k, identical on every rank."""
        nq = d_offsets.numel() - 1
        dev = d_offsets.device
        keys = torch.zeros(nq * k, dtype=torch.int64, device=dev)
        cnts = torch.zeros(nq, dtype=torch.int32, device=dev)
        self.ix.griffin_query_batch_device(d_offsets, d_terms, max_terms, k, keys, cnts, stream)
        if self.world > 1:
            all_keys, all_cnts = gather_runs(keys, cnts, self.group)
            out_k = torch.zeros(nq * k, dtype=torch.int64, device=dev)
            out_c = torch.zeros(nq, dtype=torch.int32, device=dev)
            self.ix.griffin_merge_topk_device(self.world, nq, k, all_keys, all_cnts, out_k, out_c,
                                              stream)
            keys, cnts = out_k, out_c
        dd = torch.empty(nq * k, dtype=torch.int32, device=dev)
        ds = torch.empty(nq * k, dtype=torch.float32, device=dev)
        self.ix.griffin_keys_to_results_device(nq, k, keys, cnts, dd, ds, stream)
        return dd.view(nq, k), ds.view(nq, k), cnts

    def search_sliced(self, d_offsets, d_terms, max_terms: int, k: int, stream=None):
        """Batch search with the query-sliced exchange: returns (q_lo, q_hi, docids,
        scores, counts) — the global top-k of queries [q_lo, q_hi) only, merged on
        this rank (each rank answers its own slice; nothing is all-gathered)."""
        nq = d_offsets.numel() - 1
        dev = d_offsets.device
        keys = torch.zeros(nq * k, dtype=torch.int64, device=dev)
        cnts = torch.zeros(nq, dtype=torch.int32, device=dev)
        self.ix.griffin_query_batch_device(d_offsets, d_terms, max_terms, k, keys, cnts, stream)
        if self.world > 1:
            ak, ac, (lo, hi) = exchange_sliced(keys, cnts, k, self.group)
            m = hi - lo
            keys = torch.zeros(m * k, dtype=torch.int64, device=dev)
            cnts = torch.zeros(m, dtype=torch.int32, device=dev)
            if m:
                self.ix.griffin_merge_topk_device(self.world, m, k, ak, ac, keys, cnts, stream)
        else:
            lo, hi, m = 0, nq, nq
        dd = torch.empty(m * k, dtype=torch.int32, device=dev)
        ds = torch.empty(m * k, dtype=torch.float32, device=dev)
        if m:
            self.ix.griffin_keys_to_results_device(m, k, keys, cnts, dd, ds, stream)
        return lo, hi, dd.view(m, k), ds.view(m, k), cnts


class ReplicatedSearcher:
    """Replicated-index throughput mode: when the index
    fits one GPU every rank holds all of it and answers its own queries; there is
    no exchange on the data path."""

    def __init__(self, corpus, block_size: int = 128, device: Optional[int] = None):
        from . import GriffinIndex
        dev = torch.cuda.current_device() if device is None else device
        self.ix = GriffinIndex(corpus, block_size=block_size, device=dev)

    def search(self, d_offsets, d_terms, max_terms: int, k: int, stream=None):
        nq = d_offsets.numel() - 1
        dev = d_offsets.device
        keys = torch.zeros(nq * k, dtype=torch.int64, device=dev)
        cnts = torch.zeros(nq, dtype=torch.int32, device=dev)
        self.ix.griffin_query_batch_device(d_offsets, d_terms, max_terms, k, keys, cnts, stream)
        dd = torch.empty(nq * k, dtype=torch.int32, device=dev)
        ds = torch.empty(nq * k, dtype=torch.float32, device=dev)
        self.ix.griffin_keys_to_results_device(nq, k, keys, cnts, dd, ds, stream)
        return dd.view(nq, k), ds.view(nq, k), cnts
