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
    all_keys = torch.empty((world,) + tuple(keys.shape), dtype=keys.dtype, device=keys.device)
    all_cnts = torch.empty((world,) + tuple(counts.shape), dtype=counts.dtype, device=counts.device)
    if keys.is_cuda:
        dist.all_gather_into_tensor(all_keys.view(-1), keys.contiguous().view(-1), group=group)
        dist.all_gather_into_tensor(all_cnts.view(-1), counts.contiguous().view(-1), group=group)
    else:  # gloo (CPU tests): list form
        dist.all_gather(list(all_keys.unbind(0)), keys.contiguous(), group=group)
        dist.all_gather(list(all_cnts.unbind(0)), counts.contiguous(), group=group)
    return all_keys, all_cnts


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
