"""Sharded in-place Data Sliding across GPUs.

The array is split into contiguous shards, one per rank (one process per
GPU).  Every rank slides its own shard in place with the single-GPU libds
kernels -- there is no inter-GPU dependency during the slide, because each
shard's in-place hazards are internal to it.  One tiny exchange follows:
an all-gather of the per-shard kept counts (8 bytes per rank, NCCL over
NVLink), from which libds' ds_shard_offsets kernel derives this shard's
global output offset and the global out_n.  The global result is the
concatenation, in rank order, of every shard's [0, count) prefix.

Unique needs one more 8-byte all-gather *before* the slide: each shard's
(non-empty, last word) "halo" entry, so that a shard's first word is
compared with the last word of the nearest non-empty earlier shard (R18).

The device steps are delegated to a ``local`` object; the default,
``LibdsLocal``, calls the libds C ABI on CUDA tensors.  Tests substitute a
CPU stand-in to exercise the orchestration and the collectives with gloo.
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as dist


def shard_range(n_total: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous shard [lo, hi) of rank; the remainder goes to the last rank."""
    base = n_total // world
    lo = rank * base
    hi = n_total if rank == world - 1 else lo + base
    return lo, hi


class LibdsLocal:
    """Device steps on CUDA tensors through the libds C ABI."""

    def __init__(self):
        from . import libds
        self.libds = libds

    def alloc_u64(self, k: int, device) -> torch.Tensor:
        return torch.zeros(k, dtype=torch.int64, device=device)

    def compact(self, shard, remove_value, d_count, stream=None):
        self.libds.ds_compact_ex(shard, shard.numel(), remove_value, d_count, stream)

    def select(self, shard, predicate, param, d_count, stream=None):
        self.libds.ds_select_ex(shard, shard.numel(), predicate, param, d_count, stream)

    def halo_entry(self, shard, d_entry, stream=None):
        self.libds.ds_halo_entry(shard if shard.numel() else None, shard.numel(), d_entry, stream)

    def unique(self, shard, d_halo, halo_len, d_count, stream=None):
        self.libds.ds_unique_ex(shard if shard.numel() else None, shard.numel(),
                                d_halo if halo_len else None, halo_len, d_count, stream)

    def offsets(self, d_counts, world, rank, d_result, stream=None):
        self.libds.ds_shard_offsets(d_counts, world, rank, d_result, stream)


@dataclass
class ShardResult:
    count: torch.Tensor    # [1] kept words of this shard (device int64)
    result: torch.Tensor   # [2] (global offset of this shard, global out_n)
    counts: torch.Tensor   # [world] all shards' counts


class ShardedDS:
    """One rank's view of a sharded in-place DS operation."""

    def __init__(self, group=None, device=None, local=None):
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.device = torch.device(device) if device is not None else torch.device("cuda")
        self.local = local if local is not None else LibdsLocal()
        self.d_count = self.local.alloc_u64(1, self.device)
        self.d_counts = self.local.alloc_u64(self.world, self.device)
        self.d_result = self.local.alloc_u64(2, self.device)
        self.d_entry = self.local.alloc_u64(1, self.device)
        self.d_halo = self.local.alloc_u64(self.world, self.device)

    def _allgather(self, out: torch.Tensor, inp: torch.Tensor) -> None:
        if self.world == 1:
            out.copy_(inp)
        else:
            dist.all_gather_into_tensor(out, inp, group=self.group)

    def _finish(self, stream) -> ShardResult:
        self._allgather(self.d_counts, self.d_count)
        self.local.offsets(self.d_counts, self.world, self.rank, self.d_result, stream)
        return ShardResult(self.d_count, self.d_result, self.d_counts)

    def compact(self, shard: torch.Tensor, remove_value: int, stream=None) -> ShardResult:
        self.local.compact(shard, remove_value, self.d_count, stream)
        return self._finish(stream)

    def select(self, shard: torch.Tensor, predicate: int, param: int = 0, stream=None) -> ShardResult:
        self.local.select(shard, predicate, param, self.d_count, stream)
        return self._finish(stream)

    def unique(self, shard: torch.Tensor, stream=None) -> ShardResult:
        # Halo exchange before the slide (unique never changes a shard's last
        # word, but every rank must read its neighbour's value, R18).
        self.local.halo_entry(shard, self.d_entry, stream)
        self._allgather(self.d_halo, self.d_entry)
        self.local.unique(shard, self.d_halo, self.rank, self.d_count, stream)
        return self._finish(stream)
