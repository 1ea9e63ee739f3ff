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

Optional rebalance: ``rebalance`` turns the ragged
layout into the contiguous one -- global output g lands where input word g
lived, i.e. exactly what one in-place DS of the whole distributed array
would leave (rank r holds outputs [B_r, B_{r+1}) clipped to out_n, B_r the
shard starts).  Every output moves to a lower or equal global position
(out(p) <= p), so data only flows to lower ranks: each rank sends its
first min(c_r, d_r) outputs (d_r = B_r - off_r >= 0) to the ranks below,
closes the gap with one in-place regular DS (ds_slide by d_r), then
receives from higher ranks.  A rank may receive only after its own send
and slide, so the ranks go in "waves" (wave = 1 + the largest wave of the
ranks it sends to); each wave is one batch of NCCL send/recv over NVLink.

The device steps are delegated to a ``local`` object; the default,
``LibdsLocal``, calls the libds C ABI on CUDA tensors.  The two collectives
(all-gather of 8-byte values, the rebalance's point-to-point pieces) go
through a ``comm`` object; the default, ``DistComm``, runs them on the
process group (NCCL over NVLink on a GPU box) on the device tensors.  Tests
substitute a CPU stand-in for ``local`` (orchestration over gloo) and a
CPU-staged gloo ``comm`` (the real kernels, several ranks on one GPU).

Stream ordering: every call takes the stream the libds kernels run on (None
= torch's current stream).  The collectives are issued with that stream
current, so they start after the kernels before them on it, and the work
after them on it (offsets kernel, slide) waits for them.
"""
from __future__ import annotations

import bisect
import contextlib
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

    def slide(self, shard, n, shift, stream=None):
        self.libds.ds_slide_ex(shard if n else None, n, shift, 4, stream)

    # Count boards (fused count publication over peer memory).
    def board_alloc(self, world):
        return self.libds.ds_board_alloc(world)

    def board_free(self, board):
        self.libds.ds_board_free(board)

    def board_handle(self, board):
        return self.libds.ds_board_ipc_handle(board)

    def board_open(self, handle):
        return self.libds.ds_board_ipc_open(handle)

    def board_close(self, peer):
        self.libds.ds_board_ipc_close(peer)

    def compact_pub(self, shard, remove_value, d_count, pub, stream=None):
        self.libds.ds_compact_pub_ex(shard if shard.numel() else None, shard.numel(), remove_value, d_count,
                                     *pub, stream)

    def select_pub(self, shard, predicate, param, d_count, pub, stream=None):
        self.libds.ds_select_pub_ex(shard if shard.numel() else None, shard.numel(), predicate, param, d_count,
                                    *pub, stream)

    def unique_pub(self, shard, d_halo, halo_len, d_count, pub, stream=None):
        self.libds.ds_unique_pub_ex(shard if shard.numel() else None, shard.numel(), d_halo if halo_len else None,
                                    halo_len, d_count, *pub, stream)

    def board_offsets(self, board, world, rank, tag, d_counts, d_result, stream=None):
        self.libds.ds_shard_offsets_board(board, world, rank, tag, d_counts, d_result, stream)


class DistComm:
    """Collectives on the process group, on device tensors (NCCL on a GPU box).
    Issued with the caller's stream current (ShardedDS), so torch orders the
    NCCL stream after it and, through req.wait(), it after the NCCL stream."""

    def __init__(self, group=None):
        self.group = group

    def all_gather(self, out: torch.Tensor, inp: torch.Tensor) -> None:
        dist.all_gather_into_tensor(out, inp, group=self.group)

    def exchange(self, sends, recvs) -> None:
        """sends / recvs: lists of (tensor, peer rank); one batched round."""
        ops = [dist.P2POp(dist.isend, t, peer, self.group) for t, peer in sends]
        ops += [dist.P2POp(dist.irecv, t, peer, self.group) for t, peer in recvs]
        if ops:
            for req in dist.batch_isend_irecv(ops):
                req.wait()


@dataclass(frozen=True)
class Piece:
    """count words of rank src's local [src_lo, ...) -> rank dst's local [dst_lo, ...)."""
    src: int
    src_lo: int
    dst: int
    dst_lo: int
    count: int


@dataclass
class RebalancePlan:
    pieces: list          # every transfer between ranks
    shift: list           # per rank: ds_slide shift (min(c_r, d_r)); 0 = no slide
    kept: list            # per rank: words kept locally (c_r - shift)
    wave: list            # per rank: the wave in which it sends and slides
    final: list           # per rank: words holding outputs after the rebalance
    total: int

    @property
    def waves(self) -> int:
        return max(self.wave) + 1 if self.wave else 0


def rebalance_plan(counts: list[int], sizes: list[int]) -> RebalancePlan:
    """Host-side schedule of the rebalance from every shard's kept count and
    capacity (pure function of the all-gathered counts; the same on every rank)."""
    G = len(counts)
    assert len(sizes) == G and all(0 <= c <= s for c, s in zip(counts, sizes))
    B = [0] * (G + 1)
    off = [0] * (G + 1)
    for r in range(G):
        B[r + 1] = B[r] + sizes[r]
        off[r + 1] = off[r] + counts[r]
    total = off[G]
    pieces, shift, kept = [], [], []
    for r in range(G):
        d = B[r] - off[r]                      # >= 0: off_r <= B_r
        assert d >= 0
        down = min(counts[r], d)
        shift.append(down)
        kept.append(counts[r] - down)
        g, end = off[r], off[r] + down        # global range going below rank r
        while g < end:
            q = bisect.bisect_right(B, g) - 1     # B[q] <= g < B[q+1] (skips empty shards)
            n = min(end, B[q + 1]) - g
            pieces.append(Piece(r, g - off[r], q, g - B[q], n))
            g += n
    wave = [0] * G
    for r in range(G):                         # destinations are lower ranks: ascending order works
        dests = [p.dst for p in pieces if p.src == r]
        wave[r] = 1 + max(wave[q] for q in dests) if dests else 0
    final = [max(0, min(sizes[r], total - B[r])) for r in range(G)]
    return RebalancePlan(pieces, shift, kept, wave, final, total)


@dataclass
class ShardResult:
    count: torch.Tensor    # [1] kept words of this shard (device int64)
    result: torch.Tensor   # [2] (global offset of this shard, global out_n)
    counts: torch.Tensor   # [world] all shards' counts


class ShardedDS:
    """One rank's view of a sharded in-place DS operation."""

    def __init__(self, group=None, device=None, local=None, comm=None, count_exchange="collective"):
        """count_exchange: "collective" -- the counts travel by an all-gather
        (NCCL); "board" -- each shard's DS kernel writes its count straight into
        every rank's count board (peer memory mapped by CUDA IPC, NVLink between
        GPUs) and ds_shard_offsets_board reads the local board: no all-gather
        launch.  The board is set up once here (IPC handles exchanged over the
        process group)."""
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.device = torch.device(device) if device is not None else torch.device("cuda")
        self.local = local if local is not None else LibdsLocal()
        self.comm = comm if comm is not None else DistComm(group)
        if count_exchange not in ("collective", "board"):
            raise ValueError("count_exchange is 'collective' or 'board'")
        self.count_exchange = count_exchange
        self._board = None
        self._peers = []
        self._tag = 0
        self.d_count = self.local.alloc_u64(1, self.device)
        self.d_counts = self.local.alloc_u64(self.world, self.device)
        self.d_result = self.local.alloc_u64(2, self.device)
        self.d_entry = self.local.alloc_u64(1, self.device)
        self.d_halo = self.local.alloc_u64(self.world, self.device)
        self._sizes = None  # every rank's shard capacity (rebalance), gathered once
        if count_exchange == "board":
            self._board_setup()

    def _board_setup(self):
        self._board = self.local.board_alloc(self.world)
        handle = self.local.board_handle(self._board)
        if self.world > 1:
            handles = [None] * self.world
            dist.all_gather_object(handles, handle, group=self.group)
        else:
            handles = [handle]
        ptrs = []
        for r, h in enumerate(handles):
            if r == self.rank:
                ptrs.append(self._board)
            else:
                p = self.local.board_open(h)
                self._peers.append(p)
                ptrs.append(p)
        self.d_boards = torch.tensor(ptrs, dtype=torch.int64, device=self.device)

    def close(self):
        """Unmap the peers' boards and free this rank's (board mode)."""
        if self._board is not None:
            torch.cuda.synchronize(self.device)
            if self.world > 1:
                dist.barrier(group=self.group)  # no peer writes into this board any more
            for p in self._peers:
                self.local.board_close(p)
            self.local.board_free(self._board)
            self._board, self._peers = None, []

    def _pub(self):
        self._tag += 1
        return (self.d_boards, self.world, self.rank, self._tag)

    def _finish_board(self, stream) -> ShardResult:
        self.local.board_offsets(self._board, self.world, self.rank, self._tag, self.d_counts, self.d_result, stream)
        return ShardResult(self.d_count, self.d_result, self.d_counts)

    @staticmethod
    def _on(stream):
        """Issue torch work (collectives, copies) on the libds stream."""
        if isinstance(stream, torch.cuda.Stream):
            return torch.cuda.stream(stream)
        if stream is not None:
            raise TypeError("ShardedDS needs a torch.cuda.Stream (or None for the current stream)")
        return contextlib.nullcontext()

    def _allgather(self, out: torch.Tensor, inp: torch.Tensor, stream=None) -> None:
        with self._on(stream):
            if self.world == 1:
                out.copy_(inp)
            else:
                self.comm.all_gather(out, inp)

    def _finish(self, stream) -> ShardResult:
        self._allgather(self.d_counts, self.d_count, stream)
        self.local.offsets(self.d_counts, self.world, self.rank, self.d_result, stream)
        return ShardResult(self.d_count, self.d_result, self.d_counts)

    def compact(self, shard: torch.Tensor, remove_value: int, stream=None) -> ShardResult:
        if self._board is not None:
            self.local.compact_pub(shard, remove_value, self.d_count, self._pub(), stream)
            return self._finish_board(stream)
        self.local.compact(shard, remove_value, self.d_count, stream)
        return self._finish(stream)

    def select(self, shard: torch.Tensor, predicate: int, param: int = 0, stream=None) -> ShardResult:
        if self._board is not None:
            self.local.select_pub(shard, predicate, param, self.d_count, self._pub(), stream)
            return self._finish_board(stream)
        self.local.select(shard, predicate, param, self.d_count, stream)
        return self._finish(stream)

    def rebalance(self, shard: torch.Tensor, res: ShardResult, stream=None) -> int:
        """Contiguous global layout after a sharded compact/select/unique
        (module docstring).  Returns the number of outputs this rank holds
        at shard[0, ret); words past it are unspecified.  Host-synchronising
        (the plan needs the counts on the host)."""
        with self._on(stream):
            counts = [int(c) for c in res.counts.tolist()]  # host sync on the libds stream
        if self._sizes is None:
            mine = torch.tensor([shard.numel()], dtype=torch.int64, device=self.device)
            allsz = torch.zeros(self.world, dtype=torch.int64, device=self.device)
            self._allgather(allsz, mine, stream)
            with self._on(stream):
                self._sizes = [int(x) for x in allsz.tolist()]
        plan = rebalance_plan(counts, self._sizes)
        me = self.rank
        for w in range(plan.waves):
            sends, recvs = [], []
            if plan.wave[me] == w:
                sends = [(shard[pc.src_lo:pc.src_lo + pc.count], pc.dst) for pc in plan.pieces if pc.src == me]
            recvs = [(shard[pc.dst_lo:pc.dst_lo + pc.count], pc.src) for pc in plan.pieces
                     if pc.dst == me and plan.wave[pc.src] == w]
            if sends or recvs:
                # sends read, receives write the shard: both after the kernels
                # before them on the stream, and the slide below after both
                with self._on(stream):
                    self.comm.exchange(sends, recvs)
            if plan.wave[me] == w and plan.shift[me] and plan.kept[me]:
                self.local.slide(shard, counts[me], plan.shift[me], stream)
        return plan.final[me]

    def unique(self, shard: torch.Tensor, stream=None) -> ShardResult:
        # Halo exchange before the slide (unique never changes a shard's last
        # word, but every rank must read its neighbour's value, R18).
        self.local.halo_entry(shard, self.d_entry, stream)
        self._allgather(self.d_halo, self.d_entry, stream)
        if self._board is not None:
            self.local.unique_pub(shard, self.d_halo, self.rank, self.d_count, self._pub(), stream)
            return self._finish_board(stream)
        self.local.unique(shard, self.d_halo, self.rank, self.d_count, stream)
        return self._finish(stream)
