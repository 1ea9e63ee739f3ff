"""Multi-process (world_size 2 and 3, gloo, CPU) tests of the sharded path's
host logic (T5): shard ranges, the count / halo all-gathers, the offsets, and
the global result = concatenation of the shards' outputs in rank order.

The device steps are replaced by a CPU stand-in built on the oracle
(TEST-ONLY); the product's LibdsLocal runs the same steps in libds kernels
and is exercised on the GPU by tests/test_dist_gpu.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import dsgen
import oracle
from paper_conf_icpp_gomez_lunacshg15_b200.dist import ShardedDS, rebalance_plan, shard_range


class OracleLocal:
    """CPU stand-in for LibdsLocal (tests only): same contract, oracle arithmetic."""

    def alloc_u64(self, k, device):
        return torch.zeros(k, dtype=torch.int64)

    @staticmethod
    def _u32(t):
        return t.numpy().view(np.uint32)

    def compact(self, shard, remove_value, d_count, stream=None):
        d_count[0] = oracle.compact(self._u32(shard), remove_value)

    def select(self, shard, predicate, param, d_count, stream=None):
        d_count[0] = oracle.select(self._u32(shard), predicate, param)

    def halo_entry(self, shard, d_entry, stream=None):
        d_entry[0] = ((1 << 32) | int(self._u32(shard)[-1])) if shard.numel() else 0

    def unique(self, shard, d_halo, halo_len, d_count, stream=None):
        prev = None
        for h in range(halo_len - 1, -1, -1):
            ent = int(d_halo[h])
            if ent >> 32:
                prev = ent & 0xFFFFFFFF
                break
        d_count[0] = oracle.unique(self._u32(shard), prev=prev)

    def offsets(self, d_counts, world, rank, d_result, stream=None):
        c = d_counts.tolist()
        d_result[0] = sum(c[:rank])
        d_result[1] = sum(c)

    def slide(self, shard, n, shift, stream=None):
        oracle.slide(self._u32(shard), n, shift, 4)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, case, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        kind, n, arr_seed = case
        if kind == "unique":
            full = dsgen.unique_runs_input(n, 0.3, arr_seed)
        else:
            full = dsgen.compact_input(n, 0.5, arr_seed)
        lo, hi = shard_range(n, world, rank)
        shard = full[lo:hi].clone()
        ds = ShardedDS(device="cpu", local=OracleLocal())
        if kind == "unique":
            res = ds.unique(shard)
        else:
            res = ds.compact(shard, 0)
        cnt = int(res.count[0])
        q.put((rank, lo, hi, cnt, res.result.tolist(), res.counts.tolist(),
               shard[:cnt].numpy().copy()))
    finally:
        dist.destroy_process_group()


def _run(world, case):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(out, key=lambda x: x[0])


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("case", [("compact", 100_003, 5), ("unique", 50_001, 6),
                                  ("compact", 2, 7), ("unique", 2, 8)])  # n=2: empty shards
def test_sharded_equals_global_oracle(world, case):
    kind, n, seed = case
    out = _run(world, case)
    full = (dsgen.unique_runs_input(n, 0.3, seed) if kind == "unique"
            else dsgen.compact_input(n, 0.5, seed)).numpy().view(np.uint32).copy()
    m = oracle.unique(full) if kind == "unique" else oracle.compact(full, 0)
    counts = [o[3] for o in out]
    for rank, lo, hi, cnt, result, allc, _ in out:
        assert allc == counts                           # all-gather of counts
        assert result == [sum(counts[:rank]), m]         # offset, global out_n
    glob = np.concatenate([o[6].view(np.uint32) for o in out])
    assert np.array_equal(glob, full[:m])                # decomposition property


def test_unique_halo_across_shards():
    """Runs crossing the shard boundary: the second shard's first word must be
    compared with the first shard's last word (R18)."""
    n = 20_000
    out = _run(2, ("unique", n, 9))
    full = dsgen.unique_runs_input(n, 0.3, 9).numpy().view(np.uint32).copy()
    m = oracle.unique(full)
    assert sum(o[3] for o in out) == m


def test_shard_range_partition():
    for n in (0, 1, 7, 100):
        for w in (1, 2, 3, 8):
            rs = [shard_range(n, w, r) for r in range(w)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(w - 1))


# ------------------------------------------------------------ rebalance (8(f)-1)
def _mixed_input(n, fracs, seed):
    """Concatenation of len(fracs) equal blocks with different kept fractions
    (so shards keep very different counts and the waves vary)."""
    k = len(fracs)
    parts = []
    for i, f in enumerate(fracs):
        lo, hi = shard_range(n, k, i)
        parts.append(dsgen.compact_input(hi - lo, f, seed + 31 * i))
    return torch.cat(parts)


def _rebalance_worker(rank, world, port, case, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n, fracs, seed = case
        full = _mixed_input(n, fracs, seed)
        lo, hi = shard_range(n, world, rank)
        shard = full[lo:hi].clone()
        ds = ShardedDS(device="cpu", local=OracleLocal())
        res = ds.compact(shard, 0)
        held = ds.rebalance(shard, res)
        q.put((rank, lo, hi, held, shard[:held].numpy().copy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,case", [
    (2, (100_003, [0.5, 0.5], 11)),
    (3, (60_001, [0.9, 0.1, 0.7], 12)),
    (4, (80_000, [0.0, 1.0, 0.3, 0.6], 13)),
    (4, (40_000, [1.0, 1.0, 1.0, 1.0], 14)),   # nothing moves
    (3, (30_000, [0.0, 0.0, 0.0], 15)),        # nothing kept
    (4, (3, [0.5, 0.5, 0.5], 16)),             # empty shards
])
def test_rebalance_equals_single_array_in_place_result(world, case):
    """After compact + rebalance, rank r holds the global outputs that one
    in-place compaction of the whole array leaves in rank r's index range."""
    ctx = mp.get_context("spawn")
    qq = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rebalance_worker, args=(r, world, port, case, qq)) for r in range(world)]
    for p in procs:
        p.start()
    out = sorted([qq.get(timeout=120) for _ in range(world)], key=lambda x: x[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    n, fracs, seed = case
    full = _mixed_input(n, fracs, seed).numpy().view(np.uint32).copy()
    m = oracle.compact(full, 0)
    for rank, lo, hi, held, data in out:
        exp_held = max(0, min(hi, m) - lo)
        assert held == exp_held
        assert np.array_equal(data.view(np.uint32), full[lo:lo + held])


def test_rebalance_plan_properties():
    """Host plan: pieces only go down, cover exactly the sent outputs, never
    overlap at a destination, and a receiver's wave precedes its senders'."""
    rng = np.random.default_rng(5)
    for _ in range(300):
        G = int(rng.integers(1, 9))
        sizes = [int(x) for x in rng.integers(0, 50, G)]
        counts = [int(rng.integers(0, s + 1)) for s in sizes]
        p = rebalance_plan(counts, sizes)
        B = np.concatenate([[0], np.cumsum(sizes)])
        off = np.concatenate([[0], np.cumsum(counts)])
        cover = {}
        for pc in p.pieces:
            assert pc.dst < pc.src and pc.count > 0
            assert p.wave[pc.dst] < p.wave[pc.src]
            for j in range(pc.count):
                g = off[pc.src] + pc.src_lo + j
                assert B[pc.dst] + pc.dst_lo + j == g          # lands at its global position
                assert pc.dst_lo + j < sizes[pc.dst]
                assert g not in cover
                cover[g] = pc.src
        for r in range(G):
            assert p.shift[r] + p.kept[r] == counts[r]
            for j in range(p.shift[r]):
                assert cover.get(off[r] + j) == r
            assert sum(p.final) == p.total == sum(counts)
