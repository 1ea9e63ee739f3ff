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
from paper_conf_icpp_gomez_lunacshg15_b200.dist import ShardedDS, shard_range


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
