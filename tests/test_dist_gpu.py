"""Sharded path on one GPU (T5 "fake shards"): one array split into G
contiguous sub-ranges, each slid in place by the libds kernels; the halo
entries and counts that NCCL would all-gather are gathered into device
arrays directly, then ds_shard_offsets produces offsets and out_n.  The
concatenation of the shards' outputs must equal the global oracle result."""
import numpy as np
import pytest
import torch

import dsgen
import oracle
from paper_conf_icpp_gomez_lunacshg15_b200 import libds
from paper_conf_icpp_gomez_lunacshg15_b200.dist import ShardedDS, shard_range

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("G", [1, 2, 3, 8])
@pytest.mark.parametrize("kind", ["compact", "unique", "select"])
@pytest.mark.parametrize("n", [5, 123_457, 3_000_001])
def test_fake_shards(G, kind, n):
    if kind == "unique":
        full = dsgen.unique_runs_input(n, 0.4, 17 + G, device="cuda")
    elif kind == "select":
        full = dsgen.select_input(n, 18 + G, device="cuda")
    else:
        full = dsgen.compact_input(n, 0.5, 19 + G, device="cuda")
    host = full.cpu().numpy().view(np.uint32).copy()
    t = dsgen.select_threshold(0.3) & 0xFFFFFFFF
    if kind == "unique":
        m = oracle.unique(host)
    elif kind == "select":
        m = oracle.select(host, oracle.PRED_I32_GT, t)
    else:
        m = oracle.compact(host, 0)

    halo = torch.zeros(G, dtype=torch.int64, device="cuda")
    counts = torch.zeros(G, dtype=torch.int64, device="cuda")
    shards = []
    for r in range(G):
        lo, hi = shard_range(n, G, r)
        shards.append(full[lo:hi])
        libds.ds_halo_entry(full[lo:hi] if hi > lo else None, hi - lo, halo[r:r + 1], None)
    for r, sh in enumerate(shards):
        ptr = sh if sh.numel() else None
        if kind == "unique":
            libds.ds_unique_ex(ptr, sh.numel(), halo if r else None, r, counts[r:r + 1], None)
        elif kind == "select":
            libds.ds_select_ex(ptr, sh.numel(), libds.DS_PRED_I32_GT, t, counts[r:r + 1], None)
        else:
            libds.ds_compact_ex(ptr, sh.numel(), 0, counts[r:r + 1], None)
    res = torch.zeros(2 * G, dtype=torch.int64, device="cuda")
    for r in range(G):
        libds.ds_shard_offsets(counts, G, r, res[2 * r:2 * r + 2], None)
    torch.cuda.synchronize()
    c = counts.tolist()
    rr = res.view(G, 2).tolist()
    assert sum(c) == m
    for r in range(G):
        assert rr[r] == [sum(c[:r]), m]
    glob = np.concatenate([shards[r][:c[r]].cpu().numpy().view(np.uint32) for r in range(G)])
    assert np.array_equal(glob, host[:m])


def test_sharded_ds_world1_on_gpu():
    """The ShardedDS driver itself (no process group: world 1) on CUDA."""
    n = 1_000_003
    a = dsgen.compact_input(n, 0.5, 3, device="cuda")
    host = a.cpu().numpy().view(np.uint32).copy()
    m = oracle.compact(host, 0)
    ds = ShardedDS(device="cuda")
    res = ds.compact(a, 0)
    torch.cuda.synchronize()
    assert int(res.count[0]) == m and res.result.tolist() == [0, m]
    assert np.array_equal(a.cpu().numpy().view(np.uint32), host)


@pytest.mark.parametrize("G,fracs", [(2, [0.5, 0.5]), (4, [0.9, 0.1, 0.0, 1.0]), (8, [0.5] * 8),
                                     (3, [0.0, 0.7, 0.2])])
def test_fake_shard_rebalance(G, fracs):
    """Rebalance plan executed on one GPU in one process: the NCCL send/recv of
    each wave replaced by device copies between the fake shards, the gap
    closed by the real ds_slide kernel.  Result: the single-array in-place
    compaction.  (The product's ShardedDS.rebalance itself runs, with real
    kernels and one process per rank, in tests/test_dist_multiproc_gpu.py.)"""
    from paper_conf_icpp_gomez_lunacshg15_b200.dist import rebalance_plan
    n = 2_000_003
    parts = []
    for i, f in enumerate(fracs):
        lo, hi = shard_range(n, len(fracs), i)
        parts.append(dsgen.compact_input(hi - lo, f, 50 + i, device="cuda"))
    full = torch.cat(parts)
    host = full.cpu().numpy().view(np.uint32).copy()
    m = oracle.compact(host, 0)
    shards, counts = [], torch.zeros(G, dtype=torch.int64, device="cuda")
    for r in range(G):
        lo, hi = shard_range(n, G, r)
        shards.append(full[lo:hi])
        libds.ds_compact_ex(full[lo:hi], hi - lo, 0, counts[r:r + 1], None)
    c = [int(x) for x in counts.tolist()]
    plan = rebalance_plan(c, [s.numel() for s in shards])
    for w in range(plan.waves):
        for r in range(G):
            if plan.wave[r] != w:
                continue
            for pc in plan.pieces:
                if pc.src == r:
                    shards[pc.dst][pc.dst_lo:pc.dst_lo + pc.count].copy_(
                        shards[r][pc.src_lo:pc.src_lo + pc.count])
            if plan.shift[r] and plan.kept[r]:
                libds.ds_slide_ex(shards[r], c[r], plan.shift[r], 4, None)
    torch.cuda.synchronize()
    got = full.cpu().numpy().view(np.uint32)
    assert plan.total == m
    assert np.array_equal(got[:m], host[:m])


def test_sharded_ds_world1_board():
    """Count-board mode without a process group (world 1: the rank's own board)."""
    n = 1_000_003
    a = dsgen.compact_input(n, 0.3, 4, device="cuda")
    host = a.cpu().numpy().view(np.uint32).copy()
    m = oracle.compact(host.copy(), 0)
    ds = ShardedDS(device="cuda", count_exchange="board")
    for rep in range(3):  # three calls: both slots and a reuse of the first
        b = torch.from_numpy(host.copy().view(np.int32)).cuda() if rep else a
        res = ds.compact(b, 0)
        torch.cuda.synchronize()
        assert res.result.tolist() == [0, m] and res.counts.tolist() == [m]
    ds.close()
