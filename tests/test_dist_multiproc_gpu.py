"""The sharded product path end to end on real kernels (T5, §8(e), 8(f)-1):
several processes, one rank each, ALL on cuda:0, each sliding its shard
with the libds kernels through the product's ShardedDS + LibdsLocal.
Only the transport differs from a multi-GPU box: NCCL cannot put two ranks
on one GPU, so the collectives go through a TEST-ONLY communicator that
stages the 8-byte values and the rebalance pieces through host memory over
gloo (StagedGlooComm, the same all_gather / exchange contract as the
product's DistComm).  Results are compared with the global oracle."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import dsgen
import oracle

pytestmark = pytest.mark.gpu


class StagedGlooComm:
    """Test-only transport: device tensors staged through host memory over gloo."""

    def all_gather(self, out, inp):
        host = inp.cpu()
        parts = [torch.empty_like(host) for _ in range(dist.get_world_size())]
        dist.all_gather(parts, host)
        out.copy_(torch.cat(parts).to(out.device))

    def exchange(self, sends, recvs):
        reqs, staged = [], []
        for t, peer in sends:
            h = t.cpu()
            staged.append(h)
            reqs.append(dist.isend(h, peer))
        for t, peer in recvs:
            h = torch.empty(t.shape, dtype=t.dtype)
            staged.append((t, h))
            reqs.append(dist.irecv(h, peer))
        for r in reqs:
            r.wait()
        for item in staged:
            if isinstance(item, tuple):
                item[0].copy_(item[1].to(item[0].device))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _global_input(kind, n, fracs, seed):
    """Concatenated blocks with different kept fractions (host tensor)."""
    k = len(fracs)
    parts = []
    for i, f in enumerate(fracs):
        lo = i * (n // k)
        hi = n if i == k - 1 else lo + n // k
        if kind == "unique":
            parts.append(dsgen.unique_runs_input(hi - lo, f, seed + 31 * i))
        elif kind == "select":
            parts.append(dsgen.select_input(hi - lo, seed + 31 * i))
        else:
            parts.append(dsgen.compact_input(hi - lo, f, seed + 31 * i))
    return torch.cat(parts)


SELECT_T = dsgen.select_threshold(0.4) & 0xFFFFFFFF


def _worker(rank, world, port, case, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icpp_gomez_lunacshg15_b200 import libds
        from paper_conf_icpp_gomez_lunacshg15_b200.dist import LibdsLocal, ShardedDS, shard_range
        torch.cuda.set_device(0)
        kind, n, fracs, seed, use_stream, exchange = case
        full = _global_input(kind, n, fracs, seed)
        lo, hi = shard_range(n, world, rank)
        shard = full[lo:hi].clone().cuda()
        stream = torch.cuda.Stream() if use_stream else None
        ds = ShardedDS(device="cuda", local=LibdsLocal(), comm=StagedGlooComm(), count_exchange=exchange)
        if kind == "unique":
            res = ds.unique(shard, stream=stream)
        elif kind == "select":
            res = ds.select(shard, libds.DS_PRED_I32_GT, SELECT_T, stream=stream)
        else:
            res = ds.compact(shard, 0, stream=stream)
        if stream is not None:
            stream.synchronize()
        cnt = int(res.count[0])
        ragged = shard[:cnt].cpu().numpy().copy()
        result = res.result.tolist()
        counts = res.counts.tolist()
        held = ds.rebalance(shard, res, stream=stream)
        torch.cuda.synchronize()
        if exchange == "board":  # a second call on the same board (the other slot), then unmap
            again = shard.clone()
            res2 = ds.compact(again, 0, stream=stream) if kind != "unique" else ds.unique(again, stream=stream)
            torch.cuda.synchronize()
            c2 = res2.counts.tolist()
            assert c2[rank] == int(res2.count[0]) and res2.result.tolist() == [sum(c2[:rank]), sum(c2)]
            ds.close()
        q.put((rank, lo, hi, cnt, result, counts, ragged, held, shard[:held].cpu().numpy().copy()))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, "error", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


def _run(world, case):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
    errs = [o for o in out if o[1] == "error"]
    assert not errs, errs
    for p in procs:
        assert p.exitcode == 0
    return sorted(out, key=lambda x: x[0])


CASES = [
    (2, ("compact", 3_000_001, [0.5, 0.5], 41, False)),
    (3, ("compact", 2_000_003, [0.9, 0.1, 0.6], 42, True)),
    (4, ("compact", 1_000_000, [0.0, 1.0, 0.3, 0.7], 43, False)),
    (2, ("unique", 2_000_001, [0.3, 0.8], 44, True)),
    (4, ("unique", 500_001, [0.0, 0.5, 0.0, 1.0], 45, False)),
    (3, ("select", 1_500_007, [0.5, 0.5, 0.5], 46, True)),
    (4, ("compact", 5, [0.5], 47, False)),   # tiny: empty shards
]


@pytest.mark.parametrize("exchange", ["collective", "board"])
@pytest.mark.parametrize("world,case", CASES)
def test_sharded_product_path_on_gpu(world, case, exchange):
    """ShardedDS (LibdsLocal kernels, count / halo all-gathers, ds_shard_offsets)
    then ShardedDS.rebalance (wave-scheduled pieces + ds_slide) against the
    global oracle: ragged layout = concatenation of the shard outputs, and the
    rebalanced layout = the single in-place DS of the whole array.  exchange
    "board": the counts go through the count boards (each shard's DS kernel
    stores its count into every rank's board via CUDA IPC mappings) instead of
    the all-gather; a second call then uses the boards' other slot."""
    kind, n, fracs, seed, _ = case
    out = _run(world, case + (exchange,))
    full = _global_input(kind, n, fracs, seed).numpy().view(np.uint32).copy()
    if kind == "unique":
        m = oracle.unique(full)
    elif kind == "select":
        m = oracle.select(full, oracle.PRED_I32_GT, SELECT_T)
    else:
        m = oracle.compact(full, 0)
    counts = [o[3] for o in out]
    assert sum(counts) == m
    for rank, lo, hi, cnt, result, allc, ragged, held, data in out:
        assert allc == counts                                   # count all-gather
        assert result == [sum(counts[:rank]), m]                # ds_shard_offsets
        off = sum(counts[:rank])
        assert np.array_equal(ragged.view(np.uint32), full[off:off + cnt])   # ragged layout
        exp_held = max(0, min(hi, m) - lo)
        assert held == exp_held                                  # rebalanced layout
        assert np.array_equal(data.view(np.uint32), full[lo:lo + held])
