"""bench.py -- libds on B200: effective HBM GB/s of the in-place Data Sliding path.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl libds|reference]
                    [--no-rows] [--no-e2e] [--no-cpu]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 \\
        --master-port P bench.py --gpus N ...

Headline (BASELINE.json configs[4], C5): sharded in-place stream compaction of
4G int32 words (2^32, 16 GiB), 50 % kept, contiguous shards over N GPUs
(strong scaling).  One step = on every rank: ds_compact_ex on its shard (the
irregular DS kernel), NCCL all-gather of the 8-byte
counts, ds_shard_offsets (global offset + out_n).  Between steps, outside the
timed events, the pristine shard is restored (D2D copy) and L2 is flushed by
reading a 512 MiB buffer.  value = sum over ranks of 4*(n_r + out_r) bytes /
max-over-ranks device time of the step.

rows (N == 1 only): the other BASELINE configs through the same C ABI --
C1 compact 1M (flushed and L2-hot kernel time, blocking-API wall time, the
oracle in seconds), C2 pad / unpad 4000x3990 <-> 4000, pad / unpad at >= 256M
elements (16384x16383 <-> 16384 in f32 and in 8-byte elements) and the Table-I
shape 12000x11999 -> 12000, C3 select and unique on 256M over f = 0..1, C4
compact 1G float32 at 10/50/90 %, partition, out-of-place select, int64
compaction, 1- and 2-byte pad/unpad.  Every time is the median of the reps,
with min and p90 beside it; fractions are given of the measured copy peak
(MEASURED_PEAKS.json) and of the nominal 8 TB/s.

--impl reference: the CPU oracle (oracle/, sequential C, one core) on a
bounded sample of the same workload, rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "effective GB/s (read+write) and % of HBM peak for in-place compact/pad, 1/2/4/8 B200"
N_TOTAL = 1 << 32
# Test mode only (tests/test_bench.py): several ranks on ONE GPU over gloo with
# host-staged collectives and a smaller array, to exercise the N > 1 logic of
# this script on a one-GPU box.  Never used for a reported number.
TEST_GLOO = os.environ.get("DS_BENCH_TEST_GLOO") == "1"
if TEST_GLOO:
    N_TOTAL = 1 << int(os.environ.get("DS_BENCH_N_LOG2", "26"))
FRAC = 0.5
SEED = 0xD5201500 + 16 * 4  # dsgen.seed_for(4): C5
SETTLE_S = 3.0  # idle before the timed region (see run_libds)
STEP_GAP_S = float(os.environ.get("DS_BENCH_STEP_GAP_S", "0.02"))  # idle between timed steps (host side)
WORKLOAD = "C5: sharded in-place stream compaction of 4G int32 (2^32 words), 50% kept, remove_value 0"


NOMINAL_HBM_GBS = 8000.0  # B200 HBM3e nominal (B200_PROFILING.md); the measured copy rate is the ceiling


def summarize(ts_ms):
    """median / min / p90 of a list of times (ms) -> microseconds."""
    xs = sorted(ts_ms)
    p90 = xs[min(len(xs) - 1, int(round(0.9 * (len(xs) - 1))))]
    return {"us": round(statistics.median(xs) * 1e3, 2), "min_us": round(xs[0] * 1e3, 2),
            "p90_us": round(p90 * 1e3, 2), "reps": len(xs)}


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as fh:
            pk = json.load(fh)
        return float(pk["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, torch copy_)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_ncu_traffic():
    """DRAM bytes per launch of the headline kernel from the committed ncu capture."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(path) as fh:
            d = json.load(fh)
        return d.get("headline", {}).get("dram_bytes_per_launch")
    except Exception:
        return None


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.proc = None
        self.gpu = gpu_index

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.12)
        self.proc.terminate()
        out, _ = self.proc.communicate(timeout=10)
        sm, smax, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                smax = float(parts[1])
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": smax,
                "reasons": sorted(reasons), "samples": len(sm)}


def timed(fn, stream, restore=None, flush=None, reps=5, warmup=2):
    """Device times (ms, one per rep) of fn() on `stream`, events around fn only."""
    import torch
    ts = []
    for r in range(warmup + reps):
        if restore:
            restore()
        if flush:
            flush()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        fn()
        b.record(stream)
        b.synchronize()
        if r >= warmup:
            ts.append(a.elapsed_time(b))
    return ts


def bench_rows(peak, flush):
    """The other BASELINE configs (rank 0, N == 1)."""
    import numpy as np
    import torch

    import dsgen
    import oracle
    from paper_conf_icpp_gomez_lunacshg15_b200 import libds
    s = torch.cuda.current_stream()
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    rows = []

    def row(op, cfg, ts, nbytes, extra=None, dram_bytes=None):
        st = summarize(ts)
        gbs = nbytes / (st["us"] * 1e-6) / 1e9
        r = {"op": op, "config": cfg, **st, "gbs": round(gbs, 1), "frac": round(gbs / peak, 4),
             "frac_nominal": round(gbs / NOMINAL_HBM_GBS, 4)}
        if dram_bytes is not None and dram_bytes != nbytes:
            # identity moves store nothing: the DRAM bytes the kernel must move
            r["dram_bytes"] = dram_bytes
            r["frac_dram"] = round(dram_bytes / (st["us"] * 1e-6) / 1e9 / peak, 4)
        if extra:
            r.update(extra)
        rows.append(r)
        return r

    def irregular(op, name, src, call, reps=5):
        work = torch.empty_like(src)
        ts = timed(lambda: call(work), s, restore=lambda: work.copy_(src), flush=flush, reps=reps)
        m = int(d_n.item())
        n = src.numel()
        # an in-place call that removes nothing is an identity move: every tile
        # is skipped by the storers, only the reads reach DRAM
        row(op, name, ts, 4 * (n + m), {"n": n, "out_n": m}, dram_bytes=4 * n if m == n else None)

    def batched(call, base, copies=10, reps=5):
        """Small configs: the events' ~2 us granularity on this box blurs one
        call of 15-30 us, so also time `copies` back-to-back calls, each on its
        own restored copy (all restored + L2 flushed before the events), and
        report the per-call average (launch latency overlapped by the queue)."""
        bufs = [torch.empty_like(base) for _ in range(copies)]

        def restore():
            for b in bufs:
                b.copy_(base)

        ts = timed(lambda: [call(b) for b in bufs], s, restore=restore, flush=flush, reps=reps)
        del bufs
        return summarize([t / copies for t in ts])

    def graph_time(call, base, reps=20):
        """One call captured in a CUDA graph on a side stream (workspace made by a
        warm-up call there first), replayed on a restored, L2-flushed input:
        the device time without the host's launch path."""
        gs = torch.cuda.Stream()
        work = torch.empty_like(base)
        gs.wait_stream(s)
        with torch.cuda.stream(gs):
            work.copy_(base)
            call(work)
        s.wait_stream(gs)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=gs):
            call(work)
        ts = timed(lambda: g.replay(), s, restore=lambda: work.copy_(base), flush=flush, reps=reps)
        del g, work
        return summarize(ts)

    def regular(op, name, src, call, nbytes, reps=5, restore_src=None, batch=False):
        work = torch.empty_like(src)
        base = restore_src if restore_src is not None else src
        ts = timed(lambda: call(work), s, restore=lambda: work.copy_(base), flush=flush, reps=reps)
        extra = None
        if batch:
            b = batched(call, base)
            gr = graph_time(call, base)
            extra = {"back_to_back": {**b, "gbs": round(nbytes / (b["us"] * 1e-6) / 1e9, 1),
                                      "frac": round(nbytes / (b["us"] * 1e-6) / 1e9 / peak, 4)},
                     "graph_replay": {**gr, "gbs": round(nbytes / (gr["us"] * 1e-6) / 1e9, 1),
                                      "frac": round(nbytes / (gr["us"] * 1e-6) / 1e9 / peak, 4)}}
        row(op, name, ts, nbytes, extra)

    # C1: 1M int32 compaction, 50 %: kernel time flushed and L2-hot, the blocking
    # call's wall time (launch + sync + D2H of out_n), and the oracle in seconds
    n = 1 << 20
    src = dsgen.compact_input(n, 0.5, dsgen.seed_for(0), device="cuda")
    work = torch.empty_like(src)
    ts = timed(lambda: libds.ds_compact_ex(work, n, 0, d_n, None), s, restore=lambda: work.copy_(src),
               flush=flush, reps=50)
    m = int(d_n.item())
    ts_hot = timed(lambda: libds.ds_compact_ex(work, n, 0, d_n, None), s, restore=lambda: work.copy_(src),
                   reps=50)
    wall = []
    for r in range(53):
        work.copy_(src)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        libds.ds_compact(work, n, 0)
        if r >= 3:
            wall.append((time.perf_counter() - t0) * 1e3)
    host = src.cpu().numpy().view(np.uint32).copy()
    ot = []
    for _ in range(5):
        hcopy = host.copy()
        t0 = time.perf_counter()
        oracle.compact(hcopy, 0)
        ot.append(time.perf_counter() - t0)
    b2b = batched(lambda w: libds.ds_compact_ex(w, n, 0, d_n, None), src, copies=20)
    gr = graph_time(lambda w: libds.ds_compact_ex(w, n, 0, d_n, torch.cuda.current_stream()), src)
    row("compact", "C1 1M int32 f=0.5", ts, 4 * (n + m),
        {"n": n, "out_n": m, "l2_hot": summarize(ts_hot), "blocking_wall": summarize(wall),
         "back_to_back": {**b2b, "gbs": round(4 * (n + m) / (b2b["us"] * 1e-6) / 1e9, 1)},
         "graph_replay": {**gr, "gbs": round(4 * (n + m) / (gr["us"] * 1e-6) / 1e9, 1)},
         "oracle_s": round(statistics.median(ot), 6),
         "note": "flushed: 512 MiB read between reps; l2_hot: input restored by a D2D copy only "
                 "(it stays in L2); blocking_wall: ds_compact (legacy stream) incl. the D2H of out_n; "
                 "back_to_back: 20 calls on 20 restored copies between the events, per call; graph_replay: "
                 "the call captured in a CUDA graph, one replay between the events"})
    del src, work
    # C2: pad 4000x3990 -> 4000 f32 and unpad back
    R, C, NC = 4000, 3990, 4000
    src = dsgen.matrix_input(R, C, NC, 4, kind="f32", device="cuda")
    regular("pad", "C2 4000x3990->4000 f32", src, lambda w: libds.ds_pad_ex(w, R, C, NC, 4, None, None),
            4 * (R * C + R * NC), reps=20, batch=True)
    padded = src.clone()
    libds.ds_pad(padded, R, C, NC, 4)
    regular("unpad", "C2 4000x4000->3990 f32", src, lambda w: libds.ds_unpad_ex(w, R, NC, C, 4, None),
            4 * (2 * R * C), reps=20, restore_src=padded, batch=True)
    del src, padded
    # Pad / unpad where the >= 70 % target applies (>= 256M elements): 16384 x
    # 16383 <-> 16384 in f32 and in 8-byte elements, and the
    # Table-I shape 12000 x 11999 -> 12000
    for (R, C, NC, eb, tag) in ((16384, 16383, 16384, 4, "f32"), (16384, 16383, 16384, 8, "8-byte"),
                                (12000, 11999, 12000, 4, "f32 Table I")):
        src = dsgen.matrix_input(R, C, NC, eb, device="cuda")
        regular("pad", f"{R}x{C}->{NC} {tag}", src, lambda w: libds.ds_pad_ex(w, R, C, NC, eb, None, None),
                eb * (R * C + R * NC), reps=5)
        padded = src.clone()
        libds.ds_pad(padded, R, C, NC, eb)
        regular("unpad", f"{R}x{NC}->{C} {tag}", src, lambda w: libds.ds_unpad_ex(w, R, NC, C, eb, None),
                eb * 2 * R * C, reps=5, restore_src=padded)
        del src, padded
        torch.cuda.empty_cache()
    # C3: select (x > t) and unique, 256M int32, f = 0 .. 1
    n = 1 << 28
    src = dsgen.select_input(n, dsgen.seed_for(2), device="cuda")
    for i in range(11):
        f = i / 10
        t = dsgen.select_threshold(f) & 0xFFFFFFFF
        irregular("select", f"C3 256M int32 x>t f={f:.1f}", src,
                  lambda w, t=t: libds.ds_select_ex(w, n, libds.DS_PRED_I32_GT, t, d_n, None), reps=5)
    del src
    for i in range(11):
        f = i / 10
        src = dsgen.unique_runs_input(n, f, dsgen.seed_for(2, 11 + i), device="cuda")
        irregular("unique", f"C3 256M int32 runs f={f:.1f}", src,
                  lambda w: libds.ds_unique_ex(w, n, None, 0, d_n, None), reps=5)
        del src
    # Partition (in place through an aux buffer) and out-of-place
    # select (Copy_if) on 256M int32 at 50 %
    n = 1 << 28
    src = dsgen.select_input(n, dsgen.seed_for(5), device="cuda")
    t = dsgen.select_threshold(0.5) & 0xFFFFFFFF
    aux = torch.empty_like(src)
    work = torch.empty_like(src)
    ts = timed(lambda: libds.ds_partition_ex(work, n, libds.DS_PRED_I32_GT, t, aux, d_n, None), s,
               restore=lambda: work.copy_(src), flush=flush, reps=5)
    m = int(d_n.item())
    row("partition", "256M int32 x>t f=0.5 (in place, aux)", ts, 4 * (2 * n + 2 * (n - m)),
        {"n": n, "out_n": m, "bytes": "read n + write n_true in place + write/read/write n_false via aux"})
    ts = timed(lambda: libds.ds_select_copy_ex(src, n, libds.DS_PRED_I32_GT, t, work, d_n, None), s,
               flush=flush, reps=5)
    m = int(d_n.item())
    row("select_copy", "256M int32 x>t f=0.5 (out of place)", ts, 4 * (n + m), {"n": n, "out_n": m})
    del src, aux, work
    # C4: 1G float32 compaction at 10 / 50 / 90 %
    n = 1 << 30
    for f in (0.1, 0.5, 0.9):
        src = dsgen.compact_input(n, f, dsgen.seed_for(3, int(f * 10)), kind="f32", device="cuda")
        irregular("compact", f"C4 1G f32 f={f}", src,
                  lambda w: libds.ds_compact_ex(w, n, 0, d_n, None), reps=5)
        del src
    # 8(f)-3: 8-byte elements (int64 compaction, 256M elements = 2 GiB, 50 % kept)
    n = 1 << 28
    h = dsgen.hash_range(dsgen.seed_for(6), 0, n, device="cuda")
    src = torch.where(dsgen._hi32(h) < dsgen.keep_threshold(0.5), h | 1, torch.zeros_like(h))
    del h
    work = torch.empty_like(src)
    ts = timed(lambda: libds.ds_compact64_ex(work, n, 0, d_n, None), s, restore=lambda: work.copy_(src),
               flush=flush, reps=5)
    m = int(d_n.item())
    row("compact64", "256M int64 f=0.5 (8-byte elements)", ts, 8 * (n + m), {"n": n, "out_n": m})
    del src, work
    # 8(f)-4: sub-word elements, C2 shape (byte-granular kernel for 1-byte rows of
    # 3990 bytes; 2-byte rows are whole words and take the word kernel), and a
    # >= 256M-element byte shape (16384 x 16383 -> 16384, 1-byte elements)
    for (R, C, NC) in ((4000, 3990, 4000), (16384, 16383, 16384)):
        for eb in ((1, 2) if R == 4000 else (1,)):
            src = torch.randint(0, 256, (R * NC * eb,), dtype=torch.uint8, device="cuda")
            reps = 20 if R == 4000 else 5
            regular("pad", f"{R}x{C}->{NC} eb={eb}", src,
                    lambda w: libds.ds_pad_ex(w, R, C, NC, eb, None, None), eb * (R * C + R * NC), reps=reps,
                    batch=R == 4000)
            regular("unpad", f"{R}x{NC}->{C} eb={eb}", src,
                    lambda w: libds.ds_unpad_ex(w, R, NC, C, eb, None), eb * 2 * R * C, reps=reps,
                    batch=R == 4000)
            del src
    return rows


def oracle_sample_input(n_sample):
    import numpy as np

    import dsgen
    return dsgen.compact_input(n_sample, FRAC, SEED).numpy().view(np.uint32)


def cpu_oracle_sample(n_sample, reps, src=None):
    """The oracle (sequential C, 1 core) on a prefix-shaped sample of C5."""
    import oracle
    if src is None:
        src = oracle_sample_input(n_sample)
    ts, m = [], 0
    for _ in range(reps):
        a = src.copy()
        t0 = time.perf_counter()
        m = oracle.compact(a, 0)
        ts.append(time.perf_counter() - t0)
    t = statistics.median(ts)
    gbs = 4 * (n_sample + m) / t / 1e9
    return gbs, t, m


def bench_config(world, count_exchange):
    """The workload both arms report (identical dicts: the driver compares them)."""
    from paper_conf_icpp_gomez_lunacshg15_b200.dist import shard_range
    lo, hi = shard_range(N_TOTAL, world, 0)
    return {"workload": WORKLOAD if not TEST_GLOO else "TEST MODE (gloo, one GPU): " + WORKLOAD,
            "n_total": N_TOTAL, "n_per_rank": hi - lo, "valid_fraction": FRAC, "seed": SEED,
            "parallelism": f"shard{world} (contiguous ranges)",
            "l2": "inputs 16/N GiB per rank >> 126 MB L2; L2 also flushed by reading 512 MiB between steps",
            "restore": "pristine shard restored by a D2D copy between steps, outside the events "
                       "(the prefix [0, out_n) the compaction rewrites; the tail is checked untouched once)",
            "step": ("ds_compact_pub_ex (count stored into every rank's count board over peer memory) + "
                     "ds_shard_offsets_board" if count_exchange == "board" else
                     "ds_compact_ex + NCCL all-gather of counts + ds_shard_offsets"),
            "count_exchange": count_exchange,
            "settle": f"{SETTLE_S:g} s idle between the warm-up and the timed steps, "
                      f"{STEP_GAP_S * 1e3:g} ms between timed steps (host sleep after a synchronize, "
                      "outside the events)"}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    n_sample = 1 << 26
    src = oracle_sample_input(n_sample)
    steps = []
    for i in range(args.warmup + args.steps):
        gbs, t, m = cpu_oracle_sample(n_sample, 1, src)
        if i >= args.warmup:
            steps.append((gbs, t))
    value = statistics.median(g for g, _ in steps)
    ms = statistics.median(t for _, t in steps) * 1e3
    sample = (f"one step = oracle_compact on a 2^26-word (256 MiB) sample of the C5 recipe "
              f"(seed {SEED:#x}, f={FRAC}); 1 thread")
    line = {"metric": METRIC, "value": round(value, 3), "unit": "GB/s", "impl": "reference",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(ms, 3), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic (counter-based hash, dsgen)",
            "config": bench_config(int(os.environ.get("WORLD_SIZE", str(args.gpus))), args.count_exchange),
            "cpu_baseline": {"value": round(value, 3), "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": round(value, 3), "unit": "GB/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


class HostStagedComm:
    """TEST_GLOO only: the ShardedDS collectives staged through host memory."""

    def all_gather(self, out, inp):
        import torch
        import torch.distributed as dist
        parts = [torch.empty_like(inp.cpu()) for _ in range(dist.get_world_size())]
        dist.all_gather(parts, inp.cpu())
        out.copy_(torch.cat(parts).to(out.device))

    def exchange(self, sends, recvs):
        import torch
        import torch.distributed as dist
        reqs, back = [], []
        for t, peer in sends:
            h = t.cpu()
            back.append(None)
            reqs.append(dist.isend(h, peer))
            back[-1] = h
        for t, peer in recvs:
            h = torch.empty(t.shape, dtype=t.dtype)
            reqs.append(dist.irecv(h, peer))
            back.append((t, h))
        for r in reqs:
            r.wait()
        for item in back:
            if isinstance(item, tuple):
                item[0].copy_(item[1].to(item[0].device))


def all_gather_dev(out, inp):
    """Device all-gather (NCCL); host-staged over gloo in TEST_GLOO mode."""
    import torch
    import torch.distributed as dist
    if TEST_GLOO:
        HostStagedComm().all_gather(out, inp)
    else:
        dist.all_gather_into_tensor(out, inp)


def all_reduce_max_dev(t):
    import torch
    import torch.distributed as dist
    if TEST_GLOO:
        h = t.cpu()
        dist.all_reduce(h, op=dist.ReduceOp.MAX)
        t.copy_(h.to(t.device))
    else:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)


def run_libds(args):
    import torch
    import torch.distributed as dist

    import dsgen
    from paper_conf_icpp_gomez_lunacshg15_b200 import libds
    from paper_conf_icpp_gomez_lunacshg15_b200.dist import ShardedDS, shard_range

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if TEST_GLOO:
        local = 0  # every rank on the one GPU
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1 and TEST_GLOO:
        dist.init_process_group("gloo")
    elif world > 1:
        # the driver reads NCCL's communicator-init lines (nRanks) from stderr
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        dist.init_process_group("nccl", device_id=dev)
    peak, peak_src = load_peaks()

    # ---- the rank's shard of the C5 array (generated in place, seeded by global index)
    lo, hi = shard_range(N_TOTAL, world, rank)
    n = hi - lo
    pristine = torch.empty(n, dtype=torch.int32, device=dev)
    for s0 in range(0, n, 1 << 27):
        c = min(1 << 27, n - s0)
        h = dsgen.hash_range(SEED, lo + s0, c, device=dev)
        keep = dsgen._hi32(h) < dsgen.keep_threshold(FRAC)
        val = dsgen._as_i32(dsgen._lo32(h) | 1)
        pristine[s0:s0 + c] = torch.where(keep, val, torch.zeros_like(val))
        del h, keep, val
    work = torch.empty_like(pristine)
    flush_buf = torch.empty(1 << 27, dtype=torch.int32, device=dev)  # 512 MiB > 126 MB L2
    flush = lambda: flush_buf.sum()  # noqa: E731  (read-only flush: leaves no dirty lines)
    stream = torch.cuda.current_stream()
    ds = ShardedDS(device=dev, count_exchange=args.count_exchange, comm=HostStagedComm() if TEST_GLOO else None)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def step_once(kernel_ev):
        a, b, c = kernel_ev
        a.record(stream)
        if args.count_exchange == "board":
            # the DS kernel also stores its count into every rank's count board
            ds.local.compact_pub(work, 0, ds.d_count, ds._pub(), stream)
            b.record(stream)
            ds._finish_board(stream)
        else:
            libds.ds_compact_ex(work, n, 0, ds.d_count, stream)
            b.record(stream)
            ds._finish(stream)
        c.record(stream)

    # The compaction writes only words [0, out_n) (R5: the tail keeps its
    # bytes), so once out_n is known the restore copies that prefix alone; the
    # first warm-up step restores everything and checks the tail is untouched.
    restore_n = [n]

    def one_step(timed_events):
        work[:restore_n[0]].copy_(pristine[:restore_n[0]])
        flush()
        step_once(timed_events)

    # ---- warm-up
    for i in range(args.warmup):
        one_step([torch.cuda.Event(enable_timing=True) for _ in range(3)])
        if i == 0:
            m = int(ds.d_count.item())
            if not torch.equal(work[m:], pristine[m:]):
                raise SystemExit("bench: compaction changed words past out_n")
            restore_n[0] = m
    barrier()
    # Settle: the input generation and the warm-up just ran seconds of
    # full-bandwidth work; a short idle lets the board's power average fall
    # back, so the timed steps are not clocked down by sw_power_cap because of
    # the harness's own set-up (the clocks are still sampled and reported).
    torch.cuda.synchronize()
    time.sleep(SETTLE_S)
    barrier()

    # ---- timed region: exactly K steps, barrier + sync on both sides
    clocks = ClockSampler(local)
    clocks.start()
    launches0 = libds.ds_launch_count()
    evs = []
    barrier()
    for _ in range(args.steps):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        one_step(e)
        evs.append(e)
        if STEP_GAP_S:
            # idle between steps, outside the events: the restore copy of ~8 GiB
            # per step is harness work that would otherwise keep the board at its
            # power cap (sw_power_cap) during the timed steps
            torch.cuda.synchronize()
            time.sleep(STEP_GAP_S)
    barrier()
    launches = libds.ds_launch_count() - launches0
    clk = clocks.stop()
    step_list = [e[0].elapsed_time(e[2]) for e in evs]
    kern_list = [e[0].elapsed_time(e[1]) for e in evs]
    coll_list = [e[1].elapsed_time(e[2]) for e in evs]
    step_ms = sum(step_list)
    kern_ms = sum(kern_list) / args.steps
    coll_ms = sum(coll_list) / args.steps
    out_n = int(ds.d_count.item())
    total_out = int(ds.d_result[1].item())
    my_bytes = 4 * (n + out_n)
    # per-rank [step total, bytes, kernel ms/step, collective ms/step]; max / sum over ranks
    t = torch.tensor([step_ms, float(my_bytes), kern_ms, coll_ms], dtype=torch.float64, device=dev)
    if world > 1:
        allt = torch.zeros(world * 4, dtype=torch.float64, device=dev)
        all_gather_dev(allt, t)
        per_rank = allt.view(world, 4).tolist()
    else:
        per_rank = [t.tolist()]
    step_ms_max = max(r[0] for r in per_rank)
    all_bytes = sum(r[1] for r in per_rank)
    ms_per_step = step_ms_max / args.steps
    value = all_bytes / (ms_per_step * 1e-3) / 1e9

    # ---- optional rebalance leg (8(f)-1), timed separately after a compact step
    rebal = None
    if args.rebalance:
        rts = []
        for i in range(1 + max(1, args.steps // 4)):
            work.copy_(pristine)
            barrier()
            res = ds.compact(work, 0, stream=stream)
            barrier()
            t0 = torch.cuda.Event(enable_timing=True)
            t1 = torch.cuda.Event(enable_timing=True)
            t0.record(stream)
            held = ds.rebalance(work, res, stream=stream)
            t1.record(stream)
            barrier()
            if i > 0:
                rts.append(t0.elapsed_time(t1))
        mine = torch.tensor([statistics.median(rts)], dtype=torch.float64, device=dev)
        if world > 1:
            all_reduce_max_dev(mine)
        rebal = {"ms": round(float(mine.item()), 4), "held_rank0": held,
                 "note": "ShardedDS.rebalance after the compact step: wave-scheduled NCCL send/recv of "
                         "the pieces + ds_slide; host-synchronising plan; max over ranks"}

    # ---- e2e through the public API with host buffers (pinned), copies inside the timing.
    # The shard goes through in E2E_CHUNKS pieces on three streams so that the
    # H2D copy of piece j+1, the in-place compaction of piece j (ds_compact_ex)
    # and the D2H copy of piece j-1's kept prefix overlap; the host output is the
    # concatenation of the pieces' kept prefixes, which is the compaction of the
    # whole shard (the decomposition property).
    e2e = None
    if not args.no_e2e:
        host_in = torch.empty(n, dtype=torch.int32, pin_memory=True)
        host_in.copy_(pristine)
        host_out = torch.empty(n, dtype=torch.int32, pin_memory=True)
        K = max(1, min(args.e2e_chunks, n >> 20))
        bounds = [n * j // K for j in range(K + 1)]
        s_in, s_cmp, s_out = (torch.cuda.Stream(device=dev) for _ in range(3))
        d_cnt = torch.zeros(K, dtype=torch.int64, device=dev)
        h_cnt = torch.zeros(K, dtype=torch.int64, pin_memory=True)
        e2e_t, e2e_out = [], 0
        for i in range(1 + args.e2e_steps):
            barrier()
            t0 = time.perf_counter()
            ev_in = [torch.cuda.Event() for _ in range(K)]
            ev_cmp = [torch.cuda.Event() for _ in range(K)]
            off = 0

            def drain(j):
                nonlocal off
                ev_cmp[j].synchronize()
                c = int(h_cnt[j])
                with torch.cuda.stream(s_out):
                    s_out.wait_event(ev_cmp[j])
                    host_out[off:off + c].copy_(work[bounds[j]:bounds[j] + c], non_blocking=True)
                off += c

            for j in range(K):
                lo_j, hi_j = bounds[j], bounds[j + 1]
                with torch.cuda.stream(s_in):
                    work[lo_j:hi_j].copy_(host_in[lo_j:hi_j], non_blocking=True)  # H2D
                    ev_in[j].record(s_in)
                s_cmp.wait_event(ev_in[j])
                libds.ds_compact_ex(work[lo_j:hi_j], hi_j - lo_j, 0, d_cnt[j:j + 1], s_cmp)
                with torch.cuda.stream(s_cmp):
                    h_cnt[j:j + 1].copy_(d_cnt[j:j + 1], non_blocking=True)  # D2H of the count
                    ev_cmp[j].record(s_cmp)
                if j > 0:
                    drain(j - 1)
            drain(K - 1)
            total_local = torch.tensor([off], dtype=torch.int64, device=dev)
            if world > 1:  # the count exchange of the sharded step (global offsets)
                allc = torch.empty(world, dtype=torch.int64, device=dev)
                all_gather_dev(allc, total_local)
            torch.cuda.synchronize()
            dt = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
            if world > 1:
                all_reduce_max_dev(dt)
            if i > 0:
                e2e_t.append(float(dt.item()))
            e2e_out = off
        if e2e_out != out_n:
            raise RuntimeError(f"e2e: chunked output length {e2e_out} != {out_n}")
        ms_e2e = statistics.median(e2e_t) * 1e3
        e2e = {"value": round(all_bytes / (ms_e2e * 1e-3) / 1e9, 2), "unit": "GB/s",
               "h2d_bytes_per_step": 4 * n, "d2h_bytes_per_step": 4 * out_n + 8 * K,
               "ms_per_step": round(ms_e2e, 2), "steps": args.e2e_steps, "chunks": K,
               "note": "per rank; pinned host buffers; the shard in K pieces on three streams: H2D of a "
                       "piece, ds_compact_ex on it in place, D2H of its count and kept prefix, "
                       "overlapped across pieces (+ NCCL count all-gather when N > 1)"}
        del host_in, host_out

    rows = None
    if rank == 0 and world == 1 and not args.no_rows:
        del work, pristine
        torch.cuda.empty_cache()
        rows = bench_rows(peak, flush)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        n_sample = 1 << 26
        gbs, t_s, _ = cpu_oracle_sample(n_sample, 3)
        cpu = {"value": round(gbs, 3), "unit": "GB/s", "cores": 1, "kind": "oracle",
               "sample": f"oracle_compact (sequential C, 1 thread of {os.cpu_count()}) on a "
                         f"2^26-word sample of the C5 recipe, median of 3 ({t_s * 1e3:.0f} ms each)"}

    if rank == 0:
        kbytes = 4 * (n + out_n)
        achieved = kbytes / (kern_ms * 1e-3) / 1e9
        traffic = load_ncu_traffic()
        step_stats = summarize(step_list)
        line = {
            "metric": METRIC, "value": round(value, 1), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "int32", "data": "synthetic (counter-based hash, dsgen; seeded per global index)",
            "impl": "libds",
            "config": bench_config(world, args.count_exchange),
            "out_n": total_out,
            "frac_of_peak": round(value / world / peak, 4),
            "frac_of_nominal": round(value / world / NOMINAL_HBM_GBS, 4),
            "elems_per_s": round(N_TOTAL / (ms_per_step * 1e-3), 1),
            "step_stats_rank0": step_stats,
            "per_rank": [{"rank": r, "step_ms": round(x[0] / args.steps, 4), "kernel_ms": round(x[2], 4),
                          "collective_ms": round(x[3], 4)} for r, x in enumerate(per_rank)],
            "kernel_ms_max": round(max(x[2] for x in per_rank), 4),
            "collective_ms_max": round(max(x[3] for x in per_rank), 4),
            "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4), "traffic": traffic,
                         "frac_nominal": round(achieved / NOMINAL_HBM_GBS, 4),
                         "kernel_stats": summarize(kern_list),
                         "kernel": "irregular_kernel<OpCompact> (rank 0)", "peak_source": peak_src,
                         "kernel_ms": round(kern_ms, 4),
                         "algorithmic_bytes_per_launch": kbytes},
            "clocks": clk, "gpu_launches": launches,
        }
        if e2e:
            line["e2e"] = e2e
        if rebal:
            line["rebalance"] = rebal
        if cpu:
            line["cpu_baseline"] = cpu
        if rows:
            line["rows"] = rows
        print(json.dumps(line), flush=True)
    ds.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="libds", choices=["libds", "reference"])
    ap.add_argument("--no-rows", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--e2e-chunks", type=int, default=256)
    ap.add_argument("--rebalance", action="store_true", help="also time ShardedDS.rebalance (8(f)-1)")
    ap.add_argument("--count-exchange", default="collective", choices=["collective", "board"],
                    help="counts by NCCL all-gather (default) or through the count boards (peer memory)")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "libds" and not os.environ.get("DS_BENCH_ALLOW_SHORT"):
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_libds(args)


if __name__ == "__main__":
    main()
