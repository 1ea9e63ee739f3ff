"""Targeted device timing of a few libds calls (development aid, not the bench).

    LIBDS_PATH=... python tools/qt.py OP[:F] ...
OP in compact1g, select, unique, uniqueh, pad, unpad, c1; F the valid fraction.
Events on the launching stream; pristine input restored (D2D) and L2 flushed
between reps, both outside the events."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dsgen  # noqa: E402
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402

dev = torch.device("cuda")
flush = torch.empty(256 << 20, dtype=torch.int32, device=dev)
PEAK = 6547.8


PRIME = os.environ.get("QT_PRIME")  # run a 1-tile libds call after the flush (same smem carve-out)
prime_buf = torch.ones(64, dtype=torch.int32, device=dev)
prime_n = torch.zeros(1, dtype=torch.int64, device=dev)


def timeit(name, pristine, fn, bytes_fn, reps=10):
    work = pristine.clone()
    d_n = torch.zeros(1, dtype=torch.int64, device=dev)
    ts = []
    for r in range(reps + 3):
        work.copy_(pristine)
        flush.sum()
        if PRIME:
            libds.ds_compact_ex(prime_buf, 64, 0, prime_n, None)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn(work, d_n)
        e.record()
        torch.cuda.synchronize()
        if r >= 3:
            ts.append(s.elapsed_time(e) * 1e-3)
    ts.sort()
    t = ts[len(ts) // 2]
    b = bytes_fn(int(d_n.item()))
    tag = os.path.basename(os.environ.get("LIBDS_PATH", "libds.so"))
    print(f"{tag:28s} {name:28s} {t * 1e6:9.1f} us  {b / t / 1e9:8.1f} GB/s  "
          f"({b / t / PEAK / 1e9 * 100:5.1f}%)  min {ts[0] * 1e6:.1f} us", flush=True)


def run(spec):
    op, _, fs = spec.partition(":")
    f = float(fs) if fs else 0.5
    if op == "compact1g":
        n = 1 << 30
        a = dsgen.compact_input(n, f, dsgen.seed_for(3, int(f * 10)), kind="f32", device=dev)
        timeit(f"compact 1G f={f}", a, lambda w, d: libds.ds_compact_ex(w, n, 0, d, None), lambda m: 4 * (n + m))
    elif op == "c1":
        n = 1 << 20
        a = dsgen.compact_input(n, f, dsgen.seed_for(0), device=dev)
        timeit(f"compact 1M f={f}", a, lambda w, d: libds.ds_compact_ex(w, n, 0, d, None), lambda m: 4 * (n + m),
               reps=30)
    elif op == "c1b2b":  # 20 back-to-back calls between the events (launch-to-launch time)
        n = 1 << 20
        a = dsgen.compact_input(n, f, dsgen.seed_for(0), device=dev)

        def calls(w, d):
            for _ in range(20):
                libds.ds_compact_ex(w, n, 0, d, None)
        timeit(f"compact 1M f={f} x20", a, calls, lambda m: 20 * 4 * (n + m), reps=10)
    elif op == "select":
        n = 1 << 28
        a = dsgen.select_input(n, 3, device=dev)
        t = dsgen.select_threshold(f) & 0xFFFFFFFF
        timeit(f"select 256M f={f}", a, lambda w, d: libds.ds_select_ex(w, n, 1, t, d, None), lambda m: 4 * (n + m))
    elif op == "unique":
        n = 1 << 28
        a = dsgen.unique_runs_input(n, f, 5, device=dev)
        timeit(f"unique 256M f={f}", a, lambda w, d: libds.ds_unique_ex(w, n, None, 0, d, None),
               lambda m: 4 * (n + m))
    elif op in ("pad", "unpad"):
        R, C, NC = 4000, 3990, 4000
        a = dsgen.matrix_input(R, C, NC, 4, device=dev)
        if op == "pad":
            timeit("pad 4000x3990->4000", a, lambda w, d: libds.ds_pad_ex(w, R, C, NC, 4, None, None),
                   lambda m: 4 * (R * C + R * NC), reps=30)
        else:
            libds.ds_pad(a, R, C, NC, 4)
            timeit("unpad 4000x4000->3990", a, lambda w, d: libds.ds_unpad_ex(w, R, NC, C, 4, None),
                   lambda m: 4 * (2 * R * C), reps=30)
    elif op in ("padb1", "padb2", "unpadb1", "unpadb2"):  # sub-word elements, byte-granular kernel
        R, C, NC = 4000, 3990, 4000
        eb = int(op[-1])
        a = torch.randint(0, 256, (R * NC * eb,), dtype=torch.uint8, device=dev)
        if op.startswith("pad"):
            timeit(f"pad {R}x{C}->{NC} eb={eb}", a, lambda w, d: libds.ds_pad_ex(w, R, C, NC, eb, None, None),
                   lambda m: eb * (R * C + R * NC), reps=30)
        else:
            timeit(f"unpad {R}x{NC}->{C} eb={eb}", a, lambda w, d: libds.ds_unpad_ex(w, R, NC, C, eb, None),
                   lambda m: eb * (2 * R * C), reps=30)
    elif op in ("padbig1", "unpadbig1"):  # >= 256M 1-byte elements (byte-granular kernel)
        R, C, NC = 16384, 16383, 16384
        a = torch.randint(0, 256, (R * NC,), dtype=torch.uint8, device=dev)
        if op == "padbig1":
            timeit(f"pad {R}x{C}->{NC} eb=1", a, lambda w, d: libds.ds_pad_ex(w, R, C, NC, 1, None, None),
                   lambda m: R * C + R * NC)
        else:
            timeit(f"unpad {R}x{NC}->{C} eb=1", a, lambda w, d: libds.ds_unpad_ex(w, R, NC, C, 1, None),
                   lambda m: 2 * R * C)
    elif op == "part":  # in-place partition through aux
        n = 1 << 28
        a = dsgen.select_input(n, dsgen.seed_for(5), device=dev)
        t = dsgen.select_threshold(f) & 0xFFFFFFFF
        aux = torch.empty_like(a)
        timeit(f"partition 256M f={f}", a, lambda w, d: libds.ds_partition_ex(w, n, 1, t, aux, d, None),
               lambda m: 4 * (2 * n + 2 * (n - m)))
    elif op in ("padbig", "unpadbig", "padbig8"):  # >= 256M elements, word kernel
        R, C, NC = 16384, 16383, 16384
        eb = 8 if op == "padbig8" else 4
        a = dsgen.matrix_input(R, C, NC, eb, device=dev)
        if op.startswith("pad"):
            timeit(f"pad {R}x{C}->{NC} eb={eb}", a, lambda w, d: libds.ds_pad_ex(w, R, C, NC, eb, None, None),
                   lambda m: eb * (R * C + R * NC))
        else:
            libds.ds_pad(a, R, C, NC, eb)
            timeit(f"unpad {R}x{NC}->{C} eb={eb}", a, lambda w, d: libds.ds_unpad_ex(w, R, NC, C, eb, None),
                   lambda m: eb * (2 * R * C))
    elif op == "partcopy":  # the partition's DS pass alone, out of place (trues and falses)
        n = 1 << 28
        a = dsgen.select_input(n, dsgen.seed_for(5), device=dev)
        t = dsgen.select_threshold(f) & 0xFFFFFFFF
        ot, of = torch.empty_like(a), torch.empty_like(a)
        timeit(f"partition_copy 256M f={f}", a,
               lambda w, d: libds.ds_partition_copy_ex(w, n, 1, t, ot, of, d, None), lambda m: 4 * (2 * n))
    elif op == "pad12k":
        R, C, NC = 12000, 11999, 12000
        a = dsgen.matrix_input(R, C, NC, 4, device=dev)
        timeit("pad 12000x11999->12000", a, lambda w, d: libds.ds_pad_ex(w, R, C, NC, 4, None, None),
               lambda m: 4 * (R * C + R * NC))
    else:
        raise SystemExit(f"unknown op {op}")
    torch.cuda.empty_cache()


if __name__ == "__main__":
    for spec in sys.argv[1:]:
        run(spec)
