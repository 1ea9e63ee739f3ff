"""Quick device timing of each libds primitive (development aid, not the bench).

Times each call with CUDA events on the launching stream, restoring the
pristine input (D2D copy, untimed) and flushing L2 between reps."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dsgen  # noqa: E402
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402

dev = torch.device("cuda")
flush = torch.empty(256 << 20, dtype=torch.int32, device=dev)


def timeit(name, pristine, fn, bytes_fn, reps=15):
    work = pristine.clone()
    d_n = torch.zeros(1, dtype=torch.int64, device=dev)
    ts = []
    for r in range(reps + 3):
        work.copy_(pristine)
        flush.sum()
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
    print(f"{name:40s} {t * 1e6:9.1f} us  {b / t / 1e9:8.1f} GB/s  ({b / t / 6546.6e9 * 100:5.1f}% of 6546.6)  min {ts[0]*1e6:.1f} us", flush=True)


def main():
    n = 1 << 30
    for f in (0.1, 0.5, 0.9):
        a = dsgen.compact_input(n, f, dsgen.seed_for(3, int(f * 10)), kind="f32", device=dev)
        timeit(f"compact 1G f32 f={f}", a, lambda w, d: libds.ds_compact_ex(w, n, 0, d, None),
               lambda m: 4 * (n + m))
        del a
    n = 1 << 28
    for f in (0.0, 0.5, 1.0):
        a = dsgen.select_input(n, 3, device=dev)
        t = dsgen.select_threshold(f) & 0xFFFFFFFF
        timeit(f"select 256M f={f}", a, lambda w, d: libds.ds_select_ex(w, n, 1, t, d, None),
               lambda m: 4 * (n + m))
        a = dsgen.unique_runs_input(n, f, 5, device=dev)
        timeit(f"unique 256M f={f}", a, lambda w, d: libds.ds_unique_ex(w, n, None, 0, d, None),
               lambda m: 4 * (n + m))
    R, C, NC = 4000, 3990, 4000
    a = dsgen.matrix_input(R, C, NC, 4, device=dev)
    timeit("pad 4000x3990->4000", a, lambda w, d: libds.ds_pad_ex(w, R, C, NC, 4, None, None),
           lambda m: 4 * (R * C + R * NC))
    b = a.clone()
    libds.ds_pad(b, R, C, NC, 4)
    timeit("unpad 4000x4000->3990", b, lambda w, d: libds.ds_unpad_ex(w, R, NC, C, 4, None),
           lambda m: 4 * (2 * R * C))
    for eb in (1, 2):
        a = torch.randint(0, 256, (R * NC * eb,), dtype=torch.uint8, device=dev)
        timeit(f"pad {R}x{C}->{NC} eb={eb}", a, lambda w, d, eb=eb: libds.ds_pad_ex(w, R, C, NC, eb, None, None),
               lambda m, eb=eb: eb * (R * C + R * NC))
        timeit(f"unpad {R}x{NC}->{C} eb={eb}", a, lambda w, d, eb=eb: libds.ds_unpad_ex(w, R, NC, C, eb, None),
               lambda m, eb=eb: eb * (2 * R * C))
    R, C, NC = 12000, 11999, 12000
    a = dsgen.matrix_input(R, C, NC, 4, device=dev)
    timeit("pad 12000x11999->12000", a, lambda w, d: libds.ds_pad_ex(w, R, C, NC, 4, None, None),
           lambda m: 4 * (R * C + R * NC))
    n = 1 << 30
    a = torch.empty(n, dtype=torch.int32, device=dev)
    o = torch.empty_like(a)
    timeit("torch copy_ 1G int32 (reference)", a, lambda w, d: o.copy_(w), lambda m: 8 * n)


if __name__ == "__main__":
    main()
