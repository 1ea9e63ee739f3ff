"""Per-tile pipeline trace of one pad / unpad launch (ds_debug_set_trace).
    python tools/trace_regular.py pad 12000 11999 12000
Events: 0 drawn, 1 landed, 2 LOADED published, 3 window wait start,
4 window wait end, 5 consumers passed the store barrier, 6 stores issued."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dsgen  # noqa: E402
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402

T = 8192


def main():
    op = sys.argv[1]
    R, C, NC = (int(x) for x in sys.argv[2:5])
    eb = int(sys.argv[5]) if len(sys.argv) > 5 else 4
    global T
    if eb in (1, 2) and (C * eb) % 4:  # byte-granular kernel: 32 KB output tiles
        T = (32768 if R * max(C, NC) * eb >= (64 << 20) else 16384) // eb
    if eb == 4:
        src = dsgen.matrix_input(R, C, NC, 4, device="cuda")
    else:
        src = torch.randint(0, 256, (R * max(C, NC) * eb,), dtype=torch.uint8, device="cuda")
    if op == "unpad":
        libds.ds_pad(src, R, NC, C, 4) if False else None
    work = torch.empty_like(src)
    out_words = R * NC
    ntiles = (out_words + T - 1) // T
    tr = torch.zeros(ntiles * 16, dtype=torch.int64, device="cuda")
    fn = (lambda: libds.ds_pad_ex(work, R, C, NC, eb, None, None)) if op == "pad" else \
         (lambda: libds.ds_unpad_ex(work, R, C, NC, eb, None))
    for rep in range(3):
        work.copy_(src)
        torch.cuda.synchronize()
        libds.ds_debug_set_trace(tr if rep == 2 else None, ntiles if rep == 2 else 0)
        fn()
        torch.cuda.synchronize()
    libds.ds_debug_set_trace(None, 0)
    t = tr.cpu().numpy().reshape(ntiles, 16).astype(np.int64)
    t0 = t[:, 0].min()
    ev = (t[:, :7] - t0) / 1e3
    span = ev[:, 6].max()
    nbytes = eb * (R * C + R * NC) if op == "pad" else 2 * eb * R * NC
    print(f"{op} {R}x{C}->{NC} tiles={ntiles} span={span:.1f} us  {nbytes / span / 1e3:.0f} GB/s")
    for k, name in enumerate(["load", "publish", "->consumers", "window", "gather", "store"]):
        d = ev[:, k + 1] - ev[:, k]
        q = np.percentile(d, [5, 50, 95, 99])
        print(f"{name:12s} p5 {q[0]:7.2f}  p50 {q[1]:7.2f}  p95 {q[2]:7.2f}  p99 {q[3]:7.2f}")
    life = ev[:, 6] - ev[:, 0]
    print(f"life p50 {np.median(life):.2f}  first draw->last store {span:.1f} us; "
          f"first tile done at {ev[:, 6].min():.2f} us")


if __name__ == "__main__":
    main()
