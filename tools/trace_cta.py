"""Kernel-level trace of one irregular launch (ds_debug_set_trace with room for
the per-CTA events): when the CTAs start, when their roles finish, against the
tile work (first draw .. last region released).  For small arrays (C1) this
shows where the time outside the tile pipeline goes.

    python tools/trace_cta.py [n_log2] [f]
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dsgen  # noqa: E402
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402


def pct(name, d):
    q = np.percentile(d, [0, 50, 100])
    print(f"{name:26s} min {q[0]:6.2f} p50 {q[1]:6.2f} max {q[2]:6.2f} us")


def main():
    lg = int(sys.argv[1]) if len(sys.argv) > 1 else 20
    f = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
    n = 1 << lg
    T = libds.ds_tile_size(libds.DS_KERNEL_IRREGULAR)
    src = dsgen.compact_input(n, f, 7, device="cuda")
    work = torch.empty_like(src)
    ntiles = (n + T - 1) // T
    cap = ntiles + 1024
    tr = torch.zeros(cap * 16, dtype=torch.int64, device="cuda")
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.int32, device="cuda")
    for rep in range(4):
        work.copy_(src)
        flush.sum()
        torch.cuda.synchronize()
        tr.zero_()
        libds.ds_debug_set_trace(tr if rep == 3 else None, cap if rep == 3 else 0)
        libds.ds_compact_ex(work, n, 0, d_n, None)
        torch.cuda.synchronize()
    libds.ds_debug_set_trace(None, 0)
    t = tr.cpu().numpy().reshape(cap, 16).astype(np.int64)
    tiles, ctas = t[:ntiles], t[ntiles:]
    ctas = ctas[ctas[:, 0] > 0]
    t0 = ctas[:, 0].min()
    us = lambda a: (a - t0) / 1e3  # noqa: E731
    print(f"n=2^{lg} f={f} tiles={ntiles} CTAs={len(ctas)}")
    ends = ctas[:, 2:10]
    kernel_end = us(ends[ends > 0].max())
    print(f"first CTA entry -> last role done: {kernel_end:.2f} us; tile work: first draw {us(tiles[:, 0].min()):.2f}"
          f" .. last release {us(tiles[:, 12].max()):.2f} us")
    pct("CTA entry", us(ctas[:, 0]))
    pct("entry -> initialised", (ctas[:, 1] - ctas[:, 0]) / 1e3)
    pct("initialised -> 1st draw", np.array([us(tiles[:, 0][(tiles[:, 7] & 0xffff) == sm].min()) - us(c)
                                             for sm, c in zip(ctas[:, 15], ctas[:, 1])
                                             if ((tiles[:, 7] & 0xffff) == sm).any()]))
    for ev, name in ((2, "producer done"), (3, "storers 0 done"), (4, "storers 1 done"), (5, "rankers 0 done"),
                     (6, "rankers 1 done"), (7, "resolver 0 done"), (8, "resolver 1 done"), (9, "resolver 2 done")):
        v = ctas[:, ev]
        if (v > 0).any():
            pct(name, us(v[v > 0]))


if __name__ == "__main__":
    main()
