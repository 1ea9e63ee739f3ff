"""Storer-side trace of one irregular launch (ds_debug_set_trace): how long a
resolved tile waits for the CTA's storers, how long the re-phase + issue
takes, how long the bulk engine takes to read the region (issue -> released),
and the storers' busy share per CTA.

    [DS_OP=unique] python tools/trace_storer.py [n_log2] [f]
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dsgen  # noqa: E402
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402


def pct(name, d):
    q = np.percentile(d, [5, 50, 95])
    print(f"{name:22s} p5 {q[0]:6.2f} p50 {q[1]:6.2f} p95 {q[2]:6.2f} mean {d.mean():6.2f} us")


def main():
    lg = int(sys.argv[1]) if len(sys.argv) > 1 else 28
    f = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
    n = 1 << lg
    T = libds.ds_tile_size(libds.DS_KERNEL_IRREGULAR)
    op = os.environ.get("DS_OP", "compact")
    if op == "unique":
        src = dsgen.unique_runs_input(n, f, 5, device="cuda")
    elif op == "partcopy":  # the partition's DS pass, out of place
        src = dsgen.select_input(n, dsgen.seed_for(5), device="cuda")
        thr = dsgen.select_threshold(f) & 0xFFFFFFFF
        ot, of = torch.empty_like(src), torch.empty_like(src)
    else:
        src = dsgen.compact_input(n, f, 7, device="cuda")
    work = torch.empty_like(src)
    ntiles = (n + T - 1) // T
    tr = torch.zeros(ntiles * 16, dtype=torch.int64, device="cuda")
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    for rep in range(3):
        work.copy_(src)
        torch.cuda.synchronize()
        libds.ds_debug_set_trace(tr if rep == 2 else None, ntiles if rep == 2 else 0)
        if op == "unique":
            libds.ds_unique_ex(work, n, None, 0, d_n, None)
        elif op == "partcopy":
            libds.ds_partition_copy_ex(work, n, 1, thr, ot, of, d_n, None)
        else:
            libds.ds_compact_ex(work, n, 0, d_n, None)
        torch.cuda.synchronize()
    libds.ds_debug_set_trace(None, 0)
    t = tr.cpu().numpy().reshape(ntiles, 16).astype(np.int64)
    t0 = t[:, 0].min()
    us = lambda c: (t[:, c] - t0) / 1e3  # noqa: E731
    drawn, resolved, sstart, issued, released, ranked = us(0), us(4), us(5), us(6), us(12), us(15)
    span = released.max()
    print(f"{op} n=2^{lg} f={f} tiles={ntiles} span {span:.1f} us rate {ntiles / span:.1f} tiles/us; "
          f"in ring {((t[:, 7] >> 16) & 1).mean():.1%}")
    pct("ranked->resolved", resolved - ranked)
    pct("resolved->storer", sstart - resolved)
    pct("rephase+issue", issued - sstart)
    pct("issue->released", released - issued)
    if os.environ.get("DS_TRACE_STORER"):  # library built with -DDS_TRACE_STORER: sub-steps (slots 8-11)
        sub = [us(c) for c in (8, 9, 10, 11)]
        ok = (t[:, 8] > 0) & (t[:, 11] > 0)
        for name, a, b in (("  start->rephased", sstart, sub[0]), ("  rephased->fenced", sub[0], sub[1]),
                           ("  fenced->barrier", sub[1], sub[2]), ("  barrier->issued", sub[2], sub[3]),
                           ("  bulk issued->end", sub[3], issued)):
            pct(name, (b - a)[ok])
    pct("draw->released", released - drawn)
    sm = t[:, 7] & 0xffff
    busy, life = [], []
    for s_ in np.unique(sm):
        idx = np.where(sm == s_)[0]
        busy.append(np.sum(released[idx] - sstart[idx]))
        life.append(released[idx].max() - drawn[idx].min())
    busy, life = np.array(busy), np.array(life)
    print(f"storer busy share per CTA: p50 {np.median(busy / life):.1%} mean {np.mean(busy / life):.1%}")


if __name__ == "__main__":
    main()
