"""Input-stage / ring usage of one irregular launch (ds_debug_set_trace):
the share of tiles compacted into the output ring vs in place, the producer's
wait for a free input stage, and the stage hold time (draw -> ranked).

    [DS_OP=unique] python tools/trace_stage.py [n_log2] [f]
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dsgen  # noqa: E402
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402


def main():
    lg = int(sys.argv[1]) if len(sys.argv) > 1 else 28
    f = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
    n = 1 << lg
    T = libds.ds_tile_size(libds.DS_KERNEL_IRREGULAR)
    src = dsgen.compact_input(n, f, 7, device="cuda")
    work = torch.empty_like(src)
    ntiles = (n + T - 1) // T
    tr = torch.zeros(ntiles * 16, dtype=torch.int64, device="cuda")
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    for rep in range(3):
        work.copy_(src)
        torch.cuda.synchronize()
        libds.ds_debug_set_trace(tr if rep == 2 else None, ntiles if rep == 2 else 0)
        libds.ds_compact_ex(work, n, 0, d_n, None)
        torch.cuda.synchronize()
    libds.ds_debug_set_trace(None, 0)
    t = tr.cpu().numpy().reshape(ntiles, 16).astype(np.int64)
    in_ring = (t[:, 7] >> 16) & 1
    wait = (t[:, 0] - t[:, 13]) / 1e3
    hold = (t[:, 15] - t[:, 0]) / 1e3
    land = (t[:, 1] - t[:, 0]) / 1e3
    span = (t[:, 6].max() - t[:, 0].min()) / 1e3
    print(f"n=2^{lg} f={f} tiles={ntiles} rate={ntiles / span:.1f} tiles/us; in ring {in_ring.mean():.1%}"
          " ('stage wait' = claim -> drawn: the wait for a free stage + the ticket atomic)")
    # producer loop, per CTA in draw order: after a draw until the next claim
    # starts (load issue, slot wait) and claim -> draw (stage wait + ticket atomic)
    sm = t[:, 7] & 0xffff
    post = []
    for s_ in np.unique(sm):
        idx = np.where(sm == s_)[0]
        idx = idx[np.argsort(t[idx, 0])]
        post.append((t[idx[1:], 13] - t[idx[:-1], 0]) / 1e3)
    post = np.concatenate(post)
    if os.environ.get("DS_TRACE_PRODUCER"):  # library built with -DDS_TRACE_PRODUCER: slots 8-11
        for name, a, b in (("claim->taken", 13, 8), ("taken->drawn", 8, 0), ("drawn->pre-fence", 0, 9),
                           ("fence", 9, 10), ("bulk issue", 10, 11)):
            d = (t[:, b] - t[:, a]) / 1e3
            q = np.percentile(d, [5, 50, 95])
            print(f"  {name:16s} p5 {q[0]:6.2f} p50 {q[1]:6.2f} p95 {q[2]:6.2f} mean {d.mean():6.2f} us")
    for name, d in (("stage wait", wait), ("draw->landed", land), ("draw->ranked", hold),
                    ("draw->next claim", post)):
        q = np.percentile(d, [5, 50, 95])
        print(f"{name:16s} p5 {q[0]:6.2f} p50 {q[1]:6.2f} p95 {q[2]:6.2f} mean {d.mean():6.2f} us")


if __name__ == "__main__":
    main()
