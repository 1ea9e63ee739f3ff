"""Per-tile pipeline trace of one irregular DS launch (ds_debug_set_trace).

Prints, over all tiles, percentiles of the stage latencies (us):
  load     landed - drawn          (TMA bulk copy)
  count    agg - landed            (producer's aggregate)
  lbwait   lbstart - agg           (waiting for the CTA's resolver)
  lookback incl - lbstart          (decoupled look-back)
  cwait    cstart - incl           (waiting for the CTA's consumers)
  consume  cend - cstart           (rank, scatter, stores issued)
and the overall tile rate.
    [DS_OP=unique] python tools/trace_pipeline.py [n_log2] [f]
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dsgen  # noqa: E402
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402

T = int(os.environ.get("DS_TILE", "8192"))


def main():
    lg = int(sys.argv[1]) if len(sys.argv) > 1 else 28
    f = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
    n = 1 << lg
    op = os.environ.get("DS_OP", "compact")
    if op == "unique":
        src = dsgen.unique_runs_input(n, f, 5, device="cuda")
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
        else:
            libds.ds_compact_ex(work, n, 0, d_n, None)
        torch.cuda.synchronize()
    libds.ds_debug_set_trace(None, 0)
    t = tr.cpu().numpy().reshape(ntiles, 16).astype(np.int64)
    t0 = t[:, 0].min()
    ev = (t[:, :7] - t0) / 1e3
    names = ["load", "count", "lbwait", "lookback", "cwait", "consume"]
    print(f"n=2^{lg} f={f} tiles={ntiles} span={ev[:, 6].max():.1f} us "
          f"rate={ntiles / ev[:, 6].max():.1f} tiles/us")
    for k, name in enumerate(names):
        d = ev[:, k + 1] - ev[:, k]
        q = np.percentile(d, [5, 50, 95, 99])
        print(f"{name:9s} p5 {q[0]:7.2f}  p50 {q[1]:7.2f}  p95 {q[2]:7.2f}  p99 {q[3]:7.2f}  mean {d.mean():7.2f}")
    lb = (t[:, [10, 11, 12]] - t0) / 1e3
    for name, d in (("lb:first-read", lb[:, 0] - ev[:, 3]), ("lb:resolve", lb[:, 1] - lb[:, 0]),
                    ("lb:publish", ev[:, 4] - lb[:, 1])):
        q = np.percentile(d[1:], [5, 50, 95, 99])
        print(f"{name:13s} p5 {q[0]:7.2f}  p50 {q[1]:7.2f}  p95 {q[2]:7.2f}  p99 {q[3]:7.2f}")
    sub = (t[:, [1, 13, 14, 2]] - t0) / 1e3
    for name, d in (("cnt:own-warp", sub[:, 1] - sub[:, 0]), ("cnt:barrier", sub[:, 2] - sub[:, 1]),
                    ("cnt:publish", sub[:, 3] - sub[:, 2])):
        q = np.percentile(d, [5, 50, 95, 99])
        print(f"{name:13s} p5 {q[0]:7.2f}  p50 {q[1]:7.2f}  p95 {q[2]:7.2f}  p99 {q[3]:7.2f}")
    print("rounds p50/p99", np.percentile(t[1:, 8], [50, 99]), "polls p50/p99", np.percentile(t[1:, 9], [50, 99]))
    agg_max_lower = np.maximum.accumulate(np.concatenate([[0.0], ev[:-1, 2]]))
    ready = np.maximum(agg_max_lower, ev[:, 3])  # every lower AGG published and look-back started
    for name, d in (("wait-for-lower-AGG", agg_max_lower - ev[:, 3]), ("incl-after-ready", ev[:, 4] - ready)):
        q = np.percentile(d[1:], [5, 50, 95, 99])
        print(f"{name:19s} p5 {q[0]:7.2f}  p50 {q[1]:7.2f}  p95 {q[2]:7.2f}  p99 {q[3]:7.2f}")
    # ranker occupancy: busy = own tile (landed .. compacted), gap = until the CTA's next tile lands
    sm = t[:, 7]
    r1, r15 = (t[:, 1] - t0) / 1e3, (t[:, 15] - t0) / 1e3
    busy = r15 - r1
    gaps = []
    for s_ in np.unique(sm):
        idx = np.where(sm == s_)[0]
        idx = idx[np.argsort(r1[idx])]
        gaps.append(r1[idx[1:]] - r15[idx[:-1]])
    gaps = np.concatenate(gaps)
    for name, d in (("rank:busy", busy), ("rank:gap", gaps), ("rank:agg->end", r15 - ev[:, 2])):
        q = np.percentile(d, [5, 50, 95, 99])
        print(f"{name:13s} p5 {q[0]:7.2f}  p50 {q[1]:7.2f}  p95 {q[2]:7.2f}  p99 {q[3]:7.2f}  mean {d.mean():7.2f}")
    total = ev[:, 6] - ev[:, 0]
    print(f"{'tile':9s} p50 {np.median(total):7.2f} mean {total.mean():7.2f}")
    # how far behind the newest drawn tile is the INCL frontier, sampled over time
    order = np.argsort(ev[:, 0])
    print("draw order vs ticket order: max |rank-ticket| =",
          int(np.max(np.abs(np.arange(ntiles) - np.argsort(order)))))
    sms = np.bincount(t[:, 7].astype(np.int64))
    print("tiles per SM: min", sms[sms > 0].min(), "max", sms.max(), "SMs used", int((sms > 0).sum()))
    np.save("gpurun_out/trace.npy", t)


if __name__ == "__main__":
    main()
