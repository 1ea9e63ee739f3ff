"""Partition time breakdown (development aid, not the bench): in-place
ds_partition_ex (DS pass + tail copy) vs ds_partition_copy_ex (DS pass only)
vs a torch copy of the false half (the tail copy's lower bound)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dsgen  # noqa: E402
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402

dev = torch.device("cuda")
flush = torch.empty(256 << 20, dtype=torch.int32, device=dev)


def timeit(name, pristine, fn, reps=15):
    work = pristine.clone()
    ts = []
    for r in range(reps + 3):
        work.copy_(pristine)
        flush.sum()
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn(work)
        e.record()
        torch.cuda.synchronize()
        if r >= 3:
            ts.append(s.elapsed_time(e) * 1e3)
    ts.sort()
    print(f"{name:44s} median {ts[len(ts) // 2]:8.1f} us  min {ts[0]:8.1f} us", flush=True)


def main():
    n = 1 << 28
    a = dsgen.select_input(n, 3, device=dev)
    t = dsgen.select_threshold(0.5) & 0xFFFFFFFF
    aux = torch.empty(n, dtype=torch.int32, device=dev)
    o1 = torch.empty(n, dtype=torch.int32, device=dev)
    o2 = torch.empty(n, dtype=torch.int32, device=dev)
    d_n = torch.zeros(1, dtype=torch.int64, device=dev)
    P = libds.DS_PRED_I32_GT
    timeit("partition_ex (in place, aux)", a, lambda w: libds.ds_partition_ex(w, n, P, t, aux, d_n))
    timeit("partition_copy_ex (DS pass only)", a, lambda w: libds.ds_partition_copy_ex(w, n, P, t, o1, o2, d_n))
    timeit("select_copy_ex", a, lambda w: libds.ds_select_copy_ex(w, n, P, t, o1, d_n))
    half = n // 2
    timeit("torch copy n/2 words (aligned)", a, lambda w: o1[:half].copy_(aux[:half]))
    timeit("torch copy n/2 words (dst +1 word)", a, lambda w: o1[1:half + 1].copy_(aux[:half]))


if __name__ == "__main__":
    main()
