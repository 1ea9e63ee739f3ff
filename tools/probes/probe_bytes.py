"""Timing of the sub-word (1/2-byte) pad/unpad paths on a few shapes (development aid)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402

dev = torch.device("cuda")
flush = torch.empty(256 << 20, dtype=torch.int32, device=dev)


def t_call(fn, work, src, reps=10):
    ts = []
    for r in range(reps + 3):
        work.copy_(src)
        flush.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        if r >= 3:
            ts.append(a.elapsed_time(b) * 1e3)
    ts.sort()
    return ts[len(ts) // 2]


for (R, C, NC) in ((4000, 3990, 4000), (4000, 3992, 4000), (12000, 11999, 12000), (1000, 16000, 16003)):
    for eb in (1, 2, 4):
        src = torch.randint(0, 256, (R * NC * eb,), dtype=torch.uint8, device=dev)
        work = src.clone()
        us = t_call(lambda: libds.ds_pad_ex(work, R, C, NC, eb, None, None), work, src)
        gb = eb * (R * C + R * NC) / (us * 1e-6) / 1e9
        us2 = t_call(lambda: libds.ds_unpad_ex(work, R, NC, C, eb, None), work, src)
        gb2 = eb * (2 * R * C) / (us2 * 1e-6) / 1e9
        print(f"R={R} C={C} NC={NC} eb={eb}: pad {us:8.1f} us {gb:7.1f} GB/s   unpad {us2:8.1f} us {gb2:7.1f} GB/s",
              flush=True)
