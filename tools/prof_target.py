"""Small target for ncu: one op at one size, a few launches.

    python tools/prof_target.py compact 268435456 0.5
    python tools/prof_target.py pad 4000 3990 4000
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dsgen  # noqa: E402
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402


def main():
    op = sys.argv[1]
    reps = int(os.environ.get("REPS", "3"))
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    if op in ("compact", "select", "unique"):
        n, f = int(sys.argv[2]), float(sys.argv[3])
        if op == "compact":
            src = dsgen.compact_input(n, f, dsgen.seed_for(3, 5), device="cuda")
            fn = lambda w: libds.ds_compact_ex(w, n, 0, d_n, None)  # noqa: E731
        elif op == "select":
            src = dsgen.select_input(n, 3, device="cuda")
            t = dsgen.select_threshold(f) & 0xFFFFFFFF
            fn = lambda w: libds.ds_select_ex(w, n, 1, t, d_n, None)  # noqa: E731
        else:
            src = dsgen.unique_runs_input(n, f, 5, device="cuda")
            fn = lambda w: libds.ds_unique_ex(w, n, None, 0, d_n, None)  # noqa: E731
    else:
        R, C, NC = (int(x) for x in sys.argv[2:5])
        src = dsgen.matrix_input(R, C, NC, 4, device="cuda")
        if op == "pad":
            fn = lambda w: libds.ds_pad_ex(w, R, C, NC, 4, None, None)  # noqa: E731
        else:
            libds.ds_pad(src, R, NC, C, 4) if False else None
            fn = lambda w: libds.ds_unpad_ex(w, R, C, NC, 4, None)  # noqa: E731
    work = torch.empty_like(src)
    for _ in range(reps):
        work.copy_(src)
        fn(work)
    torch.cuda.synchronize()
    print("done", int(d_n.item()))


if __name__ == "__main__":
    main()
