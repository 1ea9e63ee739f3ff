"""Scheduling-stress parity run (T3), executed in a subprocess by
tests/test_stress_gpu.py with LIBDS_PATH pointing at libds_stress.so, the
build with -DDS_DEBUG_DELAY: every CTA sleeps pseudo-random 0..4 us between
ticket, load, publish and store, reordering the pipeline across CTAs.
Every result is compared bit-exact with the oracle; exits non-zero on the
first mismatch."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import dsgen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_icpp_gomez_lunacshg15_b200 import libds  # noqa: E402



def u32(t):
    return t.cpu().numpy().view(np.uint32).copy()


def main(reps):
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    for rep in range(reps):
        for n in (1 << 20, 3 * 8192 + 5, 700_001):
            f = [0.0, 0.3, 0.5, 0.97, 1.0][rep % 5]
            a = dsgen.compact_input(n, f, 1000 + rep, device="cuda")
            exp = u32(a)
            m = oracle.compact(exp, 0)
            libds.ds_compact_ex(a, n, 0, d_n, None)
            torch.cuda.synchronize()
            assert int(d_n.item()) == m and np.array_equal(u32(a), exp), ("compact", rep, n)

            a = dsgen.unique_runs_input(n, f, 2000 + rep, device="cuda")
            exp = u32(a)
            m = oracle.unique(exp)
            libds.ds_unique_ex(a, n, None, 0, d_n, None)
            torch.cuda.synchronize()
            assert int(d_n.item()) == m and np.array_equal(u32(a), exp), ("unique", rep, n)
        for (R, C, NC) in ((3000, 1999, 2003), (1000, 1, 300), (50, 20000, 19990)):
            a = dsgen.matrix_input(R, C, NC, 4, device="cuda")
            exp = u32(a)
            if NC >= C:
                oracle.pad(exp, R, C, NC, 4)
                libds.ds_pad_ex(a, R, C, NC, 4, None, None)
            else:
                oracle.unpad(exp, R, C, NC, 4)
                libds.ds_unpad_ex(a, R, C, NC, 4, None)
            torch.cuda.synchronize()
            assert np.array_equal(u32(a), exp), ("regular", rep, R, C, NC)
            if NC > C:
                oracle.unpad(exp, R, NC, C, 4)
                libds.ds_unpad_ex(a, R, NC, C, 4, None)
                torch.cuda.synchronize()
                assert np.array_equal(u32(a), exp), ("unpad-back", rep, R, C, NC)
    print(f"stress OK: {reps} reps with {libds.LIB_PATH}")


if __name__ == "__main__":
    main(int(sys.argv[1]) if len(sys.argv) > 1 else 10)
