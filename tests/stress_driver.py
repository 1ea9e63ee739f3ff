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
        _more(rep, d_n)
    print(f"stress OK: {reps} reps with {libds.LIB_PATH}")


def _dev(host_u32, mis):
    """Device copy of host words starting `mis` words past a 16-byte boundary
    (+ the tensor that owns the memory)."""
    t = torch.zeros(host_u32.size + 8, dtype=torch.int32, device="cuda")
    t[mis:mis + host_u32.size] = torch.from_numpy(host_u32.view(np.int32))
    return t, t[mis:mis + host_u32.size]


def _more(rep, d_n):
    """The other kernel paths under the same reordering: partition (in place
    through aux, and out of place), out-of-place select, 8-byte elements,
    byte-granular pad/unpad, and ds_slide, at misaligned pointer phases."""
    mis = rep % 4
    n = 300_007 + rep
    f = [0.0, 0.3, 0.5, 0.97, 1.0][rep % 5]
    t = dsgen.select_threshold(f) & 0xFFFFFFFF
    host = dsgen.select_input(n, 3000 + rep).numpy().view(np.uint32).copy()
    # partition in place through aux
    own, a = _dev(host, mis)
    aown, aux = _dev(np.zeros(n, dtype=np.uint32), (mis + 1) % 4)
    exp = host.copy()
    m = oracle.partition(exp, oracle.PRED_I32_GT, t)
    libds.ds_partition_ex(a, n, libds.DS_PRED_I32_GT, t, aux, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == m and np.array_equal(u32(a), exp), ("partition", rep)
    # partition_copy and select_copy (out of place)
    own, a = _dev(host, mis)
    town, ot = _dev(np.zeros(n, dtype=np.uint32), (mis + 2) % 4)
    fown, of = _dev(np.zeros(n, dtype=np.uint32), (mis + 3) % 4)
    keep = (host.view(np.int32) > np.int32(t if t < 2**31 else t - 2**32))
    libds.ds_partition_copy_ex(a, n, libds.DS_PRED_I32_GT, t, ot, of, d_n, None)
    torch.cuda.synchronize()
    k = int(keep.sum())
    assert int(d_n.item()) == k, ("partition_copy count", rep)
    assert np.array_equal(u32(ot)[:k], host[keep]) and np.array_equal(u32(of)[:n - k], host[~keep])
    kept = oracle.select_copy(host, oracle.PRED_I32_GT, t)
    libds.ds_select_copy_ex(a, n, libds.DS_PRED_I32_GT, t, ot, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == kept.size and np.array_equal(u32(ot)[:kept.size], kept), ("select_copy", rep)
    # 8-byte elements
    rng = np.random.default_rng(rep)
    h64 = np.where(rng.random(n // 2) < f, rng.integers(1, 2**63, n // 2, dtype=np.int64), 0).view(np.uint64)
    own, a = _dev(h64.view(np.uint32), 2 * (rep % 2))
    exp = h64.copy()
    m = oracle.compact64(exp, 0)
    libds.ds_compact64_ex(a, h64.size, 0, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == m and np.array_equal(u32(a).view(np.uint64), exp), ("compact64", rep)
    runs = np.repeat(rng.integers(0, 3, n // 2, dtype=np.int64), 3)[:n // 2].view(np.uint64)
    own, a = _dev(runs.view(np.uint32), 2 * (rep % 2))
    exp = runs.copy()
    m = oracle.unique64(exp)
    libds.ds_unique64_ex(a, runs.size, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == m and np.array_equal(u32(a).view(np.uint64), exp), ("unique64", rep)
    # byte-granular pad / unpad (rows not whole words)
    for (R, C, NC, eb) in ((2000, 999, 1003, 1), (700, 1501, 1510, 2)):
        hb = rng.integers(0, 256, R * NC * eb, dtype=np.uint8)
        tb = torch.zeros(hb.size + 64, dtype=torch.uint8, device="cuda")
        off = (rep * eb) % 16
        tb[off:off + hb.size] = torch.from_numpy(hb)
        view = tb[off:off + hb.size]
        exp = hb.copy()
        oracle.pad(exp, R, C, NC, eb)
        libds.ds_pad_ex(view, R, C, NC, eb, None, None)
        torch.cuda.synchronize()
        assert np.array_equal(view.cpu().numpy(), exp), ("pad bytes", rep, eb)
        oracle.unpad(exp, R, NC, C, eb)
        libds.ds_unpad_ex(view, R, NC, C, eb, None)
        torch.cuda.synchronize()
        assert np.array_equal(view.cpu().numpy(), exp), ("unpad bytes", rep, eb)
    # slide
    for shift in (1, 8195, 100_003):
        own, a = _dev(host, mis)
        exp = host.copy()
        oracle.slide(exp, n, shift, 4)
        libds.ds_slide_ex(a, n, shift, 4, None)
        torch.cuda.synchronize()
        assert np.array_equal(u32(a), exp), ("slide", rep, shift)


def main_large(reps):
    """Full-size reordering stress (R10): 256M-word compaction at f = 0.1 /
    0.5 / 0.9 and unique, `reps` launches each, every result compared with
    the oracle's (computed once per input)."""
    n = 1 << 28
    cases = []
    for f in (0.1, 0.5, 0.9):
        cases.append(("compact", dsgen.compact_input(n, f, 4000 + int(10 * f), device="cuda")))
    cases.append(("unique", dsgen.unique_runs_input(n, 0.4, 4100, device="cuda")))
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    for kind, src in cases:
        exp = u32(src)
        m = oracle.unique(exp) if kind == "unique" else oracle.compact(exp, 0)
        want = torch.from_numpy(exp.view(np.int32)).cuda()
        work = torch.empty_like(src)
        for rep in range(reps):
            work.copy_(src)
            if kind == "unique":
                libds.ds_unique_ex(work, n, None, 0, d_n, None)
            else:
                libds.ds_compact_ex(work, n, 0, d_n, None)
            assert int(d_n.item()) == m and torch.equal(work, want), (kind, rep)
        del want, work
    print(f"stress OK: large, {reps} reps x {len(cases)} inputs with {libds.LIB_PATH}")


if __name__ == "__main__":
    if len(sys.argv) > 2 and sys.argv[2] == "large":
        main_large(int(sys.argv[1]))
    else:
        main(int(sys.argv[1]) if len(sys.argv) > 1 else 10)
