"""Small invocation of every libds kernel, for compute-sanitizer (T4):
run under `compute-sanitizer --tool memcheck|racecheck|synccheck` by
tests/test_sanitizer_gpu.py.  PYTORCH_NO_CUDA_MEMORY_CACHING=1 makes every
tensor its own cudaMalloc of the exact size, so memcheck sees reads past an
array's end.  Arrays END at their allocation's end (views at an offset into
a tensor of exactly offset + n words), at every pointer phase.  Each result
is also checked against the oracle; exits non-zero on a mismatch."""
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


def at_end(host_u32, mis):
    """Device words at `mis` words into an allocation that ends with them."""
    t = torch.empty(mis + host_u32.size, dtype=torch.int32, device="cuda")
    t[mis:] = torch.from_numpy(host_u32.view(np.int32))
    return t, t[mis:]


def u32(t):
    return t.cpu().numpy().view(np.uint32).copy()


def check(cond, what):
    if not cond:
        print("MISMATCH", what, flush=True)
        sys.exit(3)


def main():
    which = sys.argv[1] if len(sys.argv) > 1 else "all"
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    T = libds.ds_tile_size(libds.DS_KERNEL_IRREGULAR)
    for mis in range(4):
        for n in (1, 7, T - mis + 1, 2 * T + 3 - mis):
            if which in ("all", "irregular"):
                h = dsgen.compact_input(n, 0.5, 10 + mis + n).numpy().view(np.uint32).copy()
                own, a = at_end(h, mis)
                exp = h.copy()
                m = oracle.compact(exp, 0)
                libds.ds_compact_ex(a, n, 0, d_n, None)
                torch.cuda.synchronize()
                check(int(d_n.item()) == m and np.array_equal(u32(a), exp), ("compact", n, mis))
                h = dsgen.unique_runs_input(n, 0.4, 20 + mis).numpy().view(np.uint32).copy()
                own, a = at_end(h, mis)
                exp = h.copy()
                m = oracle.unique(exp)
                libds.ds_unique_ex(a, n, None, 0, d_n, None)
                torch.cuda.synchronize()
                check(int(d_n.item()) == m and np.array_equal(u32(a), exp), ("unique", n, mis))
                h = dsgen.select_input(n, 30 + mis).numpy().view(np.uint32).copy()
                t = dsgen.select_threshold(0.5) & 0xFFFFFFFF
                own, a = at_end(h, mis)
                aown, aux = at_end(np.zeros(n, dtype=np.uint32), (mis + 1) % 4)
                exp = h.copy()
                m = oracle.partition(exp, oracle.PRED_I32_GT, t)
                libds.ds_partition_ex(a, n, libds.DS_PRED_I32_GT, t, aux, d_n, None)
                torch.cuda.synchronize()
                check(int(d_n.item()) == m and np.array_equal(u32(a), exp), ("partition", n, mis))
                own, a = at_end(h, mis)
                oown, out = at_end(np.zeros(n, dtype=np.uint32), (mis + 2) % 4)
                kept = oracle.select_copy(h, oracle.PRED_I32_GT, t)
                libds.ds_select_copy_ex(a, n, libds.DS_PRED_I32_GT, t, out, d_n, None)
                torch.cuda.synchronize()
                check(int(d_n.item()) == kept.size and np.array_equal(u32(out)[:kept.size], kept),
                      ("select_copy", n, mis))
                if mis % 2 == 0 and n % 2 == 0:
                    h64 = h.view(np.uint64).copy()
                    own, a = at_end(h64.view(np.uint32), mis)
                    exp = h64.copy()
                    m = oracle.compact64(exp, int(h64[0]))
                    libds.ds_compact64_ex(a, h64.size, int(h64[0]), d_n, None)
                    torch.cuda.synchronize()
                    check(int(d_n.item()) == m and np.array_equal(u32(a).view(np.uint64), exp), ("compact64", n))
            if which in ("all", "regular"):
                own, a = at_end(np.arange(n, dtype=np.uint32), mis)
                exp = np.arange(n, dtype=np.uint32)
                shift = max(1, n // 3)
                oracle.slide(exp, n, shift, 4)
                libds.ds_slide_ex(a, n, shift, 4, None)
                torch.cuda.synchronize()
                check(np.array_equal(u32(a), exp), ("slide", n, mis))
        if which in ("all", "regular"):
            for (R, C, NC, eb) in ((37, 129, 133, 4), (5, 2000, 2003, 4), (64, 33, 35, 8), (300, 61, 64, 1),
                                   (90, 77, 80, 2)):
                hb = np.random.default_rng(R + mis).integers(0, 256, R * NC * eb, dtype=np.uint8)
                off = mis * (4 if eb >= 4 else eb)
                tb = torch.empty(off + hb.size, dtype=torch.uint8, device="cuda")
                tb[off:] = torch.from_numpy(hb)
                view = tb[off:]
                exp = hb.copy()
                oracle.pad(exp, R, C, NC, eb)
                libds.ds_pad_ex(view, R, C, NC, eb, None, None)
                torch.cuda.synchronize()
                check(np.array_equal(view.cpu().numpy(), exp), ("pad", R, C, NC, eb, mis))
                oracle.unpad(exp, R, NC, C, eb)
                libds.ds_unpad_ex(view, R, NC, C, eb, None)
                torch.cuda.synchronize()
                check(np.array_equal(view.cpu().numpy(), exp), ("unpad", R, C, NC, eb, mis))
    if which in ("all", "shard"):
        h = dsgen.compact_input(1000, 0.5, 5).numpy().view(np.uint32).copy()
        own, a = at_end(h, 1)
        ent = torch.zeros(2, dtype=torch.int64, device="cuda")
        libds.ds_halo_entry(a, 1000, ent[:1], None)
        libds.ds_shard_offsets(torch.tensor([3, 4, 5], dtype=torch.int64, device="cuda"), 3, 1, ent, None)
        torch.cuda.synchronize()
        check(ent.tolist() == [3, 12], "shard offsets")
    print("sanitize driver OK", flush=True)


if __name__ == "__main__":
    main()
