"""GPU parity at BASELINE.json's full sizes, in the launch configuration
bench.py times (the _ex forms on torch's stream, count to device memory).
The C oracle computes every output at these sizes (it is a single pass), so
the comparison is still the whole buffer, bit-exact.

  C1  compaction of 1M int32, 50 %
  C2  pad 4000x3990 -> 4000 f32 and unpad back   (tests/test_parity_gpu.py)
  C3  select (x > t) and unique on 256M int32, f in {0, 0.5, 1}
  C4  compaction of 1G float32 at 10 / 50 / 90 %
  C5  compaction of 4G int32 at 50 % (one GPU holds the whole array)
"""
import numpy as np
import pytest
import torch

import dsgen
import oracle
from paper_conf_icpp_gomez_lunacshg15_b200 import libds

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


def _host_ram_gb():
    try:
        import psutil
        return psutil.virtual_memory().available / 2**30
    except Exception:  # pragma: no cover
        return 0.0


def _run(dev, host_expected, m_exp, op, *args):
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    n = dev.numel()
    if op == "compact":
        libds.ds_compact_ex(dev, n, args[0], d_n, None)
    elif op == "select":
        libds.ds_select_ex(dev, n, args[0], args[1], d_n, None)
    elif op == "unique":
        libds.ds_unique_ex(dev, n, None, 0, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == m_exp
    got = dev.cpu().numpy().view(np.uint32)
    assert np.array_equal(got, host_expected)


def test_c1_compact_1m():
    n = 1 << 20
    dev = dsgen.compact_input(n, 0.5, dsgen.seed_for(0), device="cuda")
    exp = dev.cpu().numpy().view(np.uint32).copy()
    m = oracle.compact(exp, 0)
    _run(dev, exp, m, "compact", 0)


@pytest.mark.parametrize("f", [0.0, 0.5, 1.0])
def test_c3_select_256m(f):
    n = 1 << 28
    dev = dsgen.select_input(n, dsgen.seed_for(2, int(f * 10)), device="cuda")
    t = dsgen.select_threshold(f) & 0xFFFFFFFF
    exp = dev.cpu().numpy().view(np.uint32).copy()
    m = oracle.select(exp, oracle.PRED_I32_GT, t)
    _run(dev, exp, m, "select", libds.DS_PRED_I32_GT, t)


@pytest.mark.parametrize("variant", ["runs0.0", "runs0.5", "runs1.0", "hashed0.5"])
def test_c3_unique_256m(variant):
    n = 1 << 28
    f = float(variant[-3:])
    gen = dsgen.unique_hashed_input if variant.startswith("hashed") else dsgen.unique_runs_input
    dev = gen(n, f, dsgen.seed_for(2, 11 + int(f * 10)), device="cuda")
    exp = dev.cpu().numpy().view(np.uint32).copy()
    m = oracle.unique(exp)
    _run(dev, exp, m, "unique")


@pytest.mark.parametrize("f", [0.1, 0.5, 0.9])
def test_c4_compact_1g_f32(f):
    n = 1 << 30
    dev = dsgen.compact_input(n, f, dsgen.seed_for(3, int(f * 10)), kind="f32", device="cuda")
    exp = dev.cpu().numpy().view(np.uint32).copy()
    m = oracle.compact(exp, 0)
    _run(dev, exp, m, "compact", 0)


def test_c5_compact_4g_single_gpu():
    if _host_ram_gb() < 48:
        pytest.skip("needs ~40 GB of host RAM for the whole-buffer comparison")
    n = 1 << 32
    dev = dsgen.compact_input(n, 0.5, dsgen.seed_for(4), device="cuda")
    exp = dev.cpu().numpy().view(np.uint32).copy()
    m = oracle.compact(exp, 0)
    _run(dev, exp, m, "compact", 0)
