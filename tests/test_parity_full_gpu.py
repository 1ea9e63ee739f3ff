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


@pytest.mark.parametrize("R,C,NC,eb", [(16384, 16383, 16384, 4), (16384, 16383, 16384, 8),
                                       (12000, 11999, 12000, 4)])
def test_pad_unpad_bench_shapes(R, C, NC, eb):
    """The bench's pad / unpad rows at >= 256M elements (f32 and 8-byte
    elements) and the Table-I shape: whole buffer."""
    dev = dsgen.matrix_input(R, C, NC, eb, device="cuda")
    exp = dev.cpu().numpy().view(np.uint32).copy()
    oracle.pad(exp, R, C, NC, eb)
    libds.ds_pad_ex(dev, R, C, NC, eb, None, None)
    torch.cuda.synchronize()
    assert np.array_equal(dev.cpu().numpy().view(np.uint32), exp)
    oracle.unpad(exp, R, NC, C, eb)
    libds.ds_unpad_ex(dev, R, NC, C, eb, None)
    torch.cuda.synchronize()
    assert np.array_equal(dev.cpu().numpy().view(np.uint32), exp)


def test_pad_unpad_bytes_bench_shape():
    """1-byte elements at 16384 x 16383 <-> 16384 (the byte-granular kernel)."""
    R, C, NC = 16384, 16383, 16384
    g = torch.Generator(device="cuda").manual_seed(7)
    dev = torch.randint(0, 256, (R * NC,), dtype=torch.uint8, device="cuda", generator=g)
    exp = dev.cpu().numpy().copy()
    oracle.pad(exp, R, C, NC, 1)
    libds.ds_pad_ex(dev, R, C, NC, 1, None, None)
    torch.cuda.synchronize()
    assert np.array_equal(dev.cpu().numpy(), exp)
    oracle.unpad(exp, R, NC, C, 1)
    libds.ds_unpad_ex(dev, R, NC, C, 1, None)
    torch.cuda.synchronize()
    assert np.array_equal(dev.cpu().numpy(), exp)


def test_partition_256m():
    """The bench's partition row (in place through aux), whole buffer."""
    n = 1 << 28
    dev = dsgen.select_input(n, dsgen.seed_for(5), device="cuda")
    t = dsgen.select_threshold(0.5) & 0xFFFFFFFF
    exp = dev.cpu().numpy().view(np.uint32).copy()
    m = oracle.partition(exp, oracle.PRED_I32_GT, t)
    aux = torch.empty_like(dev)
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    libds.ds_partition_ex(dev, n, libds.DS_PRED_I32_GT, t, aux, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == m
    assert np.array_equal(dev.cpu().numpy().view(np.uint32), exp)


@pytest.mark.parametrize("mis", [1, 3])
def test_c4_compact_1g_misaligned(mis):
    """Full size at a misaligned pointer (tile grid shifted by mis words)."""
    n = (1 << 30) - 5
    base = dsgen.compact_input(n + 8, 0.5, dsgen.seed_for(3, 7), kind="f32", device="cuda")
    dev = base[mis:mis + n]
    exp = base.cpu().numpy().view(np.uint32).copy()
    m = oracle.compact(exp[mis:mis + n], 0)
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    libds.ds_compact_ex(dev, n, 0, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == m
    assert np.array_equal(base.cpu().numpy().view(np.uint32), exp)
