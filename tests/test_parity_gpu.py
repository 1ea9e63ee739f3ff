"""GPU parity (T2): libds CUDA kernels vs the CPU oracle, bit-exact on the
WHOLE buffer including canary words around it (tolerance 0: integer /
indexing work).  Inputs come from dsgen (seeded, shared by both sides).

Sizes span several tiles with ragged tails; the tile sizes are read from the
library (ds_tile_size: T words for the irregular kernel, TR output words for
the regular kernel), and tiles start at the 16-byte boundary at or below
ptr, so a pointer misaligned by `mis` words moves every tile edge by mis.
Pointers are misaligned by 0..3 words; fractions sweep 0..100 %.  Every call
goes through the C ABI (ctypes binding)."""
import numpy as np
import pytest
import torch

import dsgen
import oracle
from gpu_util import DevBuf
from paper_conf_icpp_gomez_lunacshg15_b200 import libds

pytestmark = pytest.mark.gpu

T = libds.ds_tile_size(libds.DS_KERNEL_IRREGULAR)      # irregular input tile (words)
TR = libds.ds_tile_size(libds.DS_KERNEL_REGULAR)       # regular output tile (words)
SIZES = [1, 2, 3, 4, 5, 31, 32, 33, 1000, T - 1, T, T + 1, 2 * T - 1, 2 * T + 1, 3 * T + 7,
         65537, 1_000_003]
FRACS = [0.0, 0.1, 0.5, 0.9, 1.0]


def _u32(t):
    return t.numpy().view(np.uint32).copy()


# ------------------------------------------------------------------ compaction
@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("mis", [0, 1, 2, 3])
def test_compact_sizes_misalignment(n, mis):
    for k, f in enumerate(FRACS):
        a = _u32(dsgen.compact_input(n, f, dsgen.seed_for(0, k + 7 * mis)))
        buf = DevBuf(a, mis)
        exp = buf.host_region()
        m_exp = oracle.compact(exp, 0)
        m = libds.ds_compact(buf.ptr, n, 0)
        assert m == m_exp
        buf.assert_equals(exp, f"compact n={n} mis={mis} f={f}")


def _structured(n, mis=0):
    """Keep masks (kept word = its index + 1, removed = 0) aimed at the tile
    grid the kernel sees: virtual index v = i + mis, tile = v // T."""
    i = np.arange(n, dtype=np.uint32)
    v = i.astype(np.int64) + mis
    keep = lambda m: np.where(m, i + 1, 0).astype(np.uint32)  # noqa: E731
    yield "all_removed_but_last", keep(i == n - 1)
    yield "first_half_removed", keep(i >= n // 2)
    yield "alternating", keep(i % 2 == 1)
    yield "one_per_tile_last_word", keep(v % T == T - 1)
    yield "one_per_tile_first_word", keep(v % T == 0)
    yield "one_per_tile_middle", keep(v % T == T // 2 + 1)
    yield "odd_tiles_only", keep((v // T) % 2 == 1)
    yield "even_tiles_only", keep((v // T) % 2 == 0)
    yield "run_ends_at_tile_edge", keep((v >= T // 2) & (v < 2 * T))
    yield "run_starts_at_tile_edge", keep((v >= T) & (v < 2 * T + 100))
    yield "runs_cross_tiles", keep(((i + 1000) // 3000) % 2 == 0)


@pytest.mark.parametrize("n", [5 * T + 3, 4 * T, 200_000])
@pytest.mark.parametrize("mis", [0, 1, 2, 3])
def test_compact_structured_masks(n, mis):
    for name, a in _structured(n, mis):
        buf = DevBuf(a, mis)
        exp = buf.host_region()
        m_exp = oracle.compact(exp, 0)
        assert libds.ds_compact(buf.ptr, n, 0) == m_exp, name
        buf.assert_equals(exp, f"{name} mis={mis}")


# ----------------------------------------------------------- tile edges
# n = k*T - mis + d: the last tile ends exactly at (d = 0), one word before
# (d = -1) or one word past (d = +1) a tile edge of the kernel's grid.
EDGE_CASES = [(k, mis, d) for k in (1, 2, 3) for mis in range(4) for d in (-1, 0, 1)]


@pytest.mark.parametrize("k,mis,d", EDGE_CASES)
def test_irregular_tile_edges(k, mis, d):
    n = k * T - mis + d
    for j, f in enumerate((0.0, 0.5, 1.0)):
        seed = dsgen.seed_for(0, 100 + 4 * k + mis + 16 * j)
        a = _u32(dsgen.compact_input(n, f, seed))
        buf = DevBuf(a, mis)
        exp = buf.host_region()
        m_exp = oracle.compact(exp, 0)
        assert libds.ds_compact(buf.ptr, n, 0) == m_exp
        buf.assert_equals(exp, f"compact n={n} mis={mis} f={f}")
        u = _u32(dsgen.unique_runs_input(n, f, seed + 1))
        buf = DevBuf(u, mis)
        exp = buf.host_region()
        m_exp = oracle.unique(exp)
        assert libds.ds_unique(buf.ptr, n) == m_exp
        buf.assert_equals(exp, f"unique n={n} mis={mis} f={f}")
        sel = _u32(dsgen.select_input(n, seed + 2))
        t = dsgen.select_threshold(f) & 0xFFFFFFFF
        buf = DevBuf(sel, mis)
        exp = buf.host_region()
        m_exp = oracle.select(exp, libds.DS_PRED_I32_GT, t)
        d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
        libds.ds_select_ex(buf.ptr, n, libds.DS_PRED_I32_GT, t, d_n, None)
        torch.cuda.synchronize()
        assert int(d_n.item()) == m_exp
        buf.assert_equals(exp, f"select n={n} mis={mis} f={f}")


@pytest.mark.parametrize("mis", [0, 1, 2, 3])
def test_unique_structured_tile_edges(mis):
    """Runs whose boundaries sit on the kernel's tile edges."""
    n = 4 * T + 5
    v = np.arange(n, dtype=np.int64) + mis
    cases = {"run_per_tile": v // T, "change_at_last_word": (v + 1) // T,
             "change_at_first_word": np.maximum(v - 1, 0) // T, "one_change_per_tile": (v % T == T - 1).cumsum(),
             "constant": np.zeros(n, dtype=np.int64)}
    for name, ids in cases.items():
        a = (ids * 2654435761 % (1 << 32)).astype(np.uint32)
        buf = DevBuf(a, mis)
        exp = buf.host_region()
        m_exp = oracle.unique(exp)
        assert libds.ds_unique(buf.ptr, n) == m_exp, name
        buf.assert_equals(exp, f"unique {name} mis={mis}")


@pytest.mark.parametrize("k,mis,d", [(k, mis, d) for k in (1, 2, 3) for mis in (0, 1, 3) for d in (-1, 0, 1)])
def test_regular_tile_edges(k, mis, d):
    """Pad / unpad whose output ends at (or one word around) an output-tile
    edge: rows of 7 words padded to 8, rows = (k*TR - mis + d) // 8."""
    out_words = k * TR - mis + d
    R, C, NC = max(1, out_words // 8), 7, 8
    _pad_case(R, C, NC, 4, mis, fill=[0xFEED0000 + k])
    # one long row: the whole output is a single row crossing every edge
    _pad_case(1, out_words - 3, out_words, 4, mis, fill=[0xBEEF0000 + d + 1])


def test_compact_remove_value_bitwise():
    """R13: bitwise equality (-0.0 kept when removing +0.0; NaN removable)."""
    f = np.array([0.0, -0.0, 1.5, np.nan, 0.0, np.nan] * 5000, dtype=np.float32)
    a = f.view(np.uint32).copy()
    for v in (0, int(a[3]), 0x80000000):
        buf = DevBuf(a, 1)
        exp = buf.host_region()
        m_exp = oracle.compact(exp, v)
        assert libds.ds_compact(buf.ptr, a.size, v) == m_exp
        buf.assert_equals(exp, f"v={v:#x}")


def test_compact_ex_stream_and_device_count():
    n = 300_001
    a = _u32(dsgen.compact_input(n, 0.37, 5))
    buf = DevBuf(a, 2)
    exp = buf.host_region()
    m_exp = oracle.compact(exp, 0)
    s = torch.cuda.Stream()
    d_n = torch.full((1,), -1, dtype=torch.int64, device="cuda")
    with torch.cuda.stream(s):
        libds.ds_compact_ex(buf.ptr, n, 0, d_n, s)
    s.synchronize()
    assert int(d_n.item()) == m_exp
    buf.assert_equals(exp, "ex")


def test_compact_repeated_calls_same_stream():
    """Epoch/ticket re-arming across back-to-back launches of different sizes."""
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    for rep in range(40):
        n = [T * 3 + 1, 17, 100_000, 1][rep % 4] + rep
        a = _u32(dsgen.compact_input(n, 0.5, 100 + rep))
        buf = DevBuf(a, rep % 4)
        exp = buf.host_region()
        m_exp = oracle.compact(exp, 0)
        libds.ds_compact_ex(buf.ptr, n, 0, d_n, None)
        torch.cuda.synchronize()
        assert int(d_n.item()) == m_exp
        buf.assert_equals(exp, f"rep {rep}")


def test_compact_repeat_race_hunt():
    """Same medium input 200 times: any ordering bug shows up as a mismatch."""
    n = 4_000_037
    a = _u32(dsgen.compact_input(n, 0.5, 77))
    exp = a.copy()
    m_exp = oracle.compact(exp, 0)
    src = torch.from_numpy(a.view(np.int32)).cuda()
    work = torch.empty_like(src)
    want = torch.from_numpy(exp.view(np.int32)).cuda()
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    for rep in range(200):
        work.copy_(src)
        libds.ds_compact_ex(work, n, 0, d_n, None)
        assert int(d_n.item()) == m_exp, rep
        assert torch.equal(work, want), rep


# ---------------------------------------------------------------------- select
PARAMS = [0, 1, 0x40490FDB, 0xC0000000, 0x7FFFFFFF, 0x7FC00000]


@pytest.mark.parametrize("pred", range(libds.DS_PRED_COUNT))
@pytest.mark.parametrize("n", [1, 33, T + 1, 3 * T + 7, 250_001])
def test_select_predicates(pred, n):
    a = _u32(dsgen.random_words(n, 1000 + pred + n))
    specials = np.array([0, 0x80000000, 0x7FC00000, 0xFFC00001, 0x7F800000, 0xFF800000,
                         0xFFFFFFFF, 1, 2, 0x00000003, 0x80000001], dtype=np.uint32)
    a[::13] = np.resize(specials, a[::13].size)
    for j, param in enumerate(PARAMS):
        buf = DevBuf(a, (j + n) % 4)
        exp = buf.host_region()
        m_exp = oracle.select(exp, pred, param)
        d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
        libds.ds_select_ex(buf.ptr, n, pred, param, d_n, None)
        torch.cuda.synchronize()
        assert int(d_n.item()) == m_exp, (pred, hex(param))
        buf.assert_equals(exp, f"select pred={pred} param={param:#x}")


def test_select_blocking_param_zero():
    a = _u32(dsgen.random_words(77_777, 3))
    for pred in range(libds.DS_PRED_COUNT):
        buf = DevBuf(a, 1)
        exp = buf.host_region()
        m_exp = oracle.select(exp, pred, 0)
        assert libds.ds_select(buf.ptr, a.size, pred) == m_exp
        buf.assert_equals(exp, f"pred {pred}")


@pytest.mark.parametrize("f", [i / 10 for i in range(11)])
def test_select_threshold_sweep(f):
    n = 1 << 20
    a = _u32(dsgen.select_input(n, dsgen.seed_for(2, int(f * 10))))
    t = dsgen.select_threshold(f) & 0xFFFFFFFF
    buf = DevBuf(a, 0)
    exp = buf.host_region()
    m_exp = oracle.select(exp, libds.DS_PRED_I32_GT, t)
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    libds.ds_select_ex(buf.ptr, n, libds.DS_PRED_I32_GT, t, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == m_exp
    buf.assert_equals(exp, f"f={f}")


# ---------------------------------------------------------------------- unique
@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("mis", [0, 3])
def test_unique_runs_and_small_alphabets(n, mis):
    cases = [("runs%.1f" % f, _u32(dsgen.unique_runs_input(n, f, 31 + k)))
             for k, f in enumerate(FRACS)]
    cases += [("bits1", _u32(dsgen.random_words(n, 5, bits=1))),
              ("bits2", _u32(dsgen.random_words(n, 6, bits=2))),
              ("hashed", _u32(dsgen.unique_hashed_input(n, 0.5, 7)))]
    for name, a in cases:
        buf = DevBuf(a, mis)
        exp = buf.host_region()
        m_exp = oracle.unique(exp)
        assert libds.ds_unique(buf.ptr, n) == m_exp, name
        buf.assert_equals(exp, f"unique {name} n={n} mis={mis}")


def test_unique_tile_boundary_runs():
    """Runs that end exactly at / straddle tile boundaries (P:280 boundary read)."""
    n = 8 * T
    i = np.arange(n)
    for period in (T, T // 2, T + 1, 3, 1):
        a = (i // period).astype(np.uint32)
        for mis in range(4):
            buf = DevBuf(a, mis)
            exp = buf.host_region()
            m_exp = oracle.unique(exp)
            assert libds.ds_unique(buf.ptr, n) == m_exp
            buf.assert_equals(exp, f"period {period} mis {mis}")


def test_unique_halo():
    """ds_unique_ex with a halo of earlier shards (R18): nearest non-empty wins."""
    a = np.array([5, 5, 6, 6, 7], dtype=np.uint32)
    cases = [([], None), ([(1 << 32) | 5], 5), ([(1 << 32) | 4], 4),
             ([(1 << 32) | 5, 0], 5), ([(1 << 32) | 9, (1 << 32) | 5, 0, 0], 5), ([0, 0], None)]
    for halo, prev in cases:
        buf = DevBuf(a, 1)
        exp = buf.host_region()
        m_exp = oracle.unique(exp, prev=prev)
        d_halo = torch.tensor(halo if halo else [0], dtype=torch.int64, device="cuda")
        d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
        libds.ds_unique_ex(buf.ptr, a.size, d_halo if halo else None, len(halo), d_n, None)
        torch.cuda.synchronize()
        assert int(d_n.item()) == m_exp, halo
        buf.assert_equals(exp, f"halo {halo}")


# ------------------------------------------------------------------ pad / unpad
def _pad_case(R, C, NC, eb, mis, fill=None, kind="index"):
    w = eb // 4
    a = _u32(dsgen.matrix_input(R, C, NC, eb, kind=kind))
    buf = DevBuf(a, mis, capacity=a.size)
    exp = buf.host_region()
    fb = None if fill is None else np.asarray(fill, dtype=np.uint32).tobytes()
    oracle.pad(exp, R, C, NC, eb, fb)
    if fill is None:
        libds.ds_pad(buf.ptr, R, C, NC, eb)
    else:
        libds.ds_pad_ex(buf.ptr, R, C, NC, eb, fb, None)
    buf.assert_equals(exp, f"pad R={R} C={C} NC={NC} eb={eb} mis={mis}")
    # and back (round trip; unpad leaves the tail as the padded buffer had it)
    back = exp.copy()
    oracle.unpad(back, R, NC, C, eb)
    libds.ds_unpad(buf.ptr, R, NC, C, eb)
    buf.assert_equals(back, f"unpad R={R} C={NC} NC={C} eb={eb} mis={mis}")
    assert np.array_equal(back[:R * C * w], a[:R * C * w])


def test_pad_unpad_brute_force_small():
    for eb in (4, 8, 16):
        w = eb // 4
        fill = [0xF1F1F100 + j for j in range(w)]
        for R in range(1, 5):
            for C in range(0, 6):
                for NC in range(C, 8):
                    _pad_case(R, C, NC, eb, (R + C + NC) % 4, fill)


@pytest.mark.parametrize("shape", [
    (4000, 3990, 4000, 4),      # C2
    (5000, 4900, 5000, 4),      # Fig. 2 / Fig. 8(c,d) shape
    (1000, 1, 4100, 4),         # tiny rows, huge padding: wide windows
    (3, 1_000_000, 1_000_001, 4),
    (1, 1, 100_000, 4),
    (100_000, 1, 3, 4),
    (777, 1023, 1025, 8),
    (333, 257, 300, 16),
    (64, 4096, 8192, 4),
    (4096, 1, 2, 4),
])
@pytest.mark.parametrize("mis", [0, 1])
def test_pad_unpad_shapes(shape, mis):
    R, C, NC, eb = shape
    _pad_case(R, C, NC, eb, mis, fill=[0xABCD0000 + j for j in range(eb // 4)])


def test_pad_c2_f32_values():
    _pad_case(4000, 3990, 4000, 4, 0, kind="f32")


@pytest.mark.parametrize("shape", [(10_000, 5000, 3, 4), (2000, 100_000, 10, 4), (50, 20_000, 19_000, 4),
                                   (5, 3, 1, 16)])
def test_unpad_large_drop_slow_path(shape):
    R, C, NC, eb = shape
    a = _u32(dsgen.matrix_input(R, C, NC, eb))
    for mis in (0, 2):
        buf = DevBuf(a, mis)
        exp = buf.host_region()
        oracle.unpad(exp, R, C, NC, eb)
        libds.ds_unpad(buf.ptr, R, C, NC, eb)
        buf.assert_equals(exp, f"unpad {shape} mis={mis}")


def test_pad_table1_shape():
    """Table I shape: 12000 x 11999 -> 12000, u32 index values."""
    _pad_case(12000, 11999, 12000, 4, 0)


def test_pad_repeat_race_hunt():
    R, C, NC = 2000, 1999, 2003
    a = _u32(dsgen.matrix_input(R, C, NC, 4))
    exp = a.copy()
    oracle.pad(exp, R, C, NC, 4)
    src = torch.from_numpy(a.view(np.int32)).cuda()
    want = torch.from_numpy(exp.view(np.int32)).cuda()
    work = torch.empty_like(src)
    for rep in range(100):
        work.copy_(src)
        libds.ds_pad_ex(work, R, C, NC, 4, None, None)
        assert torch.equal(work, want), rep


# ------------------------------------------------- partition / out-of-place
@pytest.mark.parametrize("n", [1, 5, T - 1, 2 * T + 1, 3 * T + 7, 65537, 1_000_003])
@pytest.mark.parametrize("mis", [0, 3])
def test_partition_in_place(n, mis):
    """Stable partition through the caller's aux buffer."""
    for k, f in enumerate([0.0, 0.3, 0.5, 1.0]):
        a = _u32(dsgen.select_input(n, 400 + k + n))
        t = dsgen.select_threshold(f) & 0xFFFFFFFF
        buf = DevBuf(a, mis)
        exp = buf.host_region()
        m_exp = oracle.partition(exp, oracle.PRED_I32_GT, t)
        aux = DevBuf(np.zeros(n, dtype=np.uint32), (mis + 1) % 4)
        d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
        libds.ds_partition_ex(buf.ptr, n, libds.DS_PRED_I32_GT, t, aux.ptr, d_n, None)
        torch.cuda.synchronize()
        assert int(d_n.item()) == m_exp, (n, f)
        buf.assert_equals(exp, f"partition n={n} f={f}")
        aux_got = aux.fetch()
        assert np.array_equal(aux_got[:aux.pre], aux.expected_full[:aux.pre])          # canaries
        assert np.array_equal(aux_got[aux.pre + n:], aux.expected_full[aux.pre + n:])


def test_partition_blocking_even_odd():
    """Fig. 18 style: evens (true) before odds, both stable; blocking form."""
    a = _u32(dsgen.random_words(300_007, 8))
    buf = DevBuf(a, 1)
    exp = buf.host_region()
    m_exp = oracle.partition(exp, oracle.PRED_I32_EVEN)
    aux = torch.empty(a.size, dtype=torch.int32, device="cuda")
    assert libds.ds_partition(buf.ptr, a.size, libds.DS_PRED_I32_EVEN, aux) == m_exp
    buf.assert_equals(exp, "partition even")


@pytest.mark.parametrize("n", [3, T + 1, 250_001])
@pytest.mark.parametrize("mis_in,mis_out", [(0, 0), (1, 2), (3, 1)])
def test_select_copy_out_of_place(n, mis_in, mis_out):
    a = _u32(dsgen.random_words(n, 500 + n))
    src = DevBuf(a, mis_in)
    out = DevBuf(np.full(n, 0x12345678, dtype=np.uint32), mis_out)
    exp_out = out.host_region()
    kept = oracle.select_copy(a, oracle.PRED_F32_GT, 0x3F000000)
    exp_out[:kept.size] = kept
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    libds.ds_select_copy_ex(src.ptr, n, libds.DS_PRED_F32_GT, 0x3F000000, out.ptr, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == kept.size
    out.assert_equals(exp_out, "select_copy out")
    src.assert_equals(a, "select_copy input unchanged")


@pytest.mark.parametrize("n", [7, 2 * T + 3, 400_009])
def test_partition_copy_out_of_place(n):
    a = _u32(dsgen.random_words(n, 600 + n))
    src = DevBuf(a, 2)
    ot = DevBuf(np.zeros(n, dtype=np.uint32), 1)
    of = DevBuf(np.zeros(n, dtype=np.uint32), 3)
    keep = (a & 1) == 1
    et, ef = ot.host_region(), of.host_region()
    et[:keep.sum()] = a[keep]
    ef[:(~keep).sum()] = a[~keep]
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    libds.ds_partition_copy_ex(src.ptr, n, libds.DS_PRED_I32_ODD, 0, ot.ptr, of.ptr, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == int(keep.sum())
    ot.assert_equals(et, "trues")
    of.assert_equals(ef, "falses")
    src.assert_equals(a, "input unchanged")


# ---------------------------------------------------------------- slide
@pytest.mark.parametrize("n,shift", [(1, 1), (2, 1), (5, 0), (9, 4), (T, 1), (3 * T + 7, 5),
                                     (65537, 65536), (1_000_003, 3), (1_000_003, 12_345),
                                     (1_000_003, 500_001), (300_000, 2 * 8192 + 1)])
@pytest.mark.parametrize("eb", [4, 8, 16])
@pytest.mark.parametrize("mis", [0, 1, 3])
def test_slide(n, shift, eb, mis):
    w = eb // 4
    a = ((np.arange(n * w, dtype=np.uint64) * 2654435761 + 12345) & 0xFFFFFFFF).astype(np.uint32)
    buf = DevBuf(a, mis)
    exp = buf.host_region()
    oracle.slide(exp, n, shift, eb)
    libds.ds_slide(buf.ptr, n, shift, eb)
    buf.assert_equals(exp, f"slide n={n} shift={shift} eb={eb} mis={mis}")


def test_slide_ex_stream_repeated():
    """Back-to-back slides on one stream (ticket/epoch re-arming across launches)."""
    n = 200_003
    a = dsgen.compact_input(n, 0.5, 99).numpy().view(np.uint32).copy()
    buf = DevBuf(a, 2)
    exp = buf.host_region()
    s = torch.cuda.Stream()
    for shift in (1, 7, 8192, 3, 40_000):
        oracle.slide(exp, n, shift, 4)
        libds.ds_slide_ex(buf.ptr, n, shift, 4, s)
    s.synchronize()
    buf.assert_equals(exp, "slide repeated")


# ------------------------------------------------------ 8-byte elements
SIZES64 = [1, 2, 3, 16, T // 2 - 1, T // 2, T // 2 + 1, T - 1, 3 * (T // 2) + 5, 100_003, 1_000_003]  # elements (T/2 per tile)


def _dev64(host, mis):
    """DevBuf over the uint64 array's words; mis in {0, 2} keeps 8-byte alignment."""
    return DevBuf(host.view(np.uint32), mis)


@pytest.mark.parametrize("n", SIZES64)
@pytest.mark.parametrize("mis", [0, 2])
def test_compact64(n, mis):
    rng = np.random.default_rng(n + mis)
    for f in (0.0, 0.3, 1.0):
        vals = rng.integers(1, 2**64, size=n, dtype=np.uint64)
        rm = np.uint64(0xABCD000000000000)
        host = np.where(rng.random(n) < f, vals, rm).astype(np.uint64)
        host[::11] = rm ^ np.uint64(1 << 32)  # same low word as the removed value: kept
        buf = _dev64(host, mis)
        exp = buf.host_region()
        m_exp = oracle.compact64(exp.view(np.uint64), int(rm))
        m = libds.ds_compact64(buf.ptr, n, int(rm))
        assert m == m_exp
        buf.assert_equals(exp, f"compact64 n={n} mis={mis} f={f}")


@pytest.mark.parametrize("pred", range(libds.DS_PRED_COUNT))
@pytest.mark.parametrize("n", [5, 4097, 250_001])
def test_select64(pred, n):
    rng = np.random.default_rng(pred * 7 + n)
    if pred in (3, 4):
        d = rng.normal(size=n)
        d[::13] = np.nan
        host = d.view(np.uint64).copy()
        param = int(np.array([0.1]).view(np.uint64)[0])
    else:
        host = rng.integers(-2**62, 2**62, size=n, dtype=np.int64).view(np.uint64).copy()
        host[::5] = 0
        param = 1 << 40
    buf = _dev64(host, 2)
    exp = buf.host_region()
    m_exp = oracle.select64(exp.view(np.uint64), pred, param)
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    libds.ds_select64_ex(buf.ptr, n, pred, param, d_n, None)
    torch.cuda.synchronize()
    assert int(d_n.item()) == m_exp
    buf.assert_equals(exp, f"select64 pred={pred} n={n}")


@pytest.mark.parametrize("n", SIZES64)
def test_unique64(n):
    rng = np.random.default_rng(3 * n)
    letters = np.array([7, 7 + (1 << 32), 1 << 63], dtype=np.uint64)
    runs = rng.integers(1, 5, size=n)
    host = np.repeat(rng.choice(letters, size=n), runs)[:n].astype(np.uint64)
    buf = _dev64(host, 0)
    exp = buf.host_region()
    m_exp = oracle.unique64(exp.view(np.uint64))
    assert libds.ds_unique64(buf.ptr, n) == m_exp
    buf.assert_equals(exp, f"unique64 n={n}")


# ------------------------------------------------- 1- and 2-byte elements (8(f)-4)
class ByteBuf:
    """Device bytes at a chosen byte offset past a 16-byte boundary, with 64
    canary bytes on each side; compared as a whole."""

    def __init__(self, host_bytes, mis):
        self.pre = 64 + mis
        full = np.empty(self.pre + host_bytes.size + 64, dtype=np.uint8)
        full[:self.pre] = (np.arange(self.pre) * 7 + 3).astype(np.uint8)
        full[self.pre:self.pre + host_bytes.size] = host_bytes
        full[self.pre + host_bytes.size:] = (np.arange(64) * 11 + 5).astype(np.uint8)
        self.full = full
        self.n = host_bytes.size
        self.t = torch.from_numpy(full.copy()).to("cuda")
        assert self.t.data_ptr() % 16 == 0

    @property
    def ptr(self):
        return self.t.data_ptr() + self.pre

    def region(self):
        return self.full[self.pre:self.pre + self.n].copy()

    def check(self, region, what):
        torch.cuda.synchronize()
        got = self.t.cpu().numpy()
        exp = self.full.copy()
        exp[self.pre:self.pre + self.n] = region
        if not np.array_equal(got, exp):
            bad = np.nonzero(got != exp)[0]
            raise AssertionError(f"{what}: {bad.size} bytes differ, first at {int(bad[0]) - self.pre}")


def _sub_word_case(R, C, NC, eb, mis, fill):
    rng = np.random.default_rng(R * 1000003 + C * 131 + NC + eb)
    host = rng.integers(0, 256, size=R * NC * eb, dtype=np.uint8)
    buf = ByteBuf(host, mis)
    exp = buf.region()
    oracle.pad(exp, R, C, NC, eb, fill)
    libds.ds_pad_ex(buf.ptr, R, C, NC, eb, fill, None)
    buf.check(exp, f"pad R={R} C={C} NC={NC} eb={eb} mis={mis}")
    back = exp.copy()
    oracle.unpad(back, R, NC, C, eb)
    libds.ds_unpad(buf.ptr, R, NC, C, eb)
    buf.check(back, f"unpad R={R} C={NC} NC={C} eb={eb} mis={mis}")


def test_sub_word_pad_unpad_small_all():
    for eb in (1, 2):
        fill = bytes([0xC3, 0x3C][:eb])
        for R in (1, 2, 3, 5):
            for C in range(0, 7):
                for NC in range(C, 10):
                    _sub_word_case(R, C, NC, eb, (R + C + NC) * eb % 16, fill)


@pytest.mark.parametrize("shape", [
    (4000, 3990, 4000, 1),     # C2 shape in bytes (rows not whole words)
    (4000, 3990, 4000, 2),
    (5000, 4900, 5000, 1),
    (777, 1023, 1025, 2),
    (3, 1_000_001, 1_000_003, 1),
    (100_000, 3, 5, 1),        # tiny rows: byte-wise chunks everywhere
    (2000, 1, 5000, 1),        # huge padding: fill chunks, wide windows
    (300, 20_000, 19_999, 2),  # unpad-style (pad from 19_999 back: see round trip)
    (1000, 4096, 4097, 1),
    (64, 4096, 4100, 2),       # whole words: routed to the word kernel
])
@pytest.mark.parametrize("mis", [0, 1, 6, 15])
def test_sub_word_pad_unpad_shapes(shape, mis):
    R, C, NC, eb = shape
    if NC < C:
        C, NC = NC, C
    if eb == 2 and mis % 2:
        mis -= 1
    _sub_word_case(R, C, NC, eb, mis, bytes([0x81, 0x18][:eb]))


def test_sub_word_unpad_large_drop_slow_path():
    """Short rows dropping many bytes: the source span exceeds a stage, so the
    producer gathers byte by byte from global memory."""
    for (R, C, NC, eb) in ((20_000, 5000, 3, 1), (3000, 20_001, 7, 2)):
        host = np.random.default_rng(R).integers(0, 256, size=R * C * eb, dtype=np.uint8)
        buf = ByteBuf(host, 3 if eb == 1 else 2)
        exp = buf.region()
        oracle.unpad(exp, R, C, NC, eb)
        libds.ds_unpad(buf.ptr, R, C, NC, eb)
        buf.check(exp, f"unpad slow R={R} C={C} NC={NC} eb={eb}")


# ------------------------------------------------------------ host threads
def test_blocking_calls_from_threads():
    """Blocking compact / unique / partition from 6 host threads at once (the
    ctypes calls drop the GIL): every call gets its own count word, so each
    result matches the oracle (partition's shared count)."""
    import threading
    n = 600_011
    jobs = []
    for j in range(6):
        a = _u32(dsgen.select_input(n, 900 + j))
        jobs.append(a)
    results = [None] * len(jobs)

    def work(j):
        a = jobs[j]
        t = dsgen.select_threshold(0.2 + 0.1 * j) & 0xFFFFFFFF
        out = []
        for rep in range(4):
            buf = DevBuf(a, (j + rep) % 4)
            exp = buf.host_region()
            if (j + rep) % 3 == 0:
                m_exp = oracle.compact(exp, int(a[7]))
                m = libds.ds_compact(buf.ptr, n, int(a[7]))
            elif (j + rep) % 3 == 1:
                m_exp = oracle.unique(exp)
                m = libds.ds_unique(buf.ptr, n)
            else:
                exp_p = exp.copy()
                m_exp = oracle.partition(exp_p, oracle.PRED_I32_GT, 0)
                exp = exp_p
                aux = torch.empty(n, dtype=torch.int32, device="cuda")
                m = libds.ds_partition(buf.ptr, n, libds.DS_PRED_I32_GT, aux)
            out.append((m, m_exp, buf, exp))
        results[j] = out

    with torch.cuda.device(0):
        threads = [threading.Thread(target=work, args=(j,)) for j in range(len(jobs))]
        for th in threads:
            th.start()
        for th in threads:
            th.join()
    for j, out in enumerate(results):
        assert out is not None, j
        for m, m_exp, buf, exp in out:
            assert m == m_exp
            buf.assert_equals(exp, f"thread {j}")


def test_select_copy_same_chunk_not_identity():
    """out-of-place select with in and out in the same 16-byte
    chunk (n <= 3, out = in + 2 words) must still write out: the identity-tile
    skip applies only when the output IS the input (same base and phase)."""
    for n in (1, 2):
        for mis in (0, 1):
            t = torch.zeros(16, dtype=torch.int32, device="cuda")
            vals = np.array([0x11, 0x22, 0x33][:n], dtype=np.uint32)
            t[4 + mis:4 + mis + n] = torch.from_numpy(vals.view(np.int32))
            base = t.data_ptr()
            src, dst = base + 4 * (4 + mis), base + 4 * (4 + mis + n)
            d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
            libds.ds_select_copy_ex(src, n, libds.DS_PRED_NONZERO, 0, dst, d_n, None)
            torch.cuda.synchronize()
            got = t.cpu().numpy().view(np.uint32)
            assert int(d_n.item()) == n
            assert np.array_equal(got[4 + mis + n:4 + mis + 2 * n], vals), (n, mis, got)
            assert np.array_equal(got[4 + mis:4 + mis + n], vals)   # input untouched
