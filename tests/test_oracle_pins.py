"""Pins for the CPU oracle against things other than itself:
brute force on tiny inputs, the C++ standard library's in-place algorithms,
numpy library routines (boolean masking, numpy.pad, slicing), itertools.groupby,
closed forms on index-tagged data, invariants and the golden worked examples.

A plausible oracle bug (dropped element, off-by-one on the write index, a
comparison with the already-overwritten predecessor in unique, the wrong row
order or shift in pad/unpad, a wrong fill position) fails at least one test.
"""
import ctypes
import itertools
import os
import subprocess

import numpy as np
import pytest

import dsgen
import oracle
from golden_util import all_cases

HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def stdlib(tmp_path_factory):
    d = tmp_path_factory.mktemp("pins")
    so = str(d / "std_pins.so")
    subprocess.check_call(["g++", "-O1", "-std=c++17", "-fPIC", "-shared", "-o", so,
                           os.path.join(HERE, "pins", "std_pins.cpp")])
    L = ctypes.CDLL(so)
    sz, vp, u32 = ctypes.c_size_t, ctypes.c_void_p, ctypes.c_uint32
    L.std_remove.argtypes = [vp, sz, u32]
    L.std_remove.restype = sz
    L.std_unique.argtypes = [vp, sz]
    L.std_unique.restype = sz
    L.std_copy_if_mask.argtypes = [vp, sz, vp]
    L.std_copy_if_mask.restype = sz
    return L


def _p(a):
    return ctypes.c_void_p(a.ctypes.data)


# ----------------------------------------------------------------- compaction
def test_compact_brute_force_all_masks():
    """Every keep-mask for n <= 10 on index-tagged data: a[i] = keep ? i+1 : v.
    The result must be the strictly increasing list of kept tags (stability),
    out_n = popcount(mask), and the tail untouched."""
    v = 0
    for n in range(0, 11):
        for mask in range(1 << n):
            keep = [(mask >> i) & 1 for i in range(n)]
            a = np.array([i + 1 if keep[i] else v for i in range(n)], dtype=np.uint32)
            orig = a.copy()
            m = oracle.compact(a, v)
            exp = [i + 1 for i in range(n) if keep[i]]
            assert m == len(exp)
            assert list(a[:m]) == exp
            assert np.array_equal(a[m:], orig[m:])


@pytest.mark.parametrize("n,bits,seed", [(1, 32, 1), (1000, 2, 2), (4097, 3, 3), (100000, 1, 4)])
def test_compact_equals_std_remove_and_numpy_mask(stdlib, n, bits, seed):
    a = dsgen.random_words(n, seed, bits=bits).numpy().view(np.uint32).copy()
    for v in (0, 1, 0xFFFFFFFF):
        x, y = a.copy(), a.copy()
        m = oracle.compact(x, v)
        m2 = stdlib.std_remove(_p(y), n, v)
        assert m == m2 and np.array_equal(x[:m], y[:m])
        assert np.array_equal(x[:m], a[a != v])  # numpy boolean masking
        assert np.array_equal(x[m:], a[m:])      # tail untouched (R5)


def test_compact_bitwise_float_semantics():
    """R13: equality is bitwise: -0.0 is not removed by remove_value=+0.0 bits,
    and a NaN pattern equals itself."""
    f = np.array([0.0, -0.0, 1.5, np.nan, 0.0, np.nan], dtype=np.float32)
    a = f.view(np.uint32).copy()
    m = oracle.compact(a, 0)
    nanbits = f[3:4].view(np.uint32)[0]
    assert m == 4
    assert list(a[:m]) == [0x80000000, np.float32(1.5).view(np.uint32), nanbits, nanbits]
    b = f.view(np.uint32).copy()
    m = oracle.compact(b, int(nanbits))
    assert m == 4 and nanbits not in set(b[:m].tolist())


def test_compact_invariants_fraction_sweep():
    n = 20000
    for k, f in enumerate([0.0, 0.1, 0.5, 0.9, 1.0]):
        a0 = dsgen.compact_input(n, f, dsgen.seed_for(0, k)).numpy().view(np.uint32)
        a = a0.copy()
        m = oracle.compact(a, 0)
        assert m == np.count_nonzero(a0)
        if f in (0.0, 1.0):
            assert np.array_equal(a, a0)  # byte-identical at f = 0 and 1
        b = a.copy()
        assert oracle.compact(b[:m], 0) == m and np.array_equal(a, b)  # idempotent


# --------------------------------------------------------------------- select
def _numpy_pred(pred, a, param):
    i = a.view(np.int32)
    f = a.view(np.float32)
    p_i = np.array([param], dtype=np.uint32).view(np.int32)[0]
    p_f = np.array([param], dtype=np.uint32).view(np.float32)[0]
    with np.errstate(invalid="ignore"):
        return {
            oracle.PRED_NONZERO: a != 0,
            oracle.PRED_I32_GT: i > p_i,
            oracle.PRED_I32_NOT_GT: ~(i > p_i),
            oracle.PRED_F32_GT: f > p_f,
            oracle.PRED_F32_NOT_GT: ~(f > p_f),
            oracle.PRED_I32_EVEN: (i & 1) == 0,
            oracle.PRED_I32_ODD: (i & 1) == 1,
        }[pred]


@pytest.mark.parametrize("pred", range(oracle.PRED_COUNT))
def test_select_equals_numpy_and_std_copy_if(stdlib, pred):
    n = 30011
    a = dsgen.random_words(n, 77 + pred).numpy().view(np.uint32).copy()
    # sprinkle special float patterns: +-0, NaN, +-inf, negatives
    specials = np.array([0, 0x80000000, 0x7FC00000, 0xFFC00001, 0x7F800000, 0xFF800000,
                         0xFFFFFFFF, 1, 2], dtype=np.uint32)
    a[::37][:] = np.resize(specials, a[::37].size)
    for param in (0, 0x40490FDB, 0xC0000000, 12345, 0x7FC00000):
        keep = _numpy_pred(pred, a, param)
        x, y = a.copy(), a.copy()
        m = oracle.select(x, pred, param)
        keep_u8 = keep.astype(np.uint8)
        m2 = stdlib.std_copy_if_mask(_p(y), n, _p(keep_u8))
        assert m == int(keep.sum()) == m2
        assert np.array_equal(x[:m], a[keep]) and np.array_equal(x[:m], y[:m])
        assert np.array_equal(x[m:], a[m:])


@pytest.mark.parametrize("pair", [(1, 2), (3, 4), (5, 6)])
def test_select_complement_ids_partition(pair):
    a = dsgen.random_words(5000, 5).numpy().view(np.uint32).copy()
    a[::11] = 0x7FC00000  # NaN: F32_GT false, NOT_GT true
    x, y = a.copy(), a.copy()
    m1 = oracle.select(x, pair[0], 0x3F800000)
    m2 = oracle.select(y, pair[1], 0x3F800000)
    assert m1 + m2 == a.size


def test_select_threshold_recipe_counts():
    x = dsgen.select_input(40000, 21).numpy().view(np.uint32)
    for f in (0.0, 0.3, 1.0):
        t = dsgen.select_threshold(f) & 0xFFFFFFFF
        a = x.copy()
        m = oracle.select(a, oracle.PRED_I32_GT, t)
        assert m == np.count_nonzero(x.view(np.int32) > np.int32(np.uint32(t).view(np.int32)))


def test_select_unknown_predicate():
    a = np.arange(5, dtype=np.uint32)
    with pytest.raises(ValueError):
        oracle.select(a, 99)
    assert list(a) == [0, 1, 2, 3, 4]


# ------------------------------------------------------------------ partition
def test_partition_brute_force_all_masks():
    """Every mask for n <= 9 on index-tagged data (odd tag = true under I32_ODD):
    trues in order, then falses in order (stable)."""
    for n in range(0, 10):
        for mask in range(1 << n):
            a = np.array([2 * i + 1 if (mask >> i) & 1 else 2 * i + 2 for i in range(n)], dtype=np.uint32)
            orig = list(a)
            m = oracle.partition(a, oracle.PRED_I32_ODD)
            t = [x for x in orig if x % 2 == 1]
            f = [x for x in orig if x % 2 == 0]
            assert m == len(t) and list(a) == t + f


@pytest.mark.parametrize("pred", range(oracle.PRED_COUNT))
def test_partition_equals_numpy_concat(pred):
    a = dsgen.random_words(20011, 300 + pred).numpy().view(np.uint32).copy()
    keep = _numpy_pred(pred, a, 0x3F800000)
    x = a.copy()
    m = oracle.partition(x, pred, 0x3F800000)
    assert m == int(keep.sum())
    assert np.array_equal(x, np.concatenate([a[keep], a[~keep]]))  # numpy masking + concatenate


def test_select_copy_equals_numpy_and_leaves_input():
    a = dsgen.random_words(10007, 9).numpy().view(np.uint32).copy()
    b = a.copy()
    out = oracle.select_copy(a, oracle.PRED_I32_EVEN)
    assert np.array_equal(a, b)
    assert np.array_equal(out, a[(a & 1) == 0])


# --------------------------------------------------------------------- unique
def test_unique_brute_force_small_alphabet():
    """All sequences over {0,1,2} up to length 7 vs itertools.groupby."""
    for n in range(0, 8):
        for seq in itertools.product(range(3), repeat=n):
            a = np.array(seq, dtype=np.uint32)
            m = oracle.unique(a)
            exp = [k for k, _ in itertools.groupby(seq)]
            assert m == len(exp) and list(a[:m]) == exp
            assert list(a[m:]) == list(seq[m:])


@pytest.mark.parametrize("n,bits", [(1, 32), (2, 1), (1000, 1), (65537, 2), (50000, 32)])
def test_unique_equals_std_unique(stdlib, n, bits):
    a = dsgen.random_words(n, 1234 + n, bits=bits).numpy().view(np.uint32).copy()
    x, y = a.copy(), a.copy()
    m = oracle.unique(x)
    m2 = stdlib.std_unique(_p(y), n)
    assert m == m2 and np.array_equal(x[:m], y[:m])
    assert np.array_equal(x[m:], a[m:])


@pytest.mark.parametrize("f", [0.0, 0.1, 0.5, 1.0])
def test_unique_closed_form_runs(f):
    """a[i] = run id (non-decreasing, +1 w.p. f): output is 0..out_n-1."""
    n = 30000
    a0 = dsgen.unique_runs_input(n, f, 99).numpy().view(np.uint32)
    a = a0.copy()
    m = oracle.unique(a)
    assert m == int(a0[-1]) + 1
    assert np.array_equal(a[:m], np.arange(m, dtype=np.uint32))
    if f == 0.0:
        assert m == 1  # R17: all-equal input keeps exactly the first word
    if f == 1.0:
        assert np.array_equal(a, a0)


def test_unique_invariants_and_prev():
    a0 = dsgen.unique_hashed_input(20000, 0.4, 3).numpy().view(np.uint32)
    a = a0.copy()
    m = oracle.unique(a)
    assert np.all(a[1:m] != a[:m - 1])          # no adjacent equal outputs
    b = a.copy()
    assert oracle.unique(b[:m]) == m            # idempotent
    # shard decomposition with the predecessor rule (R18)
    cut = 7777
    s1, s2 = a0[:cut].copy(), a0[cut:].copy()
    m1 = oracle.unique(s1)
    m2 = oracle.unique(s2, prev=int(a0[cut - 1]))
    assert m1 + m2 == m
    assert np.array_equal(np.concatenate([s1[:m1], s2[:m2]]), a[:m])


def test_unique_prev_rule():
    a = np.array([5, 5, 6], dtype=np.uint32)
    assert oracle.unique(a.copy(), prev=5) == 1
    assert oracle.unique(a.copy(), prev=4) == 2


# ---------------------------------------------------------------- pad / unpad
def _np_pad(mat_words, rows, cols, new_cols, w, fill_words):
    m = mat_words.reshape(rows, cols * w)
    if new_cols == cols:
        return m.reshape(-1).copy()
    out = np.pad(m, ((0, 0), (0, (new_cols - cols) * w)), mode="constant")
    fill_row = np.tile(np.asarray(fill_words, dtype=np.uint32), new_cols - cols)
    out[:, cols * w:] = fill_row
    return out.reshape(-1)


def _fill_bytes(fill_words):
    return np.asarray(fill_words, dtype=np.uint32).tobytes()


def test_pad_unpad_brute_force_small():
    """All R <= 4, C <= 5, NC <= 7, eb in {4, 8}: numpy.pad closed form,
    round trip identity, untouched tail."""
    for eb in (4, 8):
        w = eb // 4
        fillw = [0xA0A0A0A0 + k for k in range(w)]
        for R in range(0, 5):
            for C in range(0, 6):
                for NC in range(C, 8):
                    buf = dsgen.matrix_input(R, C, NC, eb).numpy().view(np.uint32).copy()
                    orig = buf.copy()
                    oracle.pad(buf, R, C, NC, eb, _fill_bytes(fillw))
                    exp = _np_pad(orig[:R * C * w], R, C, NC, w, fillw)
                    assert np.array_equal(buf[:R * NC * w], exp), (R, C, NC, eb)
                    # unpad back
                    oracle.unpad(buf, R, NC, C, eb)
                    assert np.array_equal(buf[:R * C * w], orig[:R * C * w])
                    # unpad leaves [R*C*w, R*NC*w) as the padded buffer had it
                    assert np.array_equal(buf[R * C * w:], exp[R * C * w:])


def test_pad_unpad_sub_word_elements():
    """1- and 2-byte elements (8(f)-4): numpy.pad on the element view, the
    round trip, for every R <= 3, C <= 6, NC <= 9."""
    for eb, dt in ((1, np.uint8), (2, np.uint16)):
        fill = bytes([0xA5, 0x5A][:eb])
        fv = np.frombuffer(fill, dtype=dt)[0]
        for R in range(0, 4):
            for C in range(0, 7):
                for NC in range(C, 10):
                    buf = np.arange(R * NC * eb + 5, dtype=np.uint8) * np.uint8(37) + np.uint8(11)
                    orig = buf.copy()
                    oracle.pad(buf, R, C, NC, eb, fill)
                    m = orig[:R * C * eb].view(dt).reshape(R, C)
                    exp = np.pad(m, ((0, 0), (0, NC - C)), constant_values=fv).reshape(-1).view(np.uint8)
                    assert np.array_equal(buf[:R * NC * eb], exp), (eb, R, C, NC)
                    assert np.array_equal(buf[R * NC * eb:], orig[R * NC * eb:])
                    oracle.unpad(buf, R, NC, C, eb)
                    assert np.array_equal(buf[:R * C * eb], orig[:R * C * eb])


def test_unpad_equals_slicing():
    R, C, NC = 37, 53, 41
    buf = dsgen.matrix_input(R, C, NC, 4).numpy().view(np.uint32).copy()
    orig = buf.copy()
    oracle.unpad(buf, R, C, NC, 4)
    assert np.array_equal(buf[:R * NC], orig.reshape(R, C)[:, :NC].reshape(-1))
    assert np.array_equal(buf[R * NC:], orig[R * NC:])


def test_slide_brute_force_and_slicing():
    """Every n <= 9, shift <= n, eb in {4, 8, 16}: numpy slicing closed form
    (out[:n-shift] == in[shift:n]), untouched tail, buffer bytes past n."""
    for eb in (4, 8, 16):
        w = eb // 4
        for n in range(0, 10):
            for shift in range(0, n + 1):
                buf = (np.arange(n * w + 3, dtype=np.uint32) * 2654435761) & 0xFFFFFFFF
                buf = buf.astype(np.uint32)
                orig = buf.copy()
                oracle.slide(buf, n, shift, eb)
                assert np.array_equal(buf[:(n - shift) * w], orig[shift * w:n * w]), (n, shift, eb)
                assert np.array_equal(buf[(n - shift) * w:], orig[(n - shift) * w:])


def test_slide_equals_unpad_of_two_rows():
    """unpad(R=2, C, NC) moves row 1's first NC elements [C, C+NC) back by
    C-NC to [NC, 2NC); a slide of the sub-buffer starting at element NC, with
    n = C and shift = C-NC, makes the same move (cross-check of two oracle
    functions written independently: memmove per row vs. element loop)."""
    C, NC = 57, 40
    a = dsgen.matrix_input(2, C, C, 4).numpy().view(np.uint32).copy()
    b = a.copy()
    oracle.unpad(a, 2, C, NC, 4)
    sub = b[NC:2 * C].copy()          # elements NC .. 2C-1
    oracle.slide(sub, C, C - NC, 4)  # sub[C-NC, C) -> sub[0, NC)
    b[NC:2 * C] = sub
    assert np.array_equal(a[:2 * NC], b[:2 * NC])


def test_slide_invalid_args():
    buf = np.zeros(8, dtype=np.uint32)
    with pytest.raises(ValueError):
        oracle.slide(buf, 4, 5, 4)
    with pytest.raises(ValueError):
        oracle.slide(buf, 4, 1, 0)


def test_pad_default_fill_zero_and_row0_fixed():
    R, C, NC = 9, 10, 13
    buf = dsgen.matrix_input(R, C, NC, 4).numpy().view(np.uint32).copy()
    oracle.pad(buf, R, C, NC, 4)
    m = buf.reshape(R, NC)
    assert (m[:, C:] == 0).all()
    assert list(m[0, :C]) == list(range(C))       # row 0 is not moved
    for i in range(R):                            # row i moved by (NC-C)*i
        assert m[i, 0] == i * C


def test_pad_f32_c2_shape_sampled():
    """C2 shape (4000 x 3990 -> 4000) on f32 index values: every data cell
    equals (float) of its source index, every fill cell is 0."""
    R, C, NC = 4000, 3990, 4000
    buf = dsgen.matrix_input(R, C, NC, 4, kind="f32").numpy().view(np.uint32).copy()
    oracle.pad(buf, R, C, NC, 4)
    m = buf.view(np.float32).reshape(R, NC)
    rows = np.arange(R)[:, None]
    cols = np.arange(C)[None, :]
    assert np.array_equal(m[:, :C], (rows * C + cols).astype(np.float32))
    assert (buf.reshape(R, NC)[:, C:] == 0).all()
    oracle.unpad(buf, R, NC, C, 4)
    assert np.array_equal(buf[:R * C].view(np.float32), np.arange(R * C, dtype=np.float32))


def test_pad_invalid_args():
    buf = np.zeros(16, dtype=np.uint32)
    with pytest.raises(ValueError):
        oracle.pad(buf, 2, 4, 3, 4)
    with pytest.raises(ValueError):
        oracle.unpad(buf, 2, 3, 4, 4)


# -------------------------------------------------------------------- golden
@pytest.mark.parametrize("case", all_cases(), ids=lambda c: c["name"])
def test_golden_worked_examples(case):
    a = case["input"].copy()
    op = case["op"]
    if op == "compact":
        m = oracle.compact(a, case["remove_value"])
    elif op == "select":
        m = oracle.select(a, case["predicate"], case["param"])
    elif op == "unique":
        m = oracle.unique(a)
    elif op == "pad":
        eb = case["elem_bytes"]
        oracle.pad(a, case["rows"], case["cols"], case["new_cols"], eb,
                   int(case["fill"]).to_bytes(eb, "little"))
        m = None
    elif op == "unpad":
        oracle.unpad(a, case["rows"], case["cols"], case["new_cols"], case["elem_bytes"])
        m = None
    else:
        raise AssertionError(op)
    if m is not None:
        assert m == case["out_n"]
        assert np.array_equal(a[:m], case["output"])
    assert np.array_equal(a, case["buffer_after"])


# ------------------------------------------------------ 8-byte elements
def _rand64(n, seed, alphabet=None):
    rng = np.random.default_rng(seed)
    if alphabet is not None:
        return rng.choice(np.array(alphabet, dtype=np.uint64), size=n).astype(np.uint64)
    return rng.integers(0, 2**64, size=n, dtype=np.uint64)


def test_compact64_brute_force_and_numpy_mask():
    """All keep/remove patterns up to n = 10 (value 0 vs nonzero), then numpy
    boolean masking on random data; the high word alone must decide too."""
    for n in range(0, 11):
        for mask in range(1 << n):
            a = np.array([(i + 1) if (mask >> i) & 1 else 0 for i in range(n)], dtype=np.uint64)
            exp = a[a != 0].copy()
            m = oracle.compact64(a, 0)
            assert m == exp.size and np.array_equal(a[:m], exp)
    v = np.uint64(0xDEADBEEF00000001)
    a = np.array([v, 1, 0xDEADBEEF00000000, v, 0x00000001DEADBEEF], dtype=np.uint64)
    exp = a[a != v].copy()
    m = oracle.compact64(a, int(v))
    assert m == 3 and np.array_equal(a[:m], exp)
    a = _rand64(50_000, 3, alphabet=[5, 7, 1 << 40, (1 << 40) + 5])
    orig = a.copy()
    m = oracle.compact64(a, 1 << 40)
    exp = orig[orig != np.uint64(1 << 40)]
    assert m == exp.size and np.array_equal(a[:m], exp) and np.array_equal(a[m:], orig[m:])


@pytest.mark.parametrize("pred", range(oracle.PRED_COUNT))
def test_select64_equals_numpy(pred):
    rng = np.random.default_rng(10 + pred)
    if pred in (3, 4):  # doubles, with NaN / -0.0 / inf patterns
        d = rng.normal(size=20_000)
        d[::97] = np.nan
        d[::89] = -0.0
        d[::83] = np.inf
        a = d.view(np.uint64).copy()
        param = np.array([0.25]).view(np.uint64)[0]
        dd, pd = a.view(np.float64), np.array([0.25])[0]
        keep = (dd > pd) if pred == 3 else ~(dd > pd)
    else:
        a = rng.integers(-2**62, 2**62, size=20_000, dtype=np.int64).view(np.uint64).copy()
        a[::7] = 0
        param = np.uint64(12345)
        s = a.view(np.int64)
        keep = {0: a != 0, 1: s > 12345, 2: ~(s > 12345), 5: (a & np.uint64(1)) == 0,
                6: (a & np.uint64(1)) != 0}[pred]
    exp = a[keep].copy()
    m = oracle.select64(a, pred, int(param))
    assert m == exp.size and np.array_equal(a[:m], exp)


def test_unique64_brute_force_and_numpy():
    """Every sequence of length <= 7 over a 2-letter alphabet that differs only
    in the high word, then the numpy consecutive-difference mask."""
    letters = [np.uint64(3), np.uint64(3 + (1 << 32))]
    for n in range(0, 8):
        for bits in itertools.product([0, 1], repeat=n):
            a = np.array([letters[b] for b in bits], dtype=np.uint64)
            exp = [a[i] for i in range(n) if i == 0 or a[i] != a[i - 1]]
            m = oracle.unique64(a)
            assert m == len(exp) and list(a[:m]) == exp
    a = _rand64(100_000, 4, alphabet=[1, 2, 2**63])
    orig = a.copy()
    keep = np.concatenate([[True], orig[1:] != orig[:-1]])
    m = oracle.unique64(a)
    assert m == int(keep.sum()) and np.array_equal(a[:m], orig[keep])
