"""Pins for the shared input generator (dsgen): int64-tensor splitmix64 vs
pure-Python big-integer arithmetic, and the recipes' structural promises."""
import numpy as np
import pytest
import torch

import dsgen

MASK = (1 << 64) - 1


def py_splitmix64(z):
    z = (z + 0x9E3779B97F4A7C15) & MASK
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK
    return z ^ (z >> 31)


def py_h(seed, i):
    return py_splitmix64((seed ^ ((i * 0x9E3779B97F4A7C15) & MASK)) & MASK)


def test_splitmix64_known_value():
    # Reference value of the public splitmix64 sequence seeded with 0:
    # the first output of Vigna's splitmix64 (state 0) is 0xE220A8397B1DCDAF.
    assert py_splitmix64(0) == 0xE220A8397B1DCDAF
    t = dsgen.splitmix64(torch.tensor([0], dtype=torch.int64))
    assert int(t[0]) & MASK == 0xE220A8397B1DCDAF


@pytest.mark.parametrize("seed", [0, 1, dsgen.seed_for(3, 7), 0xFFFFFFFFFFFFFFFF])
def test_hash_matches_python(seed):
    h = dsgen.hash_range(seed, 1000, 257)
    for k in range(257):
        assert int(h[k]) & MASK == py_h(seed, 1000 + k)


def test_compact_input_recipe():
    n, f, seed = 50000, 0.5, dsgen.seed_for(0)
    a = dsgen.compact_input(n, f, seed).numpy().view(np.uint32)
    thr = dsgen.keep_threshold(f)
    for i in range(0, n, 997):
        h = py_h(seed, i)
        keep = (h >> 32) < thr
        assert a[i] == ((h & 0xFFFFFFFF) | 1 if keep else 0)
    frac = np.count_nonzero(a) / n
    assert abs(frac - 0.5) < 0.02


def test_compact_input_f32_never_zero_nan():
    a = dsgen.compact_input(20000, 0.9, 5, kind="f32")
    x = a.view(torch.float32)
    kept = x[a != 0]
    assert torch.isfinite(kept).all() and (kept >= 1).all()
    assert (kept == torch.floor(kept)).all()


@pytest.mark.parametrize("f", [0.0, 1.0])
def test_extreme_fractions(f):
    a = dsgen.compact_input(4096, f, 11).numpy()
    assert np.count_nonzero(a) == (0 if f == 0.0 else 4096)


def test_select_threshold_fraction():
    x = dsgen.select_input(100000, 3).numpy()
    assert x.min() >= 0
    for f in (0.0, 0.1, 0.5, 0.9, 1.0):
        t = dsgen.select_threshold(f)
        frac = np.count_nonzero(x > t) / x.size
        assert abs(frac - f) < 0.01
    assert dsgen.select_threshold(0.0) == 2**31 - 1 and dsgen.select_threshold(1.0) == -1


def test_unique_runs_closed_form_structure():
    a = dsgen.unique_runs_input(10000, 0.3, 9).numpy().astype(np.int64)
    assert a[0] == 0
    d = np.diff(a)
    assert set(np.unique(d)).issubset({0, 1})


def test_matrix_input_layout():
    b = dsgen.matrix_input(3, 5, 7, 4).numpy().view(np.uint32)
    assert b.size == 21
    assert list(b[:15]) == list(range(15))
    assert (b[15:] == dsgen.SENTINEL).all()
    b8 = dsgen.matrix_input(2, 3, 2, 8).numpy().view(np.uint32)
    assert b8.size == 12 and list(b8) == list(range(12))
