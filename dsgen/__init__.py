"""Seeded synthetic inputs for the Data Sliding workloads.

This module is shared by the tests, bench.py and smoke() to build the SAME
input for both sides of a parity check.  It holds none of the method's
arithmetic (no compaction, selection, run detection, padding or offsets):
only a counter-based hash and the value recipes of SURVEY.md section 8(d).

Counter-based generator (works identically on CPU and CUDA tensors):
    h(i) = splitmix64(seed XOR (i * 0x9E3779B97F4A7C15))      (mod 2**64)
    keep_i = (h(i) >> 32) < floor(f * 2**32)                   (f = kept fraction)
int64 tensor arithmetic wraps modulo 2**64 on both devices; logical right
shifts are emulated with a mask.  tests/test_gen.py pins this against a
pure-Python big-integer splitmix64.
"""
from __future__ import annotations

import math

import torch

GOLDEN = 0x9E3779B97F4A7C15
_M1 = 0xBF58476D1CE4E5B9
_M2 = 0x94D049BB133111EB
CHUNK = 1 << 25
SENTINEL = 0xDEADBEEF
SEED_BASE = 0xD5201500


def _s64(x: int) -> int:
    """Python int -> the int64 with the same low 64 bits."""
    x &= (1 << 64) - 1
    return x - (1 << 64) if x >= (1 << 63) else x


def _shr(z: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (z >> k) & ((1 << (64 - k)) - 1)


def splitmix64(z: torch.Tensor) -> torch.Tensor:
    z = z + _s64(GOLDEN)
    z = (z ^ _shr(z, 30)) * _s64(_M1)
    z = (z ^ _shr(z, 27)) * _s64(_M2)
    return z ^ _shr(z, 31)


def hash_range(seed: int, start: int, count: int, device="cpu") -> torch.Tensor:
    """h(i) for i in [start, start+count), as int64 bit patterns."""
    i = torch.arange(start, start + count, dtype=torch.int64, device=device)
    return splitmix64((i * _s64(GOLDEN)) ^ _s64(seed))


def keep_threshold(f: float) -> int:
    """floor(f * 2**32): keep_i iff (h >> 32) < this (f=1 keeps all)."""
    if not 0.0 <= f <= 1.0:
        raise ValueError("fraction must be in [0, 1]")
    return int(math.floor(f * (1 << 32)))


def _hi32(h: torch.Tensor) -> torch.Tensor:
    return _shr(h, 32)


def _lo32(h: torch.Tensor) -> torch.Tensor:
    return h & 0xFFFFFFFF


def _as_i32(v64: torch.Tensor) -> torch.Tensor:
    """int64 holding a value in [0, 2**32) -> int32 with the same low 32 bits."""
    return torch.where(v64 >= (1 << 31), v64 - (1 << 32), v64).to(torch.int32)


def _fill_chunks(n: int, device, body) -> torch.Tensor:
    out = torch.empty(n, dtype=torch.int32, device=device)
    for s in range(0, n, CHUNK):
        c = min(CHUNK, n - s)
        out[s:s + c] = body(s, c)
    return out


def compact_input(n: int, f: float, seed: int, remove_value: int = 0,
                  kind: str = "u32", device="cpu") -> torch.Tensor:
    """Words to compact (C1/C4/C5).  Kept words never equal remove_value.

    kind="u32": kept a[i] = low32(h(i)) | 1 (remove_value must be even);
    kind="f32": kept a[i] = bits of (float)(1 + (low32(h(i)) >> 9))  (exact,
                positive, never 0 / -0 / NaN); remove_value = bits of 0.0f.
    """
    thr = keep_threshold(f)
    rv = int(remove_value) & 0xFFFFFFFF
    if kind == "u32" and rv & 1:
        raise ValueError("u32 recipe needs an even remove_value")
    rv32 = rv - (1 << 32) if rv >= (1 << 31) else rv

    def body(s, c):
        h = hash_range(seed, s, c, device)
        keep = _hi32(h) < thr
        if kind == "u32":
            val = _as_i32(_lo32(h) | 1)
        elif kind == "f32":
            val = (1 + _shr(_lo32(h), 9)).to(torch.float32).view(torch.int32)
        else:
            raise ValueError(kind)
        return torch.where(keep, val, torch.full_like(val, rv32))
    return _fill_chunks(n, device, body)


def select_input(n: int, seed: int, device="cpu") -> torch.Tensor:
    """C3 select: x_i = (int32)(low32(h(i)) >> 1), uniform in [0, 2**31)."""
    return _fill_chunks(n, device,
                        lambda s, c: (_lo32(hash_range(seed, s, c, device)) >> 1).to(torch.int32))


def select_threshold(f: float) -> int:
    """t with P(x > t) = f for the select_input distribution (t in [-1, 2**31-1])."""
    if not 0.0 <= f <= 1.0:
        raise ValueError("fraction must be in [0, 1]")
    return (1 << 31) - 1 - int(math.floor(f * (1 << 31)))


def unique_runs_input(n: int, f: float, seed: int, device="cpu") -> torch.Tensor:
    """C3 unique, closed-form variant: a[0] = 0, a[i] = a[i-1] + keep_i.

    Run ids increase by 1 with probability f, so unique keeps a[i] iff i == 0
    or keep_i, and its output is 0, 1, ..., out_n - 1.
    """
    thr = keep_threshold(f)
    out = torch.empty(n, dtype=torch.int32, device=device)
    carry = 0
    for s in range(0, n, CHUNK):
        c = min(CHUNK, n - s)
        inc = (_hi32(hash_range(seed, s, c, device)) < thr).to(torch.int64)
        if s == 0:
            inc[0] = 0
        run = torch.cumsum(inc, 0) + carry
        carry = int(run[-1].item())
        out[s:s + c] = _as_i32(run & 0xFFFFFFFF)
    return out


def unique_hashed_input(n: int, f: float, seed: int, device="cpu") -> torch.Tensor:
    """C3 unique, random-value variant: each run carries low32(splitmix64(run_id ^ seed))."""
    runs = unique_runs_input(n, f, seed, device).to(torch.int64) & 0xFFFFFFFF
    out = torch.empty(n, dtype=torch.int32, device=device)
    for s in range(0, n, CHUNK):
        c = min(CHUNK, n - s)
        out[s:s + c] = _as_i32(_lo32(splitmix64(runs[s:s + c] ^ _s64(seed))))
    return out


def random_words(n: int, seed: int, device="cpu", bits: int = 32) -> torch.Tensor:
    """Uniform words with `bits` random low bits (small alphabets for tests)."""
    mask = (1 << bits) - 1
    return _fill_chunks(n, device, lambda s, c: _as_i32(_lo32(hash_range(seed, s, c, device)) & mask))


def matrix_input(rows: int, cols: int, new_cols: int, elem_bytes: int,
                 kind: str = "index", device="cpu") -> torch.Tensor:
    """Pad/unpad buffer as int32 words, capacity max(cols, new_cols) per row.

    Words [0, rows*cols*eb/4) hold their own word index p (kind="index") or
    the bits of (float)p (kind="f32", exact for p < 2**24); the extra space
    beyond the matrix holds SENTINEL (C2 recipe).
    """
    if elem_bytes % 4:
        raise ValueError("matrix_input builds 4-byte-word buffers")
    w = elem_bytes // 4
    used = rows * cols * w
    cap = rows * max(cols, new_cols) * w
    buf = torch.full((cap,), SENTINEL - (1 << 32), dtype=torch.int32, device=device)
    if kind == "index":
        buf[:used] = torch.arange(used, dtype=torch.int64, device=device).to(torch.int32)
    elif kind == "f32":
        if used > (1 << 24):
            raise ValueError("f32 index recipe is exact only below 2**24 words")
        buf[:used] = torch.arange(used, dtype=torch.float32, device=device).view(torch.int32)
    else:
        raise ValueError(kind)
    return buf


def seed_for(config_index: int, sweep_index: int = 0) -> int:
    """Fixed per-config seeds."""
    return SEED_BASE + 16 * config_index + sweep_index
