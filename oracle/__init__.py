"""CPU oracle for the in-place Data Sliding primitives -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and the ``cpu_baseline`` /
``--impl reference`` legs of ``bench.py`` may import this package.  The
product (``paper_conf_icpp_gomez_lunacshg15_b200``) never imports it and
shares no code with it.

The arithmetic lives in ``ds_oracle.c`` (plain sequential C, each function
citing the PAPER.md passage it follows).  This module only compiles it with
gcc and marshals numpy arrays through ctypes; every call works IN PLACE on
the array it is given, exactly like the primitive it defines.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ds_oracle.c")
_LIB_PATH = os.path.join(_HERE, "libds_oracle.so")

# Numeric predicate ids (the documented ds_select ABI, re-stated here).
PRED_NONZERO, PRED_I32_GT, PRED_I32_NOT_GT, PRED_F32_GT, PRED_F32_NOT_GT, \
    PRED_I32_EVEN, PRED_I32_ODD = range(7)
PRED_COUNT = 7

_lib = None


def build(force: bool = False) -> str:
    """Compile ds_oracle.c into oracle/libds_oracle.so (gcc -O2, 1 thread)."""
    if force or not os.path.exists(_LIB_PATH) or \
            os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared",
                               "-Wall", "-Wextra", "-o", _LIB_PATH, _SRC])
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        sz, u32, i32, vp = ctypes.c_size_t, ctypes.c_uint32, ctypes.c_int, ctypes.c_void_p
        L.oracle_predicate.argtypes = [i32, u32, u32]
        L.oracle_predicate.restype = i32
        L.oracle_compact.argtypes = [vp, sz, u32]
        L.oracle_compact.restype = sz
        L.oracle_select.argtypes = [vp, sz, i32, u32]
        L.oracle_select.restype = sz
        L.oracle_unique.argtypes = [vp, sz]
        L.oracle_unique.restype = sz
        L.oracle_unique_prev.argtypes = [vp, sz, i32, u32]
        L.oracle_unique_prev.restype = sz
        L.oracle_partition.argtypes = [vp, sz, i32, u32, vp]
        L.oracle_partition.restype = sz
        L.oracle_select_copy.argtypes = [vp, sz, i32, u32, vp]
        L.oracle_select_copy.restype = sz
        L.oracle_pad.argtypes = [vp, sz, sz, sz, sz, vp]
        L.oracle_pad.restype = i32
        L.oracle_unpad.argtypes = [vp, sz, sz, sz, sz]
        L.oracle_unpad.restype = i32
        u64 = ctypes.c_uint64
        L.oracle_predicate64.argtypes = [i32, u64, u64]
        L.oracle_predicate64.restype = i32
        L.oracle_compact64.argtypes = [vp, sz, u64]
        L.oracle_compact64.restype = sz
        L.oracle_select64.argtypes = [vp, sz, i32, u64]
        L.oracle_select64.restype = sz
        L.oracle_unique64.argtypes = [vp, sz]
        L.oracle_unique64.restype = sz
        L.oracle_slide.argtypes = [vp, sz, sz, sz]
        L.oracle_slide.restype = i32
        _lib = L
    return _lib


def _words(a: np.ndarray) -> np.ndarray:
    if not isinstance(a, np.ndarray) or a.dtype.itemsize != 4 or not a.flags.c_contiguous \
            or not a.flags.writeable:
        raise TypeError("oracle needs a writeable C-contiguous 4-byte numpy array")
    return a


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def predicate(pred: int, w: int, param: int = 0) -> int:
    return lib().oracle_predicate(int(pred), int(w) & 0xFFFFFFFF, int(param) & 0xFFFFFFFF)


def compact(a: np.ndarray, remove_value: int) -> int:
    """In place; returns out_n."""
    a = _words(a)
    return int(lib().oracle_compact(_ptr(a), a.size, int(remove_value) & 0xFFFFFFFF))


def select(a: np.ndarray, pred: int, param: int = 0) -> int:
    """In place; keeps predicate-true words; returns out_n."""
    a = _words(a)
    r = lib().oracle_select(_ptr(a), a.size, int(pred), int(param) & 0xFFFFFFFF)
    if r == ctypes.c_size_t(-1).value:
        raise ValueError(f"unknown predicate id {pred}")
    return int(r)


def unique(a: np.ndarray, prev: int | None = None) -> int:
    """In place; keeps the first of each run of equal words."""
    a = _words(a)
    if prev is None:
        return int(lib().oracle_unique(_ptr(a), a.size))
    return int(lib().oracle_unique_prev(_ptr(a), a.size, 1, int(prev) & 0xFFFFFFFF))


def partition(a: np.ndarray, pred: int, param: int = 0) -> int:
    """In place; true words first, then false words, both stable."""
    a = _words(a)
    aux = np.empty_like(a)
    r = lib().oracle_partition(_ptr(a), a.size, int(pred), int(param) & 0xFFFFFFFF, _ptr(aux))
    if r == ctypes.c_size_t(-1).value:
        raise ValueError(f"unknown predicate id {pred}")
    return int(r)


def select_copy(a: np.ndarray, pred: int, param: int = 0) -> np.ndarray:
    """Out of place (P:242 Copy_if): returns the predicate-true words."""
    a = np.ascontiguousarray(a)
    out = np.empty(a.size, dtype=np.uint32)
    r = lib().oracle_select_copy(_ptr(a), a.size, int(pred), int(param) & 0xFFFFFFFF, _ptr(out))
    if r == ctypes.c_size_t(-1).value:
        raise ValueError(f"unknown predicate id {pred}")
    return out[:r].copy()


def _bytes_view(buf: np.ndarray) -> np.ndarray:
    if not isinstance(buf, np.ndarray) or not buf.flags.c_contiguous or not buf.flags.writeable:
        raise TypeError("oracle needs a writeable C-contiguous numpy buffer")
    return buf


def pad(buf: np.ndarray, rows: int, cols: int, new_cols: int, elem_bytes: int,
        fill: bytes | None = None) -> None:
    """In place on the raw bytes of ``buf`` (capacity >= rows*new_cols*eb)."""
    buf = _bytes_view(buf)
    if rows * new_cols * elem_bytes > buf.nbytes:
        raise ValueError("buffer too small for the padded matrix")
    fb = None
    if fill is not None:
        if len(fill) != elem_bytes:
            raise ValueError("fill must be elem_bytes long")
        fb = ctypes.create_string_buffer(bytes(fill), elem_bytes)
    rc = lib().oracle_pad(_ptr(buf), rows, cols, new_cols, elem_bytes,
                          ctypes.cast(fb, ctypes.c_void_p) if fb is not None else None)
    if rc != 0:
        raise ValueError("oracle_pad: new_cols < cols or elem_bytes == 0")


def unpad(buf: np.ndarray, rows: int, cols: int, new_cols: int, elem_bytes: int) -> None:
    """In place on the raw bytes of ``buf``."""
    buf = _bytes_view(buf)
    if rows * cols * elem_bytes > buf.nbytes:
        raise ValueError("buffer too small for the matrix")
    rc = lib().oracle_unpad(_ptr(buf), rows, cols, new_cols, elem_bytes)
    if rc != 0:
        raise ValueError("oracle_unpad: new_cols > cols or elem_bytes == 0")


def slide(buf: np.ndarray, n: int, shift: int, elem_bytes: int) -> None:
    """In place on the raw bytes of ``buf``: elements [shift, n) -> [0, n - shift)."""
    buf = _bytes_view(buf)
    if n * elem_bytes > buf.nbytes:
        raise ValueError("buffer too small")
    rc = lib().oracle_slide(_ptr(buf), n, shift, elem_bytes)
    if rc != 0:
        raise ValueError("oracle_slide: shift > n or elem_bytes == 0")


def _words64(a: np.ndarray) -> np.ndarray:
    if a.dtype != np.uint64 or not a.flags.c_contiguous or not a.flags.writeable:
        raise TypeError("oracle needs a writeable C-contiguous uint64 array")
    return a


def compact64(a: np.ndarray, remove_value: int) -> int:
    """In place on uint64 ``a`` (8-byte elements); returns the kept count."""
    a = _words64(a)
    return int(lib().oracle_compact64(_ptr(a), a.size, remove_value & 0xFFFFFFFFFFFFFFFF))


def select64(a: np.ndarray, pred: int, param: int = 0) -> int:
    a = _words64(a)
    r = lib().oracle_select64(_ptr(a), a.size, pred, param & 0xFFFFFFFFFFFFFFFF)
    if r == ctypes.c_size_t(-1).value:
        raise ValueError("unknown predicate")
    return int(r)


def unique64(a: np.ndarray) -> int:
    a = _words64(a)
    return int(lib().oracle_unique64(_ptr(a), a.size))


def predicate64(pred: int, e: int, param: int = 0) -> int:
    return int(lib().oracle_predicate64(pred, e & 0xFFFFFFFFFFFFFFFF, param & 0xFFFFFFFFFFFFFFFF))
