"""Thin ctypes binding of libds (include/ds.h) -- argument marshalling only.

Every function has the name of the C entry point it calls.  Buffers may be
given as CUDA torch tensors (their ``data_ptr()`` is passed) or as raw
integer device pointers.  Nothing here computes: every step of the path
runs in libds' CUDA kernels.  If libds.so is missing the import of this
module fails loudly; there is no fallback.
"""
from __future__ import annotations

import ctypes
import os

from . import build as _build

DS_SUCCESS, DS_ERROR_INVALID_VALUE, DS_ERROR_UNSUPPORTED, DS_ERROR_OUT_OF_MEMORY, DS_ERROR_CUDA = range(5)
(DS_PRED_NONZERO, DS_PRED_I32_GT, DS_PRED_I32_NOT_GT, DS_PRED_F32_GT, DS_PRED_F32_NOT_GT,
 DS_PRED_I32_EVEN, DS_PRED_I32_ODD) = range(7)
DS_PRED_COUNT = 7

# Every entry point declared in include/ds.h: name -> (restype, argtypes).
_sz, _u32, _u64, _i = ctypes.c_size_t, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
_vp = ctypes.c_void_p
_psz = ctypes.POINTER(ctypes.c_size_t)
_pvp = ctypes.POINTER(ctypes.c_void_p)


class DsPublish(ctypes.Structure):
    """ds_publish (include/ds.h): where a shard's DS kernel publishes its count."""
    _fields_ = [("d_boards", ctypes.c_void_p), ("world", ctypes.c_size_t), ("rank", ctypes.c_size_t),
                ("tag", ctypes.c_uint64)]


_ppub = ctypes.POINTER(DsPublish)
SIGNATURES = {
    "ds_pad": (_i, [_vp, _sz, _sz, _sz, _sz]),
    "ds_unpad": (_i, [_vp, _sz, _sz, _sz, _sz]),
    "ds_pad_ex": (_i, [_vp, _sz, _sz, _sz, _sz, _vp, _vp]),
    "ds_unpad_ex": (_i, [_vp, _sz, _sz, _sz, _sz, _vp]),
    "ds_slide": (_i, [_vp, _sz, _sz, _sz]),
    "ds_slide_ex": (_i, [_vp, _sz, _sz, _sz, _vp]),
    "ds_compact": (_i, [_vp, _sz, _u32, _psz]),
    "ds_select": (_i, [_vp, _sz, _i, _psz]),
    "ds_unique": (_i, [_vp, _sz, _psz]),
    "ds_compact_ex": (_i, [_vp, _sz, _u32, _vp, _vp]),
    "ds_select_ex": (_i, [_vp, _sz, _i, _u32, _vp, _vp]),
    "ds_unique_ex": (_i, [_vp, _sz, _vp, _sz, _vp, _vp]),
    "ds_compact64": (_i, [_vp, _sz, _u64, _psz]),
    "ds_select64": (_i, [_vp, _sz, _i, _psz]),
    "ds_unique64": (_i, [_vp, _sz, _psz]),
    "ds_compact64_ex": (_i, [_vp, _sz, _u64, _vp, _vp]),
    "ds_select64_ex": (_i, [_vp, _sz, _i, _u64, _vp, _vp]),
    "ds_unique64_ex": (_i, [_vp, _sz, _vp, _vp]),
    "ds_partition": (_i, [_vp, _sz, _i, _vp, _psz]),
    "ds_partition_ex": (_i, [_vp, _sz, _i, _u32, _vp, _vp, _vp]),
    "ds_select_copy_ex": (_i, [_vp, _sz, _i, _u32, _vp, _vp, _vp]),
    "ds_partition_copy_ex": (_i, [_vp, _sz, _i, _u32, _vp, _vp, _vp, _vp]),
    "ds_halo_entry": (_i, [_vp, _sz, _vp, _vp]),
    "ds_shard_offsets": (_i, [_vp, _sz, _sz, _vp, _vp]),
    "ds_board_alloc": (_i, [_sz, _pvp]),
    "ds_board_free": (_i, [_vp]),
    "ds_board_ipc_handle": (_i, [_vp, _vp]),
    "ds_board_ipc_open": (_i, [_vp, _pvp]),
    "ds_board_ipc_close": (_i, [_vp]),
    "ds_compact_pub_ex": (_i, [_vp, _sz, _u32, _vp, _ppub, _vp]),
    "ds_select_pub_ex": (_i, [_vp, _sz, _i, _u32, _vp, _ppub, _vp]),
    "ds_unique_pub_ex": (_i, [_vp, _sz, _vp, _sz, _vp, _ppub, _vp]),
    "ds_shard_offsets_board": (_i, [_vp, _sz, _sz, _u64, _vp, _vp, _vp]),
    "ds_status_string": (ctypes.c_char_p, [_i]),
    "ds_last_error": (ctypes.c_char_p, []),
    "ds_release_workspaces": (_i, []),
    "ds_launch_count": (_u64, []),
    "ds_version": (_i, []),
    "ds_tile_size": (_sz, [_i]),
    "ds_debug_set_trace": (_i, [_vp, _sz]),
}


class DSError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str = ""):
        self.status = status
        name = _lib.ds_status_string(status).decode() if _lib is not None else str(status)
        super().__init__(f"{where}: {name}" + (f" ({detail})" if detail else ""))


def _load(path: str | None = None):
    path = path or os.environ.get("LIBDS_PATH") or _build.lib_path()
    if not os.path.exists(path):
        raise ImportError(f"libds not built: {path} is missing "
                          "(run `python -m paper_conf_icpp_gomez_lunacshg15_b200.build`)")
    lib = ctypes.CDLL(path)
    for name, (res, args) in SIGNATURES.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    return lib


_lib = _load()
LIB_PATH = _lib._name


def _addr(x) -> int | None:
    """Device address of a CUDA tensor, a raw int pointer, or None."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        if not x.is_cuda:
            raise ValueError("libds needs device (CUDA) memory")
        if not x.is_contiguous():
            raise ValueError("libds needs a contiguous tensor")
        return x.data_ptr()
    raise TypeError(f"cannot pass {type(x)!r} as a device pointer")


def _stream(s) -> int | None:
    """cudaStream_t handle: torch.cuda.Stream, raw int, or None -> torch's current stream."""
    if s is None:
        import torch
        return torch.cuda.current_stream().cuda_stream or None
    if isinstance(s, int):
        return s or None
    return s.cuda_stream or None


def _check(status: int, where: str) -> None:
    if status != DS_SUCCESS:
        detail = _lib.ds_last_error().decode() if status == DS_ERROR_CUDA else ""
        raise DSError(status, where, detail)


# ---------------------------------------------------------------- regular DS
def ds_pad(ptr, rows: int, cols: int, new_cols: int, elem_bytes: int) -> None:
    _check(_lib.ds_pad(_addr(ptr), rows, cols, new_cols, elem_bytes), "ds_pad")


def ds_unpad(ptr, rows: int, cols: int, new_cols: int, elem_bytes: int) -> None:
    _check(_lib.ds_unpad(_addr(ptr), rows, cols, new_cols, elem_bytes), "ds_unpad")


def ds_pad_ex(ptr, rows: int, cols: int, new_cols: int, elem_bytes: int,
              fill: bytes | None = None, stream=None) -> None:
    fb = None
    if fill is not None:
        if len(fill) != elem_bytes:
            raise ValueError("fill must be elem_bytes long")
        fb = ctypes.create_string_buffer(bytes(fill), elem_bytes)
    _check(_lib.ds_pad_ex(_addr(ptr), rows, cols, new_cols, elem_bytes,
                          ctypes.cast(fb, _vp) if fb is not None else None, _stream(stream)),
           "ds_pad_ex")


def ds_unpad_ex(ptr, rows: int, cols: int, new_cols: int, elem_bytes: int, stream=None) -> None:
    _check(_lib.ds_unpad_ex(_addr(ptr), rows, cols, new_cols, elem_bytes, _stream(stream)),
           "ds_unpad_ex")


def ds_slide(ptr, n: int, shift: int, elem_bytes: int) -> None:
    _check(_lib.ds_slide(_addr(ptr), n, shift, elem_bytes), "ds_slide")


def ds_slide_ex(ptr, n: int, shift: int, elem_bytes: int, stream=None) -> None:
    _check(_lib.ds_slide_ex(_addr(ptr), n, shift, elem_bytes, _stream(stream)), "ds_slide_ex")


# -------------------------------------------------------------- irregular DS
def ds_compact(ptr, n: int, remove_value: int) -> int:
    out = ctypes.c_size_t(0)
    _check(_lib.ds_compact(_addr(ptr), n, remove_value & 0xFFFFFFFF, ctypes.byref(out)), "ds_compact")
    return out.value


def ds_select(ptr, n: int, predicate_id: int) -> int:
    out = ctypes.c_size_t(0)
    _check(_lib.ds_select(_addr(ptr), n, predicate_id, ctypes.byref(out)), "ds_select")
    return out.value


def ds_unique(ptr, n: int) -> int:
    out = ctypes.c_size_t(0)
    _check(_lib.ds_unique(_addr(ptr), n, ctypes.byref(out)), "ds_unique")
    return out.value


def ds_compact_ex(ptr, n: int, remove_value: int, d_out_n=None, stream=None) -> None:
    _check(_lib.ds_compact_ex(_addr(ptr), n, remove_value & 0xFFFFFFFF, _addr(d_out_n),
                              _stream(stream)), "ds_compact_ex")


def ds_select_ex(ptr, n: int, predicate_id: int, param: int = 0, d_out_n=None, stream=None) -> None:
    _check(_lib.ds_select_ex(_addr(ptr), n, predicate_id, param & 0xFFFFFFFF, _addr(d_out_n),
                             _stream(stream)), "ds_select_ex")


def ds_unique_ex(ptr, n: int, d_halo=None, halo_len: int = 0, d_out_n=None, stream=None) -> None:
    _check(_lib.ds_unique_ex(_addr(ptr), n, _addr(d_halo), halo_len, _addr(d_out_n),
                             _stream(stream)), "ds_unique_ex")


# ------------------------------------------------- partition / out-of-place
# ------------------------------------------------------- 8-byte elements
def ds_compact64(ptr, n: int, remove_value: int) -> int:
    out = ctypes.c_size_t(0)
    _check(_lib.ds_compact64(_addr(ptr), n, remove_value & 0xFFFFFFFFFFFFFFFF, ctypes.byref(out)),
           "ds_compact64")
    return out.value


def ds_select64(ptr, n: int, predicate_id: int) -> int:
    out = ctypes.c_size_t(0)
    _check(_lib.ds_select64(_addr(ptr), n, predicate_id, ctypes.byref(out)), "ds_select64")
    return out.value


def ds_unique64(ptr, n: int) -> int:
    out = ctypes.c_size_t(0)
    _check(_lib.ds_unique64(_addr(ptr), n, ctypes.byref(out)), "ds_unique64")
    return out.value


def ds_compact64_ex(ptr, n: int, remove_value: int, d_out_n=None, stream=None) -> None:
    _check(_lib.ds_compact64_ex(_addr(ptr), n, remove_value & 0xFFFFFFFFFFFFFFFF, _addr(d_out_n),
                                _stream(stream)), "ds_compact64_ex")


def ds_select64_ex(ptr, n: int, predicate_id: int, param: int = 0, d_out_n=None, stream=None) -> None:
    _check(_lib.ds_select64_ex(_addr(ptr), n, predicate_id, param & 0xFFFFFFFFFFFFFFFF, _addr(d_out_n),
                               _stream(stream)), "ds_select64_ex")


def ds_unique64_ex(ptr, n: int, d_out_n=None, stream=None) -> None:
    _check(_lib.ds_unique64_ex(_addr(ptr), n, _addr(d_out_n), _stream(stream)), "ds_unique64_ex")


def ds_partition(ptr, n: int, predicate_id: int, aux) -> int:
    out = ctypes.c_size_t(0)
    _check(_lib.ds_partition(_addr(ptr), n, predicate_id, _addr(aux), ctypes.byref(out)), "ds_partition")
    return out.value


def ds_partition_ex(ptr, n: int, predicate_id: int, param: int, aux, d_out_n_true, stream=None) -> None:
    _check(_lib.ds_partition_ex(_addr(ptr), n, predicate_id, param & 0xFFFFFFFF, _addr(aux),
                                _addr(d_out_n_true), _stream(stream)), "ds_partition_ex")


def ds_select_copy_ex(src, n: int, predicate_id: int, param: int, out, d_out_n=None, stream=None) -> None:
    _check(_lib.ds_select_copy_ex(_addr(src), n, predicate_id, param & 0xFFFFFFFF, _addr(out),
                                  _addr(d_out_n), _stream(stream)), "ds_select_copy_ex")


def ds_partition_copy_ex(src, n: int, predicate_id: int, param: int, out_true, out_false,
                         d_out_n_true=None, stream=None) -> None:
    _check(_lib.ds_partition_copy_ex(_addr(src), n, predicate_id, param & 0xFFFFFFFF, _addr(out_true),
                                     _addr(out_false), _addr(d_out_n_true), _stream(stream)),
           "ds_partition_copy_ex")


# ------------------------------------------------------------------ sharding
def ds_halo_entry(ptr, n: int, d_entry, stream=None) -> None:
    _check(_lib.ds_halo_entry(_addr(ptr), n, _addr(d_entry), _stream(stream)), "ds_halo_entry")


def ds_shard_offsets(d_counts, world: int, rank: int, d_result, stream=None) -> None:
    _check(_lib.ds_shard_offsets(_addr(d_counts), world, rank, _addr(d_result), _stream(stream)),
           "ds_shard_offsets")


# ------------------------------------------------------------ count boards
DS_IPC_HANDLE_BYTES = 64


def ds_board_alloc(world: int) -> int:
    p = ctypes.c_void_p()
    _check(_lib.ds_board_alloc(world, ctypes.byref(p)), "ds_board_alloc")
    return int(p.value)


def ds_board_free(d_board: int) -> None:
    _check(_lib.ds_board_free(d_board), "ds_board_free")


def ds_board_ipc_handle(d_board: int) -> bytes:
    buf = ctypes.create_string_buffer(DS_IPC_HANDLE_BYTES)
    _check(_lib.ds_board_ipc_handle(d_board, buf), "ds_board_ipc_handle")
    return buf.raw


def ds_board_ipc_open(handle: bytes) -> int:
    if len(handle) != DS_IPC_HANDLE_BYTES:
        raise ValueError("an IPC handle is 64 bytes")
    p = ctypes.c_void_p()
    _check(_lib.ds_board_ipc_open(ctypes.create_string_buffer(handle, DS_IPC_HANDLE_BYTES), ctypes.byref(p)),
           "ds_board_ipc_open")
    return int(p.value)


def ds_board_ipc_close(d_peer_board: int) -> None:
    _check(_lib.ds_board_ipc_close(d_peer_board), "ds_board_ipc_close")


def _pub(d_boards, world, rank, tag):
    return ctypes.byref(DsPublish(_addr(d_boards), world, rank, tag))


def ds_compact_pub_ex(ptr, n: int, remove_value: int, d_out_n, d_boards, world: int, rank: int, tag: int,
                      stream=None) -> None:
    _check(_lib.ds_compact_pub_ex(_addr(ptr), n, remove_value & 0xFFFFFFFF, _addr(d_out_n),
                                  _pub(d_boards, world, rank, tag), _stream(stream)), "ds_compact_pub_ex")


def ds_select_pub_ex(ptr, n: int, predicate_id: int, param: int, d_out_n, d_boards, world: int, rank: int,
                     tag: int, stream=None) -> None:
    _check(_lib.ds_select_pub_ex(_addr(ptr), n, predicate_id, param & 0xFFFFFFFF, _addr(d_out_n),
                                 _pub(d_boards, world, rank, tag), _stream(stream)), "ds_select_pub_ex")


def ds_unique_pub_ex(ptr, n: int, d_halo, halo_len: int, d_out_n, d_boards, world: int, rank: int, tag: int,
                     stream=None) -> None:
    _check(_lib.ds_unique_pub_ex(_addr(ptr), n, _addr(d_halo), halo_len, _addr(d_out_n),
                                 _pub(d_boards, world, rank, tag), _stream(stream)), "ds_unique_pub_ex")


def ds_shard_offsets_board(d_board: int, world: int, rank: int, tag: int, d_counts, d_result,
                           stream=None) -> None:
    _check(_lib.ds_shard_offsets_board(d_board, world, rank, tag, _addr(d_counts), _addr(d_result),
                                       _stream(stream)), "ds_shard_offsets_board")


# ------------------------------------------------------------------ utilities
def ds_status_string(status: int) -> str:
    return _lib.ds_status_string(status).decode()


def ds_last_error() -> str:
    return _lib.ds_last_error().decode()


def ds_release_workspaces() -> None:
    _check(_lib.ds_release_workspaces(), "ds_release_workspaces")


def ds_launch_count() -> int:
    return int(_lib.ds_launch_count())


def ds_version() -> int:
    return int(_lib.ds_version())


DS_KERNEL_IRREGULAR, DS_KERNEL_REGULAR, DS_KERNEL_REGULAR_BYTES = 0, 1, 2


def ds_tile_size(kernel: int) -> int:
    return int(_lib.ds_tile_size(kernel))


def ds_debug_set_trace(d_trace, capacity_tiles: int) -> None:
    _check(_lib.ds_debug_set_trace(_addr(d_trace), capacity_tiles), "ds_debug_set_trace")


def raw_status(name: str, *args) -> int:
    """Call an entry point and return its ds_status without raising (tests)."""
    return int(getattr(_lib, name)(*args))
