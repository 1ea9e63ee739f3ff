"""C-ABI boundary checks that need no GPU (T1, host side):
the library loads, exports every entry point include/ds.h declares, and
rejects invalid arguments BEFORE touching the device (so these calls never
reach CUDA and run on a CPU-only box)."""
import ctypes
import os
import re

import pytest

from paper_conf_icpp_gomez_lunacshg15_b200 import build, libds

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ds.h")

INV, UNS = libds.DS_ERROR_INVALID_VALUE, libds.DS_ERROR_UNSUPPORTED
BAD = 0x7F0000001002      # fake device address, 4-byte misaligned
FAKE = 0x7F0000001000     # fake device address, aligned (never dereferenced below)


def declared_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(ds_[a-z_0-9]+)\s*\(", text)))


def test_header_declares_expected_api():
    names = declared_functions()
    for must in ("ds_pad", "ds_unpad", "ds_compact", "ds_select", "ds_unique"):
        assert must in names


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(build.lib_path())
    for name in declared_functions():
        assert hasattr(lib, name), name
    assert set(declared_functions()) == set(libds.SIGNATURES)


def test_library_is_sm100a():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", build.lib_path()],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_status_strings_and_version():
    assert libds.ds_status_string(0) == "DS_SUCCESS"
    assert libds.ds_status_string(INV) == "DS_ERROR_INVALID_VALUE"
    assert libds.ds_status_string(4) == "DS_ERROR_CUDA"
    assert libds.ds_version() >= 200


def test_tile_sizes():
    """The tile sizes the GPU tile-edge sweeps are keyed to (ds_tile_size)."""
    assert libds.ds_tile_size(libds.DS_KERNEL_IRREGULAR) == 8192
    assert libds.ds_tile_size(libds.DS_KERNEL_REGULAR) == 8192
    assert libds.ds_tile_size(libds.DS_KERNEL_REGULAR_BYTES) == 32768
    assert libds.ds_tile_size(7) == 0


def st(name, *args):
    return libds.raw_status(name, *args)


def out_sz():
    return ctypes.byref(ctypes.c_size_t(12345))


def test_irregular_validation_before_device():
    # NULL pointer with n > 0
    assert st("ds_compact", None, 10, 0, out_sz()) == INV
    assert st("ds_compact_ex", None, 10, 0, None, None) == INV
    # misaligned pointer
    assert st("ds_compact", BAD, 10, 0, out_sz()) == INV
    assert st("ds_select_ex", BAD, 10, 1, 0, None, None) == INV
    assert st("ds_unique_ex", BAD, 10, None, 0, None, None) == INV
    # NULL out_n on blocking forms
    assert st("ds_compact", FAKE, 10, 0, None) == INV
    assert st("ds_select", FAKE, 10, 0, None) == INV
    assert st("ds_unique", FAKE, 10, None) == INV
    # unknown predicate ids
    for pid in (-1, 7, 1000):
        assert st("ds_select", FAKE, 10, pid, out_sz()) == INV
        assert st("ds_select_ex", FAKE, 10, pid, 0, None, None) == INV
    # halo length without halo array; misaligned d_out_n
    assert st("ds_unique_ex", FAKE, 10, None, 3, None, None) == INV
    assert st("ds_compact_ex", FAKE, 10, 0, FAKE + 4, None) == INV
    # too many words for the 36-bit status count
    assert st("ds_compact_ex", FAKE, 1 << 36, 0, None, None) == UNS


def test_irregular_empty_input_needs_no_device():
    n = ctypes.c_size_t(99)
    assert st("ds_compact", None, 0, 0, ctypes.byref(n)) == 0 and n.value == 0
    n = ctypes.c_size_t(99)
    assert st("ds_unique", FAKE, 0, ctypes.byref(n)) == 0 and n.value == 0
    n = ctypes.c_size_t(99)
    assert st("ds_select", FAKE, 0, 3, ctypes.byref(n)) == 0 and n.value == 0


def test_regular_validation_before_device():
    assert st("ds_pad", FAKE, 4, 5, 4, 4) == INV          # new_cols < cols
    assert st("ds_unpad", FAKE, 4, 4, 5, 4) == INV        # new_cols > cols
    assert st("ds_pad", FAKE, 4, 4, 5, 3) == INV          # bad elem_bytes
    assert st("ds_pad", FAKE, 4, 4, 5, 0) == INV
    assert st("ds_pad", FAKE, 4, 5, 4, 2) == INV          # 2-byte elements: new_cols < cols
    assert st("ds_unpad", FAKE, 4, 4, 5, 1) == INV        # 1-byte elements: new_cols > cols
    assert st("ds_pad", FAKE + 1, 4, 4, 5, 2) == INV      # 2-byte elements, odd address
    assert st("ds_pad", None, 4, 4, 5, 1) == INV
    assert st("ds_pad", FAKE, 2, 1, 1 << 31, 1) == UNS    # row longer than 2^30 words
    assert st("ds_pad_ex", FAKE + 3, 0, 5, 9, 1, None, None) == 0   # rows == 0: nothing to do
    assert st("ds_pad", None, 4, 4, 5, 4) == INV          # NULL with data
    assert st("ds_pad", BAD, 4, 4, 5, 4) == INV           # misaligned
    assert st("ds_pad", FAKE, 1 << 40, 1 << 30, 1 << 31, 8) == INV   # size overflow
    assert st("ds_pad", FAKE, 2, 1, 1 << 29, 16) == UNS    # row longer than 2^30 words
    assert st("ds_pad_ex", FAKE, 4, 5, 4, 4, None, None) == INV


def test_regular_noops_need_no_device():
    assert st("ds_pad", FAKE, 0, 5, 9, 4) == 0            # rows == 0: no launch, no sync
    assert st("ds_unpad", FAKE, 7, 5, 5, 4) == 0           # cols == new_cols
    assert st("ds_unpad", FAKE, 7, 5, 0, 4) == 0           # nothing kept
    assert st("ds_slide", FAKE, 9, 0, 4) == 0              # shift 0
    assert st("ds_pad_ex", FAKE, 0, 5, 9, 4, None, None) == 0
    assert st("ds_pad_ex", FAKE, 7, 5, 5, 4, None, None) == 0     # new_cols == cols
    assert st("ds_unpad_ex", FAKE, 7, 5, 0, 4, None) == 0         # nothing kept


def test_shard_helper_validation():
    assert st("ds_shard_offsets", None, 2, 0, FAKE, None) == INV
    assert st("ds_shard_offsets", FAKE, 2, 2, FAKE, None) == INV
    assert st("ds_shard_offsets", FAKE, 0, 0, FAKE, None) == INV
    assert st("ds_halo_entry", FAKE, 4, None, None) == INV
    assert st("ds_halo_entry", None, 4, FAKE, None) == INV


def test_binding_rejects_host_tensors():
    import torch
    t = torch.zeros(8, dtype=torch.int32)
    with pytest.raises(ValueError):
        libds.ds_compact(t, 8, 0)


def test_partition_and_copy_validation():
    assert st("ds_partition", FAKE, 10, 0, None, out_sz()) == INV        # no aux
    assert st("ds_partition", FAKE, 10, 9, FAKE, out_sz()) == INV        # bad predicate
    assert st("ds_partition_ex", FAKE, 10, 0, 0, FAKE, None, None) == INV  # count required
    assert st("ds_select_copy_ex", FAKE, 10, 0, 0, None, None, None) == INV  # no out
    assert st("ds_select_copy_ex", FAKE, 10, 0, 0, BAD, None, None) == INV   # misaligned out
    assert st("ds_partition_copy_ex", FAKE, 10, 0, 0, FAKE, None, None, None) == INV
    # overlapping buffers are rejected before the device is touched
    W = FAKE + 0x10000
    assert st("ds_partition", FAKE, 10, 0, FAKE + 36, out_sz()) == INV            # aux inside ptr[0, 10)
    assert st("ds_partition_ex", FAKE, 10, 0, 0, FAKE - 36, W, None) == INV        # aux ends inside ptr
    assert st("ds_select_copy_ex", FAKE, 10, 0, 0, FAKE + 4, None, None) == INV    # shifted by one word
    assert st("ds_partition_copy_ex", FAKE, 10, 0, 0, W, W + 8, None, None) == INV  # true / false overlap
    assert st("ds_partition_copy_ex", FAKE, 10, 0, 0, FAKE, W, None, None) == INV   # out_true == in


def test_slide_validation_before_device():
    assert st("ds_slide_ex", FAKE, 10, 11, 4, None) == INV     # shift > n
    assert st("ds_slide_ex", FAKE, 10, 1, 3, None) == INV      # bad elem_bytes
    assert st("ds_slide_ex", FAKE, 10, 1, 2, None) == UNS      # 1/2-byte elements
    assert st("ds_slide_ex", None, 10, 1, 4, None) == INV      # NULL with data
    assert st("ds_slide_ex", BAD, 10, 1, 4, None) == INV       # misaligned
    assert st("ds_slide_ex", FAKE, 1 << 62, 1, 16, None) == INV  # size overflow
    assert st("ds_slide_ex", FAKE, 10, 0, 4, None) == 0         # nothing moves
    assert st("ds_slide_ex", FAKE, 10, 10, 4, None) == 0        # nothing kept
    assert st("ds_slide_ex", None, 0, 0, 4, None) == 0


def test_wide_validation_before_device():
    assert st("ds_compact64_ex", BAD, 10, 0, None, None) == INV          # 4-byte aligned only
    assert st("ds_compact64_ex", FAKE + 4, 10, 0, None, None) == INV     # not 8-byte aligned
    assert st("ds_compact64_ex", None, 10, 0, None, None) == INV
    assert st("ds_select64_ex", FAKE, 10, 9, 0, None, None) == INV       # bad predicate
    assert st("ds_compact64_ex", FAKE, 1 << 40, 0, None, None) == UNS    # > 2^35 elements
    assert st("ds_unique64", FAKE, 10, None) == INV                      # out_n required
    n = ctypes.c_size_t(99)
    assert st("ds_unique64", FAKE, 0, ctypes.byref(n)) == 0 and n.value == 0


def test_count_board_validation():
    """Count boards: argument checks need no device."""
    assert st("ds_board_alloc", 0, None) == INV
    assert st("ds_board_ipc_handle", None, None) == INV
    assert st("ds_board_ipc_open", None, None) == INV
    assert st("ds_board_ipc_close", None) == INV
    assert st("ds_shard_offsets_board", None, 2, 0, 1, None, FAKE, None) == INV
    assert st("ds_shard_offsets_board", FAKE, 2, 2, 1, None, FAKE, None) == INV
    assert st("ds_compact_pub_ex", FAKE, 8, 0, None, None, None) == INV        # no ds_publish
    pub = libds.DsPublish(0, 2, 0, 1)                                          # no board pointers
    assert st("ds_compact_pub_ex", FAKE, 8, 0, None, ctypes.byref(pub), None) == INV
    pub = libds.DsPublish(FAKE, 2, 2, 1)                                       # rank >= world
    assert st("ds_select_pub_ex", FAKE, 8, 1, 0, None, ctypes.byref(pub), None) == INV
    assert st("ds_unique_pub_ex", FAKE, 8, None, 3, None, ctypes.byref(libds.DsPublish(FAKE, 1, 0, 1)),
              None) == INV                                                     # halo_len without a halo
