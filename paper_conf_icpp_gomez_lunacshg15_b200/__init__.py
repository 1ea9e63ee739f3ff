"""libds -- in-place Data Sliding (pad / unpad / compact / select / unique) on B200.

The product is the C-ABI library ``libds.so`` (include/ds.h) built from
``csrc/`` for sm_100a by ``build``; ``libds`` is its ctypes binding (same
names as the C entry points) and ``dist`` the sharded multi-GPU driver.
Importing ``libds`` fails loudly if the CUDA library was not built; there is
no CPU fallback.
"""
