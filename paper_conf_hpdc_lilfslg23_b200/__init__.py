"""B200-native GPU-FPX exception scan (HPDC '23, Li et al.), hot path only.

The product is ``libfpx.so`` (C ABI declared in ``include/fpx.h``; sm_100a
kernels in ``csrc/``).  ``fpx`` is the thin ctypes binding with the same
names; ``dist`` is the multi-GPU record-shard + NCCL merge.
"""
__all__ = ["fpx", "dist"]
