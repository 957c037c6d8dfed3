"""B200-native mSTAMP (multi-dimensional matrix profile) hot path.

The compute path is the C-ABI library ``libmstamp_b200.so`` (include/mp.h),
built from ``csrc/`` for sm_100a; ``mstamp`` is its thin ctypes binding.
Importing the package does not load the library; ``mstamp.load()`` does, and
fails loudly if it is missing -- there is no CPU fallback.
"""
__all__ = ["datagen", "mstamp"]
