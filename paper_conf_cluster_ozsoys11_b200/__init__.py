"""B200-native chunked LZSS (CULZSS, Ozsoy & Swany, CLUSTER 2011).

The compute path lives in ``libculzss.so`` (hand-written sm_100a CUDA behind a
C ABI, ``include/culzss.h``); ``culzss`` is the thin ctypes binding.  Import
of this package is light: the shared library is loaded on first use and
raises if it is missing (there is no CPU fallback).
"""

__all__ = ["culzss", "datagen"]
