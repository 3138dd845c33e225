"""B200-native XSBench event-based macroscopic cross-section lookup.

The hot path of Tian et al., SC-W 2023 (XSBench "-m event", PAPER.md:835,
PAPER.md:911-915) as a C-ABI CUDA library (include/xs.h, built in-tree as
libxs.so) with a thin ctypes binding (``xs``) and a multi-GPU driver
(``dist``).  Importing ``xs`` fails loudly when libxs.so is missing: there is
no CPU fallback.
"""
__all__ = ["xs", "dist"]
