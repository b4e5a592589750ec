"""B200-native Speculative Reconvergence hot path (Damani et al., CGO'20).

The product is ``libsr.so`` (C ABI declared in ``include/sr.h``, CUDA kernels
for sm_100a in ``csrc/``); :mod:`.sr` is its thin ctypes binding.  Importing
this package does not load the library; :func:`sr.load` does, and fails
loudly when it is missing -- there is no CPU fallback.
"""
__all__ = ["inputs", "sr"]
