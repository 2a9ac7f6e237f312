"""B200-native VPIC particle hot path (Tan et al., SC Workshops '25).

The product is ``libvpic.so`` (C-ABI, ``include/vpic.h``) built from ``csrc/``
for sm_100a; ``vpic`` is its thin ctypes binding (argument marshalling only).
``inputs`` holds the seeded synthetic workloads.  Importing the package does
not load the CUDA library; the first call into ``vpic`` does, and raises if it
is missing -- there is no CPU fallback.
"""
__all__ = ["vpic", "inputs"]
