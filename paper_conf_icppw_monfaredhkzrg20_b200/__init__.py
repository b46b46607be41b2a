"""B200-native bitsliced keystream generation (BSRNG, ICPP Workshops '20).

The hot path (bitsliced MICKEY 2.0 keystream; sec. 4.4-4.5)
runs in hand-written sm_100a CUDA kernels behind the C ABI in
``include/bsrng.h``; :mod:`.bsrng` is the thin ctypes binding and
:mod:`.inputs` the seeded synthetic key/IV generator.

Submodules are imported lazily so that the input generator can be used on a
CPU-only box without loading the CUDA library.
"""

__all__ = ["bsrng", "inputs", "build"]
