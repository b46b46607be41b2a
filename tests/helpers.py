"""Test-side layout helpers: re-express oracle keystreams (row-major bytes) in
the library's SLICED and CHECKSUM layouts (include/bsrng.h definitions).
These are plain numpy re-layouts of oracle output; no cipher arithmetic."""
import numpy as np

GAMMA = 0x9E3779B97F4A7C15
C_T0 = 0xBF58476D1CE4E5B9
MASK64 = (1 << 64) - 1


def bits_of_rows(rows: np.ndarray, msb_first: bool = True) -> np.ndarray:
    """uint8[n, bytes] -> uint8[n, bits] (keystream bit t of instance i)."""
    return np.unpackbits(rows, axis=1, bitorder="big" if msb_first else "little")


def to_sliced(rows: np.ndarray, msb_first: bool = True) -> np.ndarray:
    """uint8[n, bits/8] -> uint32[bits, G]; bit j of [t][g] = bit t of 32g+j."""
    b = bits_of_rows(rows, msb_first)
    n, bits = b.shape
    G = (n + 31) // 32
    pad = np.zeros((G * 32, bits), dtype=np.uint8)
    pad[:n] = b
    pad = pad.reshape(G, 32, bits).astype(np.uint64)
    w = np.zeros((G, bits), dtype=np.uint64)
    for j in range(32):
        w |= pad[:, j, :] << np.uint64(j)
    return w.T.astype(np.uint32)


def fmix64(z: int) -> int:
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def checksum(sliced: np.ndarray, t0: int = 0, g_base: int = 0) -> int:
    """CHECKSUM layout definition (include/bsrng.h) over a SLICED block."""
    acc = np.bitwise_xor.reduce(sliced.astype(np.uint32), axis=0)
    tot = 0
    for g, a in enumerate(acc.tolist()):
        tot = (tot + fmix64(a ^ (((g_base + g) * GAMMA) & MASK64) ^ ((t0 * C_T0) & MASK64))) & MASK64
    return tot


def state_to_sliced(r: np.ndarray, s: np.ndarray) -> np.ndarray:
    """Per-instance oracle states r[n,100], s[n,100] (0/1) -> uint32[200, G]."""
    st = np.concatenate([r, s], axis=1)  # [n, 200]
    n = st.shape[0]
    G = (n + 31) // 32
    pad = np.zeros((G * 32, 200), dtype=np.uint64)
    pad[:n] = st
    pad = pad.reshape(G, 32, 200)
    w = np.zeros((G, 200), dtype=np.uint64)
    for j in range(32):
        w |= pad[:, j, :] << np.uint64(j)
    return w.T.astype(np.uint32)
