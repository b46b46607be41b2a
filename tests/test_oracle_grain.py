"""Pins for the bit-serial Grain v1 oracle (oracle/grain_ref.c).

  * the specification's test vectors (golden fixture, cited);
  * the LFSR feedback f is a primitive polynomial (period 2^80 - 1), the
    property PAPER.md:207-228 (Eq. 1) states for maximal LFSRs and the Grain
    design requires of its LFSR (Fig. 4);
  * the wiring of f, g, h and the output taps, by bit-flip probing (Fig. 4:
    LFSR feeds the NFSR through s_i, h reads 4 LFSR bits + 1 NFSR bit, the
    output adds 7 NFSR bits), and the init-mode feedback of z into both
    registers.
"""
import numpy as np
import pytest

import oracle
from conftest import read_golden

RNG = np.random.default_rng(339357)


@pytest.mark.parametrize("row", read_golden("grain_v1_spec_vectors.txt"), ids=lambda r: r[0])
def test_spec_vectors(row):
    _, key, iv, ks = row
    got = oracle.grain_keystream(bytes.fromhex(key), bytes.fromhex(iv), len(ks) * 4)
    assert got.hex() == ks


def test_prefix_consistency():
    k, v = bytes(range(10)), bytes(range(8))
    long = oracle.grain_keystream(k, v, 800)
    for n in (8, 64, 792):
        assert oracle.grain_keystream(k, v, n) == long[: n // 8]
    s = oracle.grain_keystream(k, v, 13)  # LSB-first: bits 8..12 in the low bits of byte 1
    assert s[1] == long[1] & 0x1F


def _lfsr_matrix():
    """Rows (int bitmasks) of the LFSR step s -> s' (non-init clock), from the
    oracle's own clock on unit vectors (the LFSR does not read the NFSR)."""
    cols = []
    for j in range(80):
        s = np.zeros(80, np.uint8)
        s[j] = 1
        s2, _, _ = oracle.grain_clock(s, np.zeros(80, np.uint8), 0)
        cols.append(s2)
    return [sum(int(cols[j][i]) << j for j in range(80)) for i in range(80)]


def _matmul(A, B):
    out = []
    for a in A:
        c, k = 0, 0
        while a:
            if a & 1:
                c ^= B[k]
            a >>= 1
            k += 1
        out.append(c)
    return out


def _matpow(A, e):
    R = [1 << i for i in range(len(A))]
    while e:
        if e & 1:
            R = _matmul(R, A)
        A = _matmul(A, A)
        e >>= 1
    return R


def test_lfsr_is_primitive():
    M = _lfsr_matrix()
    ident = [1 << i for i in range(80)]
    N = 2 ** 80 - 1
    primes = [3, 5, 11, 17, 31, 41, 257, 61681, 4278255361]
    rem = N
    for p in primes:
        assert all(p % d for d in range(2, int(p ** 0.5) + 1))
        while rem % p == 0:
            rem //= p
    assert rem == 1
    assert _matpow(M, N) == ident
    for p in primes:
        assert _matpow(M, N // p) != ident, p


def _deps(init_mode, trials=32):
    """dep_s79/dep_b79/dep_z: which input bits (0..79 s, 80..159 b) change the
    new LFSR bit, the new NFSR bit and the output bit."""
    ds = np.zeros(160, bool)
    db = np.zeros(160, bool)
    dz = np.zeros(160, bool)
    for _ in range(trials):
        s = RNG.integers(0, 2, 80, dtype=np.uint8)
        b = RNG.integers(0, 2, 80, dtype=np.uint8)
        s0, b0, z0 = oracle.grain_clock(s, b, init_mode)
        for i in range(160):
            s1, b1 = s.copy(), b.copy()
            if i < 80:
                s1[i] ^= 1
            else:
                b1[i - 80] ^= 1
            sa, ba, za = oracle.grain_clock(s1, b1, init_mode)
            ds[i] |= sa[79] != s0[79]
            db[i] |= ba[79] != b0[79]
            dz[i] |= za != z0
            # the other 79 bits are a plain shift
            assert np.array_equal(sa[:79], s1[1:]) and np.array_equal(ba[:79], b1[1:])
    idx = lambda d: set(np.nonzero(d)[0].tolist())
    return idx(ds), idx(db), idx(dz)


def test_wiring_keystream_mode():
    ds, db, dz = _deps(0)
    assert ds == {0, 13, 23, 38, 51, 62}                       # f
    g_taps = {0, 9, 14, 15, 21, 28, 33, 37, 45, 52, 60, 62, 63}  # g's b indices
    assert db == {0} | {80 + t for t in g_taps}                  # s_0 + g(b)
    assert dz == {3, 25, 46, 64} | {80 + t for t in (1, 2, 4, 10, 31, 43, 56, 63)}


def test_wiring_init_mode():
    """Init clocks add z to both feedbacks: the new bits depend on the union of
    f (resp. s_0 + g) and z's inputs, which are disjoint from f's taps."""
    ds0, db0, z_in = _deps(0)
    ds, db, dz = _deps(1)
    assert dz == z_in
    assert ds == ds0 | z_in
    assert db == db0 | z_in
