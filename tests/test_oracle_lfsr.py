"""Pins for the 128-bit Fibonacci LFSR oracle (oracle/lfsr_ref.c), the paper's
bitsliced-LFSR example (Eq. 2) with p(x) = x^128 + x^29 +
x^27 + x^2 + 1 (reading L1).

  * the step matrix obtained by driving the oracle has order exactly 2^128 - 1
    (p primitive: maximal period, Eq. 1);
  * Berlekamp-Massey (the textbook algorithm, written here) recovers exactly
    p(x) and linear complexity 128 from the oracle's output stream.
"""
import numpy as np

import oracle

FERMAT = [3, 5, 17, 257, 65537, 641, 6700417, 274177, 67280421310721]


def _matrix():
    cols = []
    for j in range(128):
        s = np.zeros(128, np.uint8)
        s[j] = 1
        s2, _ = oracle.lfsr128_clock(s)
        cols.append(s2)
    return [sum(int(cols[j][i]) << j for j in range(128)) for i in range(128)]


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


def test_step_matrix_order_is_maximal():
    N = 2 ** 128 - 1
    prod = 1
    for p in FERMAT:
        prod *= p
    assert prod == N
    M = _matrix()
    ident = [1 << i for i in range(128)]
    assert _matpow(M, N) == ident
    for p in FERMAT:
        assert _matpow(M, N // p) != ident


def _berlekamp_massey(bits):
    """Shortest LFSR (connection polynomial C, length L) generating bits."""
    n = len(bits)
    C = [1] + [0] * n
    B = [1] + [0] * n
    L, m = 0, 1
    for i in range(n):
        d = bits[i]
        for j in range(1, L + 1):
            d ^= C[j] & bits[i - j]
        if d == 0:
            m += 1
        elif 2 * L <= i:
            T = C[:]
            for j in range(m, n + 1):
                C[j] ^= B[j - m]
            L, B, m = i + 1 - L, T, 1
        else:
            for j in range(m, n + 1):
                C[j] ^= B[j - m]
            m += 1
    return C[: L + 1], L


def test_berlekamp_massey_recovers_polynomial():
    key = bytes(np.random.default_rng(545596).integers(0, 256, 16, dtype=np.uint8))
    ks = oracle.lfsr128_keystream(key, 600)
    bits = [(ks[t // 8] >> (7 - t % 8)) & 1 for t in range(600)]
    C, L = _berlekamp_massey(bits)
    assert L == 128
    # connection polynomial C(x) = 1 + x^99 + x^101 + x^126 + x^128 (reciprocal of p)
    assert [i for i, c in enumerate(C) if c] == [0, 128 - 29, 128 - 27, 128 - 2, 128]


def test_first_bits_are_the_key():
    key = bytes(range(16))
    assert oracle.lfsr128_keystream(key, 128) == key
