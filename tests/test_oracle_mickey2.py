"""Pins for the bit-serial MICKEY 2.0 oracle (oracle/mickey2_ref.c).

Every test here checks the oracle against something other than itself:
  * the specification's published test vectors (golden fixture, cited);
  * a mathematical property the spec fixes (R's feedback polynomial is
    primitive: Eq. 1 -- "primitive polynomial -> period
    2^n - 1" -- applied to MICKEY's linear register R);
  * the register/tap wiring the paper draws (Fig. 2, PAPER.md:258-273:
    control bits R67/S34 and S67/R33, mixing into R; sec. 4.4, PAPER.md:597-603:
    two 100-bit registers), checked by brute-force bit-flip probing;
  * the second, independently encoded form of the tables (packed masks,
    SURVEY.md A.3) against the oracle's spec-row transcription.
"""
import numpy as np
import pytest

import oracle
from conftest import read_golden

RNG = np.random.default_rng(20200817)


# --------------------------------------------------------------- spec vectors
@pytest.mark.parametrize("row", read_golden("mickey2_spec_vectors.txt"), ids=lambda r: r[0])
def test_spec_vectors(row):
    name, key, iv, iv_bits, prefix = row
    key = bytes.fromhex(key)
    iv = b"" if iv == "-" else bytes.fromhex(iv)
    iv_bits = int(iv_bits)
    nbits = len(prefix) * 4
    assert oracle.mickey2_keystream(key, iv, iv_bits, nbits).hex() == prefix


def test_prefix_consistency_and_determinism():
    key = bytes(range(10))
    iv = bytes(range(10, 20))
    long = oracle.mickey2_keystream(key, iv, 80, 1000)
    for n in (8, 96, 504, 1000):
        assert oracle.mickey2_keystream(key, iv, 80, n) == long[: n // 8]
    # non-multiple-of-8 lengths: trailing bits of the last byte are zero
    s = oracle.mickey2_keystream(key, iv, 80, 13)
    assert s[0] == long[0] and s[1] == (long[1] & 0xF8)
    assert oracle.mickey2_keystream(key, iv, 80, 1000) == long


def test_iv_bits_range():
    with pytest.raises(ValueError):
        oracle.mickey2_keystream(bytes(10), bytes(10), 81, 8)
    with pytest.raises(ValueError):
        oracle.mickey2_keystream(bytes(10), bytes(10), -1, 8)


def test_iv_length_matters():
    """Spec: the IV length is part of the init (iv_bits clocks), so a 32-bit IV
    and the same bytes zero-padded to 80 bits give different keystreams."""
    key = bytes.fromhex("123456789abcdef01234")
    a = oracle.mickey2_keystream(key, bytes.fromhex("21436587"), 32, 64)
    b = oracle.mickey2_keystream(key, bytes.fromhex("21436587") + bytes(6), 80, 64)
    assert a != b


# ------------------------------------------------------------ tables (A.2/A.3)
MASKS = {  # bit i at word i/32, bit i%32
    "RTAPS": [0x1279327B, 0xB5546660, 0xDF87818F, 0x00000003],
    "COMP0": [0x6AA97A30, 0x7942A809, 0x057EBFEA, 0x00000006],
    "COMP1": [0xDD629E9A, 0xE3A21D63, 0x91C23DD7, 0x00000001],
    "FB0": [0x9FFA7FAF, 0xAF4A9381, 0x9CEC5802, 0x00000001],
    "FB1": [0x4C8CB877, 0x4911B063, 0x40FBC52B, 0x00000008],
}


@pytest.mark.parametrize("name", list(MASKS))
def test_tables_match_packed_masks(name):
    row = oracle.mickey2_table(name)
    words = MASKS[name]
    for i in range(100):
        want = (words[i // 32] >> (i % 32)) & 1
        if name.startswith("COMP") and i in (0, 99):
            continue  # COMP0/COMP1 are only used for 1 <= i <= 98
        assert row[i] == want, (name, i)


def test_table_invariants():
    assert oracle.mickey2_table("RTAPS").sum() == 50
    fb0, fb1 = oracle.mickey2_table("FB0"), oracle.mickey2_table("FB1")
    cat = {(a, b): int(((fb0 == a) & (fb1 == b)).sum()) for a in (0, 1) for b in (0, 1)}
    assert cat == {(1, 1): 22, (1, 0): 32, (0, 1): 23, (0, 0): 23}


# ------------------------------------------------ R is a primitive-poly LFSR
def _r_matrix(ctl):
    """Rows (as int bitmasks) of the linear map r -> r' applied by one
    CLOCK_KG(mixing=0, input=0) with CONTROL_BIT_R forced to `ctl`
    (S chosen so that s34 ^ r67 == ctl)."""
    cols = []
    for j in range(100):
        r = np.zeros(100, np.uint8)
        s = np.zeros(100, np.uint8)
        r[j] = 1
        s[34] = ctl ^ r[67]
        r2, _ = oracle.mickey2_clock_kg(r, s, 0, 0)
        cols.append(r2)
    return [sum(int(cols[j][i]) << j for j in range(100)) for i in range(100)]


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


def _is_prime(p):
    return p > 1 and all(p % d for d in range(2, int(p ** 0.5) + 1))


def test_r_feedback_polynomial_is_primitive():
    """Order of the R step matrix (control bit 0) is exactly 2^100 - 1."""
    M = _r_matrix(0)
    ident = [1 << i for i in range(100)]
    N = 2 ** 100 - 1
    primes = [3, 5, 11, 31, 41, 101, 251, 601, 1801, 4051, 8101, 268501]
    assert all(_is_prime(p) for p in primes)
    rem = N
    for p in primes:
        while rem % p == 0:
            rem //= p
    assert rem == 1  # the factorisation is complete
    assert _matpow(M, N) == ident
    for p in primes:
        assert _matpow(M, N // p) != ident, p


def test_r_control_bit_adds_identity():
    """CONTROL_BIT_R = 1 clocks R by M + I (spec: r'_i ^= r_i)."""
    M0, M1 = _r_matrix(0), _r_matrix(1)
    assert [a ^ b for a, b in zip(M0, M1)] == [1 << i for i in range(100)]


# ------------------------------------------ wiring (Fig. 2) by bit-flip probing
def _deps(mixing, trials=24):
    """dep[o][b] = 1 iff flipping input bit b (0..99 = r, 100..199 = s) changed
    output bit o (0..99 = r', 100..199 = s') in some random trial."""
    dep = np.zeros((200, 200), dtype=bool)
    for _ in range(trials):
        r = RNG.integers(0, 2, 100, dtype=np.uint8)
        s = RNG.integers(0, 2, 100, dtype=np.uint8)
        inp = int(RNG.integers(0, 2))
        r0, s0 = oracle.mickey2_clock_kg(r, s, mixing, inp)
        base = np.concatenate([r0, s0])
        for b in range(200):
            r1, s1 = r.copy(), s.copy()
            if b < 100:
                r1[b] ^= 1
            else:
                s1[b - 100] ^= 1
            ra, sa = oracle.mickey2_clock_kg(r1, s1, mixing, inp)
            dep[:, b] |= np.concatenate([ra, sa]) != base
    return dep


@pytest.mark.parametrize("mixing", [0, 1])
def test_cross_register_wiring(mixing):
    dep = _deps(mixing)
    # R' reads from S only through CONTROL_BIT_R (s34) and, when mixing, s50.
    s_into_r = set(np.nonzero(dep[:100, 100:].any(axis=0))[0].tolist())
    assert s_into_r == ({34, 50} if mixing else {34})
    # S' reads from R only through CONTROL_BIT_S (r33).
    r_into_s = set(np.nonzero(dep[100:, :100].any(axis=0))[0].tolist())
    assert r_into_s == {33}
    # R' reads r67 (CONTROL_BIT_R) and S' reads s67 (CONTROL_BIT_S).
    assert dep[:100, 67].sum() > 90
    assert dep[100:, 167].sum() > 40


def test_register_locality():
    """Each new bit depends only on its neighbours, the feedback bit (r99 / s99)
    and the control bits -- the shift-register structure of Fig. 2."""
    dep = _deps(0)
    for i in range(100):
        r_src = set(np.nonzero(dep[i, :100])[0].tolist())
        assert r_src <= {i - 1, i, 99, 67}, (i, r_src)
        s_src = set(np.nonzero(dep[100 + i, 100:])[0].tolist())
        assert s_src <= {i - 1, i, i + 1, 99, 67}, (i, s_src)
