"""CPU check of the generated MixColumns + AddRoundKey circuit the AES kernels
include (csrc/aes_mc_lop3.inc, written by tools/mc_xor3.py): every output
word of the 84-gate XOR program equals FIPS-197 sec. 5.1.3's MixColumns
(out_i = 2 a_i + 3 a_{i+1} + a_{i+2} + a_{i+3} over GF(2^8)) plus the key,
evaluated here byte-wise from the definition on random bitsliced columns."""
import os
import re

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
INC = os.path.join(ROOT, "paper_conf_icppw_monfaredhkzrg20_b200", "csrc", "aes_mc_lop3.inc")


def xtime(b):
    return ((b << 1) ^ (0x1B if b & 0x80 else 0)) & 0xFF


def mix_column(col):
    a = col
    return [xtime(a[i]) ^ xtime(a[(i + 1) % 4]) ^ a[(i + 1) % 4] ^ a[(i + 2) % 4] ^ a[(i + 3) % 4]
            for i in range(4)]


def run_inc(a, kk):
    """execute the generated statements on python ints (32-lane words)"""
    env = {"a": a, "kk": kk, "o": [0] * 32,
           "x2": lambda x, y: x ^ y, "x3": lambda x, y, z: x ^ y ^ z}
    src = open(INC).read()
    n_gates = 0
    for line in src.splitlines():
        line = line.strip()
        if not line or line.startswith("//"):
            continue
        n_gates += 1
        stmt = re.sub(r"^const uint32_t ", "", line).rstrip(";")
        exec(stmt, env)
    return env["o"], n_gates


def test_mc_circuit_matches_fips197():
    rng = np.random.default_rng(197)
    for _ in range(8):
        cols = rng.integers(0, 256, size=(32, 4))      # 32 lanes x 4 bytes
        keys = rng.integers(0, 256, size=(32, 4))
        # bitslice: word (byte i, MSB-first bit b) has bit j = that bit of lane j
        a = [0] * 32
        kk = [0] * 32
        for j in range(32):
            for i in range(4):
                for b in range(8):
                    a[8 * i + b] |= ((int(cols[j, i]) >> (7 - b)) & 1) << j
                    kk[8 * i + b] |= ((int(keys[j, i]) >> (7 - b)) & 1) << j
        o, n = run_inc(a, kk)
        assert n == 84
        for j in range(32):
            want = [m ^ int(k) for m, k in zip(mix_column([int(x) for x in cols[j]]), keys[j])]
            got = [sum(((o[8 * i + b] >> j) & 1) << (7 - b) for b in range(8)) for i in range(4)]
            assert got == want, j
