"""Pins for the AES-128 / CTR oracle (oracle/aes_ref.c).

  * FIPS-197 and SP 800-38A known answers (golden fixture, cited);
  * the S-box it computes from the GF(2^8) definition is a permutation with
    no fixed points and S(0) = 0x63 (FIPS-197 Fig. 7);
  * the library routine: `cryptography` (OpenSSL) AES-128-ECB / CTR on random
    keys, blocks and counters -- an exact special case of the same function;
  * counter wrap-around at 2^128 and random access (first_block offset).
"""
import numpy as np
import pytest

import oracle
from conftest import read_golden

RNG = np.random.default_rng(288338)


@pytest.mark.parametrize("row", read_golden("aes128_vectors.txt"), ids=lambda r: r[0] + r[2][:6])
def test_known_answers(row):
    kind, key, inp, out = row
    key, inp = bytes.fromhex(key), bytes.fromhex(inp)
    if kind == "block":
        assert oracle.aes128_encrypt_block(key, inp).hex() == out
    else:
        assert oracle.aes128_ctr_keystream(key, inp, len(out) // 32).hex() == out


def test_sbox_structure():
    s = oracle.aes_sbox()
    assert sorted(s.tolist()) == list(range(256))
    assert s[0] == 0x63 and s[1] == 0x7C and s[0x53] == 0xED
    assert not np.any(s == np.arange(256))


def test_against_cryptography_library():
    cg = pytest.importorskip("cryptography.hazmat.primitives.ciphers")
    from cryptography.hazmat.primitives.ciphers import Cipher, algorithms, modes
    for _ in range(8):
        key = RNG.bytes(16)
        ctr = RNG.bytes(16)
        nb = int(RNG.integers(1, 40))
        enc = Cipher(algorithms.AES(key), modes.CTR(ctr)).encryptor()
        want = enc.update(bytes(16 * nb)) + enc.finalize()
        assert oracle.aes128_ctr_keystream(key, ctr, nb) == want
        blk = RNG.bytes(16)
        e2 = Cipher(algorithms.AES(key), modes.ECB()).encryptor()
        assert oracle.aes128_encrypt_block(key, blk) == e2.update(blk) + e2.finalize()


def test_counter_wrap_and_offset():
    key = bytes(range(16))
    ctr = bytes([0xFF] * 15 + [0xFE])
    ks = oracle.aes128_ctr_keystream(key, ctr, 4)
    # block 2 uses counter 0x00..00 after the 128-bit wrap
    assert ks[32:48] == oracle.aes128_encrypt_block(key, bytes(16))
    assert oracle.aes128_ctr_keystream(key, ctr, 2, first_block=2) == ks[32:64]
