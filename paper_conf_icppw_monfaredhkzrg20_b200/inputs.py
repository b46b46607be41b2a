"""Seeded synthetic key/IV generator shared by the oracle tests and the CUDA path.

This module holds NONE of the method's arithmetic (no cipher, no slicing, no
keystream).  It only draws the random inputs both sides consume, so that the
oracle and the GPU path are fed identical bytes.

PAPER.md:628-632 (sec. 4.4) says only that each MICKEY instance gets an 80-bit
IV expanded from "a carefully selected pre-stored random number set" by an
unspecified non-linear function.  DESIGN.md reading R5 replaces that with a
counter-based SplitMix64 stream so that any instance's key/IV is O(1) to derive
from (seed, global instance id) and sharding cannot change it
(a multi-GPU run must reproduce the single-GPU output).

Instance i uses SplitMix64 outputs 4i .. 4i+3 (x0..x3) of the stream with seed
S, where output k = fmix64(S + (k + 1) * 0x9E3779B97F4A7C15) mod 2^64:

=============  ==============================  ==============================
cipher         key                              IV / counter
=============  ==============================  ==============================
MICKEY 2.0     LE(x0) || LE(x1)[0:2]  (10 B)    LE(x2) || LE(x3)[0:2]  (10 B)
Grain v1       LE(x0) || LE(x1)[0:2]  (10 B)    LE(x2)                 (8 B)
AES-128-CTR    LE(x0) || LE(x1)       (16 B)    LE(x2) || LE(x3)       (16 B)
LFSR-128       LE(x0) || LE(x1)       (16 B)    none
=============  ==============================  ==============================

AES-128-CTR runs every instance under ONE key ("different
counter values ... with a unique key"): the handle key is global instance 0's
key row, ``aes_key(seed)``, whatever shard is being generated; each instance's
IV row is its initial 128-bit big-endian counter block.
"""
from __future__ import annotations

import numpy as np

GAMMA = np.uint64(0x9E3779B97F4A7C15)
M1 = np.uint64(0xBF58476D1CE4E5B9)
M2 = np.uint64(0x94D049BB133111EB)
DEFAULT_SEED = 0x5EED2020

KEY_BYTES = {"mickey2": 10, "grain": 10, "aes128ctr": 16, "lfsr128": 16}
IV_BYTES = {"mickey2": 10, "grain": 8, "aes128ctr": 16, "lfsr128": 0}


def fmix64(z: np.ndarray) -> np.ndarray:
    """SplitMix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * M1
        z = (z ^ (z >> np.uint64(27))) * M2
    return z ^ (z >> np.uint64(31))


def splitmix64(seed: int, k: np.ndarray) -> np.ndarray:
    """Output k (0-based) of the SplitMix64 stream with the given seed."""
    k = np.asarray(k, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + (k + np.uint64(1)) * GAMMA
    return fmix64(z)


def make_inputs(cipher: str, n: int, first_instance: int = 0, seed: int = DEFAULT_SEED):
    """Keys and IVs for instances [first_instance, first_instance + n).

    Returns (keys uint8[n, key_bytes], ivs uint8[n, iv_bytes]), row-major.
    """
    if cipher not in KEY_BYTES:
        raise ValueError(f"unknown cipher {cipher!r}")
    ids = np.arange(first_instance, first_instance + n, dtype=np.uint64)
    k = (ids * np.uint64(4))[:, None] + np.arange(4, dtype=np.uint64)[None, :]
    x = splitmix64(seed, k)                       # [n, 4] uint64
    xb = x.astype("<u8").view(np.uint8).reshape(n, 4, 8)
    kb, vb = KEY_BYTES[cipher], IV_BYTES[cipher]
    keys = np.concatenate([xb[:, 0, :], xb[:, 1, :]], axis=1)[:, :kb]
    ivs = np.concatenate([xb[:, 2, :], xb[:, 3, :]], axis=1)[:, :vb]
    return np.ascontiguousarray(keys), np.ascontiguousarray(ivs)


def aes_key(seed: int = DEFAULT_SEED) -> np.ndarray:
    """The single AES-128 key of a seeded workload: global instance 0's key row."""
    keys, _ = make_inputs("aes128ctr", 1, 0, seed)
    return keys[0].copy()
