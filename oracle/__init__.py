"""CPU oracle for the BSRNG hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product package ``paper_conf_icppw_monfaredhkzrg20_b200`` never imports it and
shares no code with it.

The arithmetic lives in plain C -- ``mickey2_ref.c`` (bit-serial MICKEY 2.0,
spec [5]), ``grain_ref.c`` (bit-serial Grain v1, spec [15],
PAPER.md:898-899), ``aes_ref.c`` (byte-oriented AES-128 + CTR, FIPS-197 [35],
PAPER.md:957-959), ``lfsr_ref.c`` (the paper's bitsliced-LFSR example, Eq. 2,
PAPER.md:545-596) -- compiled here into ``liboracle.so`` with gcc and called
through ctypes.  This module only marshals arguments.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from concurrent.futures import ThreadPoolExecutor

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SOURCES = ["mickey2_ref.c", "grain_ref.c", "aes_ref.c", "lfsr_ref.c"]
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile the C oracle with gcc (no GPU code involved)."""
    srcs = [os.path.join(_HERE, s) for s in _SOURCES]
    if (not force and os.path.exists(_LIB_PATH)
            and all(os.path.getmtime(_LIB_PATH) >= os.path.getmtime(s) for s in srcs)):
        return _LIB_PATH
    tmp = _LIB_PATH + f".tmp{os.getpid()}"
    cmd = ["gcc", "-O2", "-std=c99", "-shared", "-fPIC", "-Wall", "-Wextra", "-o", tmp] + srcs
    subprocess.run(cmd, check=True)
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        u8p = ctypes.POINTER(ctypes.c_uint8)
        L.ref_mickey2_keystream.argtypes = [u8p, u8p, ctypes.c_int, ctypes.c_uint64, u8p]
        L.ref_mickey2_keystream.restype = ctypes.c_int
        L.ref_mickey2_state.argtypes = [u8p, u8p, ctypes.c_int, ctypes.c_uint64, u8p, u8p]
        L.ref_mickey2_state.restype = ctypes.c_int
        L.ref_mickey2_clock_kg.argtypes = [u8p, u8p, ctypes.c_int, ctypes.c_int]
        L.ref_mickey2_clock_kg.restype = None
        L.ref_mickey2_table.argtypes = [ctypes.c_int, ctypes.c_int]
        L.ref_mickey2_table.restype = ctypes.c_int
        L.ref_grain_keystream.argtypes = [u8p, u8p, ctypes.c_uint64, u8p]
        L.ref_grain_keystream.restype = None
        L.ref_grain_state.argtypes = [u8p, u8p, ctypes.c_uint64, u8p, u8p]
        L.ref_grain_state.restype = None
        L.ref_grain_clock.argtypes = [u8p, u8p, ctypes.c_int]
        L.ref_grain_clock.restype = ctypes.c_int
        L.ref_aes128_encrypt_block.argtypes = [u8p, u8p, u8p]
        L.ref_aes128_encrypt_block.restype = None
        L.ref_aes128_expand_key.argtypes = [u8p, u8p]
        L.ref_aes128_expand_key.restype = None
        L.ref_aes_sbox.argtypes = [ctypes.c_uint8]
        L.ref_aes_sbox.restype = ctypes.c_uint8
        L.ref_aes128_ctr_keystream.argtypes = [u8p, u8p, ctypes.c_uint64, ctypes.c_uint64, u8p]
        L.ref_aes128_ctr_keystream.restype = None
        L.ref_lfsr128_keystream.argtypes = [u8p, ctypes.c_uint64, u8p]
        L.ref_lfsr128_keystream.restype = None
        L.ref_lfsr128_clock.argtypes = [u8p]
        L.ref_lfsr128_clock.restype = ctypes.c_int
        _lib = L
    return _lib


def _buf(b: bytes | bytearray | np.ndarray, n: int):
    a = np.zeros(max(n, 1), dtype=np.uint8)
    src = np.frombuffer(bytes(b), dtype=np.uint8)
    a[: src.size] = src
    return a


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8))


# ------------------------------------------------------------------ MICKEY 2.0
def mickey2_keystream(key: bytes, iv: bytes, iv_bits: int, nbits: int) -> bytes:
    """Keystream of one instance, ``nbits`` bits packed MSB-first."""
    k = _buf(key, 10)
    v = _buf(iv, 10)
    out = np.zeros(max((nbits + 7) // 8, 1), dtype=np.uint8)
    rc = lib().ref_mickey2_keystream(_p(k), _p(v), iv_bits, nbits, _p(out))
    if rc != 0:
        raise ValueError(f"ref_mickey2_keystream: bad iv_bits={iv_bits}")
    return out[: (nbits + 7) // 8].tobytes()


def mickey2_state(key: bytes, iv: bytes, iv_bits: int, extra_clocks: int = 0):
    """(r, s) as uint8[100] 0/1 arrays after init (+ extra keystream clocks)."""
    k = _buf(key, 10)
    v = _buf(iv, 10)
    r = np.zeros(100, dtype=np.uint8)
    s = np.zeros(100, dtype=np.uint8)
    rc = lib().ref_mickey2_state(_p(k), _p(v), iv_bits, extra_clocks, _p(r), _p(s))
    if rc != 0:
        raise ValueError(f"ref_mickey2_state: bad iv_bits={iv_bits}")
    return r, s


def mickey2_clock_kg(r: np.ndarray, s: np.ndarray, mixing: int, input_bit: int):
    r = np.ascontiguousarray(r, dtype=np.uint8).copy()
    s = np.ascontiguousarray(s, dtype=np.uint8).copy()
    lib().ref_mickey2_clock_kg(_p(r), _p(s), int(mixing), int(input_bit))
    return r, s


def mickey2_table(which: str) -> np.ndarray:
    idx = {"RTAPS": 0, "COMP0": 1, "COMP1": 2, "FB0": 3, "FB1": 4}[which]
    return np.array([lib().ref_mickey2_table(idx, i) for i in range(100)], dtype=np.uint8)


def mickey2_keystream_batch(keys: np.ndarray, ivs: np.ndarray, iv_bits: int, nbits: int,
                            threads: int | None = None) -> np.ndarray:
    """Row-major keystreams for n instances: uint8[n, ceil(nbits/8)].

    Instances are independent; each ctypes call releases the GIL, so a thread
    pool runs them on all host cores.  The per-instance arithmetic is the
    unmodified bit-serial oracle above.
    """
    keys = np.ascontiguousarray(keys, dtype=np.uint8)
    ivs = np.ascontiguousarray(ivs, dtype=np.uint8)
    n = keys.shape[0]
    nbytes = (nbits + 7) // 8
    out = np.zeros((n, max(nbytes, 1)), dtype=np.uint8)
    L = lib()
    ivpad = np.zeros((n, 10), dtype=np.uint8)
    ivpad[:, : ivs.shape[1]] = ivs[:, :10]

    def one(i):
        rc = L.ref_mickey2_keystream(_p(keys[i]), _p(ivpad[i]), iv_bits, nbits, _p(out[i]))
        if rc != 0:
            raise ValueError("bad iv_bits")

    threads = threads or os.cpu_count() or 1
    if threads == 1 or n == 1:
        for i in range(n):
            one(i)
    else:
        with ThreadPoolExecutor(max_workers=threads) as ex:
            list(ex.map(one, range(n)))
    return out[:, :nbytes]


# -------------------------------------------------------------------- Grain v1
def grain_keystream(key: bytes, iv: bytes, nbits: int) -> bytes:
    """Grain v1 keystream of one instance, packed LSB-first."""
    k = _buf(key, 10)
    v = _buf(iv, 8)
    out = np.zeros(max((nbits + 7) // 8, 1), dtype=np.uint8)
    lib().ref_grain_keystream(_p(k), _p(v), nbits, _p(out))
    return out[: (nbits + 7) // 8].tobytes()


def grain_state(key: bytes, iv: bytes, extra_clocks: int = 0):
    """(s, b) = (LFSR, NFSR) as uint8[80] 0/1 arrays after init (+ clocks)."""
    k = _buf(key, 10)
    v = _buf(iv, 8)
    s = np.zeros(80, dtype=np.uint8)
    b = np.zeros(80, dtype=np.uint8)
    lib().ref_grain_state(_p(k), _p(v), extra_clocks, _p(s), _p(b))
    return s, b


def grain_clock(s: np.ndarray, b: np.ndarray, init_mode: int):
    s = np.ascontiguousarray(s, dtype=np.uint8).copy()
    b = np.ascontiguousarray(b, dtype=np.uint8).copy()
    z = lib().ref_grain_clock(_p(s), _p(b), int(init_mode))
    return s, b, z


def grain_keystream_batch(keys: np.ndarray, ivs: np.ndarray, nbits: int, threads: int | None = None):
    """Row-major Grain keystreams, uint8[n, ceil(nbits/8)] (LSB-first)."""
    keys = np.ascontiguousarray(keys, dtype=np.uint8)
    ivs = np.ascontiguousarray(ivs, dtype=np.uint8)
    n = keys.shape[0]
    nbytes = (nbits + 7) // 8
    out = np.zeros((n, max(nbytes, 1)), dtype=np.uint8)
    L = lib()

    def one(i):
        L.ref_grain_keystream(_p(keys[i]), _p(ivs[i]), nbits, _p(out[i]))

    threads = threads or os.cpu_count() or 1
    if threads == 1 or n == 1:
        for i in range(n):
            one(i)
    else:
        with ThreadPoolExecutor(max_workers=threads) as ex:
            list(ex.map(one, range(n)))
    return out[:, :nbytes]


# --------------------------------------------------------------- AES-128-CTR
def aes128_encrypt_block(key: bytes, block: bytes) -> bytes:
    k = _buf(key, 16)
    b = _buf(block, 16)
    out = np.zeros(16, dtype=np.uint8)
    lib().ref_aes128_encrypt_block(_p(k), _p(b), _p(out))
    return out.tobytes()


def aes128_expand_key(key: bytes) -> bytes:
    k = _buf(key, 16)
    w = np.zeros(176, dtype=np.uint8)
    lib().ref_aes128_expand_key(_p(k), _p(w))
    return w.tobytes()


def aes_sbox() -> np.ndarray:
    return np.array([lib().ref_aes_sbox(x) for x in range(256)], dtype=np.uint8)


def aes128_ctr_keystream(key: bytes, ctr: bytes, nblocks: int, first_block: int = 0) -> bytes:
    k = _buf(key, 16)
    c = _buf(ctr, 16)
    out = np.zeros(max(16 * nblocks, 1), dtype=np.uint8)
    lib().ref_aes128_ctr_keystream(_p(k), _p(c), first_block, nblocks, _p(out))
    return out[: 16 * nblocks].tobytes()


def aes128_ctr_keystream_batch(key: bytes, ctrs: np.ndarray, nbits: int, first_block: int = 0,
                               threads: int | None = None) -> np.ndarray:
    """Row-major AES-CTR keystreams of n counter streams under one key:
    uint8[n, nbits/8]; nbits must be a multiple of 128."""
    assert nbits % 128 == 0
    k = _buf(key, 16)
    ctrs = np.ascontiguousarray(ctrs, dtype=np.uint8)
    n = ctrs.shape[0]
    out = np.zeros((n, max(nbits // 8, 1)), dtype=np.uint8)
    L = lib()

    def one(i):
        L.ref_aes128_ctr_keystream(_p(k), _p(ctrs[i]), first_block, nbits // 128, _p(out[i]))

    threads = threads or os.cpu_count() or 1
    if threads == 1 or n == 1:
        for i in range(n):
            one(i)
    else:
        with ThreadPoolExecutor(max_workers=threads) as ex:
            list(ex.map(one, range(n)))
    return out[:, : nbits // 8]


# ------------------------------------------------------------- 128-bit LFSR
def lfsr128_keystream(key: bytes, nbits: int) -> bytes:
    k = _buf(key, 16)
    out = np.zeros(max((nbits + 7) // 8, 1), dtype=np.uint8)
    lib().ref_lfsr128_keystream(_p(k), nbits, _p(out))
    return out[: (nbits + 7) // 8].tobytes()


def lfsr128_clock(s: np.ndarray):
    s = np.ascontiguousarray(s, dtype=np.uint8).copy()
    z = lib().ref_lfsr128_clock(_p(s))
    return s, z


def lfsr128_keystream_batch(keys: np.ndarray, nbits: int, threads: int | None = None) -> np.ndarray:
    keys = np.ascontiguousarray(keys, dtype=np.uint8)
    n = keys.shape[0]
    out = np.zeros((n, max((nbits + 7) // 8, 1)), dtype=np.uint8)
    L = lib()

    def one(i):
        L.ref_lfsr128_keystream(_p(keys[i]), nbits, _p(out[i]))

    threads = threads or os.cpu_count() or 1
    if threads == 1 or n == 1:
        for i in range(n):
            one(i)
    else:
        with ThreadPoolExecutor(max_workers=threads) as ex:
            list(ex.map(one, range(n)))
    return out[:, : (nbits + 7) // 8]
