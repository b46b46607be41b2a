"""Thin Python binding of the C ABI in include/bsrng.h (ctypes).

Argument marshalling only: every step of the keystream path runs in the CUDA
kernels of libbsrng.so.  There is no CPU fallback -- if the library is missing
or no sm_100 device is present, construction raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import inputs as _inputs

_PKG = os.path.dirname(os.path.abspath(__file__))
# BSRNG_LIB: an alternative build of the same library (A/B runs of kernel variants)
LIB_PATH = os.environ.get("BSRNG_LIB") or os.path.join(_PKG, "libbsrng.so")

MICKEY2, GRAIN_V1, AES128_CTR, LFSR128 = 1, 2, 3, 4
ROW_MAJOR, SLICED, CHECKSUM = 0, 1, 2
INPUT_HOST, INPUT_DEVICE = 0, 1
OK, EINVAL, ENOMEM, ECUDA, ERANGE, EUNSUPPORTED = 0, -1, -2, -3, -4, -5

CIPHERS = {"mickey2": MICKEY2, "grain": GRAIN_V1, "aes128ctr": AES128_CTR, "lfsr128": LFSR128}
LAYOUTS = {"row_major": ROW_MAJOR, "sliced": SLICED, "checksum": CHECKSUM}
NSTATE = {MICKEY2: 200, GRAIN_V1: 160, AES128_CTR: 128, LFSR128: 128}
DEFAULT_IV_BITS = {MICKEY2: 80, GRAIN_V1: 64, AES128_CTR: 128, LFSR128: 0}

SYMBOLS = [
    "bsrng_create", "bsrng_create_ex", "bsrng_rekey", "bsrng_generate", "bsrng_generate_host",
    "bsrng_out_bytes", "bsrng_num_instances", "bsrng_num_groups", "bsrng_bits_done",
    "bsrng_copy_state", "bsrng_set_option", "bsrng_destroy", "bsrng_last_error",
    "bsrng_launch_count",
]


class BsrngError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"bsrng error {code}: {msg}")
        self.code = code


_lib = None


def lib() -> ctypes.CDLL:
    """Load libbsrng.so (fails loudly if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built: run __graft_entry__.build() "
                          "(no CPU fallback exists)")
    L = ctypes.CDLL(LIB_PATH)
    u8p, vp, u64, u32 = ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32
    L.bsrng_create.argtypes = [ctypes.c_int, u8p, u8p, u64]
    L.bsrng_create.restype = vp
    L.bsrng_create_ex.argtypes = [ctypes.c_int, u8p, u8p, u32, u64, u64, u32, vp]
    L.bsrng_create_ex.restype = vp
    L.bsrng_rekey.argtypes = [vp, u8p, u8p, u32, vp]
    L.bsrng_rekey.restype = ctypes.c_int
    L.bsrng_generate.argtypes = [vp, vp, u64, ctypes.c_int, vp]
    L.bsrng_generate.restype = ctypes.c_int
    L.bsrng_generate_host.argtypes = [vp, vp, u64, ctypes.c_int, vp]
    L.bsrng_generate_host.restype = ctypes.c_int
    L.bsrng_out_bytes.argtypes = [vp, u64, ctypes.c_int]
    L.bsrng_out_bytes.restype = u64
    for f in ("bsrng_num_instances", "bsrng_num_groups", "bsrng_bits_done"):
        getattr(L, f).argtypes = [vp]
        getattr(L, f).restype = u64
    L.bsrng_copy_state.argtypes = [vp, vp, u64]
    L.bsrng_copy_state.restype = ctypes.c_int64
    L.bsrng_set_option.argtypes = [vp, ctypes.c_char_p, ctypes.c_int64]
    L.bsrng_set_option.restype = ctypes.c_int
    L.bsrng_destroy.argtypes = [vp]
    L.bsrng_destroy.restype = None
    L.bsrng_last_error.argtypes = []
    L.bsrng_last_error.restype = ctypes.c_char_p
    L.bsrng_launch_count.argtypes = []
    L.bsrng_launch_count.restype = u64
    _lib = L
    return L


def last_error() -> str:
    return lib().bsrng_last_error().decode()


def launch_count() -> int:
    return int(lib().bsrng_launch_count())


def _check(rc):
    if rc != OK:
        raise BsrngError(rc, last_error())
    return rc


def _stream_ptr(stream):
    if stream is None:
        try:
            import torch
            if torch.cuda.is_available():
                return torch.cuda.current_stream().cuda_stream
        except ImportError:  # pragma: no cover
            pass
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _ptr(x):
    """(pointer, is_device) for a torch tensor, numpy array, bytes or int."""
    if x is None:
        return None, False
    if isinstance(x, int):
        return x, True
    if hasattr(x, "data_ptr") and hasattr(x, "is_cuda"):
        if not x.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return x.data_ptr(), bool(x.is_cuda)
    if isinstance(x, (bytes, bytearray)):
        x = np.frombuffer(bytes(x), dtype=np.uint8)
    if isinstance(x, np.ndarray):
        if not x.flags["C_CONTIGUOUS"]:
            raise ValueError("array must be C-contiguous")
        return x.ctypes.data, False
    raise TypeError(f"unsupported buffer type {type(x)}")


class Generator:
    """One handle = n keyed cipher instances on the current CUDA device."""

    def __init__(self, cipher, keys, ivs, *, iv_bits=None, first_instance=0, stream=None):
        self._h = None
        self.cipher = CIPHERS[cipher] if isinstance(cipher, str) else int(cipher)
        self.iv_bits = DEFAULT_IV_BITS.get(self.cipher, 0) if iv_bits is None else int(iv_bits)
        kp, kdev = _ptr(keys)
        if ivs is not None and getattr(ivs, "size", 1) == 0:
            ivs = None  # no IV (LFSR)
        vp, vdev = _ptr(ivs)
        # AES-128-CTR: ONE key for all instances, n = number of counter blocks
        rows = ivs if self.cipher == AES128_CTR else keys
        n = int(rows.shape[0]) if hasattr(rows, "shape") else 0
        self._keep = (keys, ivs)  # host arrays must outlive the async copy
        flags = INPUT_DEVICE if kdev else INPUT_HOST
        if ivs is not None and vdev != kdev:
            raise ValueError("keys and ivs must both be host or both be device buffers")
        h = lib().bsrng_create_ex(self.cipher, kp, vp, self.iv_bits, n, int(first_instance), flags,
                                  _stream_ptr(stream))
        if not h:
            raise BsrngError(ECUDA, last_error())
        self._h = h
        self.n = n
        self.first_instance = int(first_instance)

    @classmethod
    def from_seed(cls, cipher, n, first_instance=0, seed=_inputs.DEFAULT_SEED, **kw):
        keys, ivs = _inputs.make_inputs(cipher, n, first_instance, seed)
        if cipher in ("aes128ctr", AES128_CTR):
            keys = _inputs.aes_key(seed)
        return cls(cipher, keys, ivs, first_instance=first_instance, **kw)

    # -- properties -------------------------------------------------------
    @property
    def handle(self):
        return self._h

    @property
    def groups(self):
        return int(lib().bsrng_num_groups(self._h))

    @property
    def bits_done(self):
        return int(lib().bsrng_bits_done(self._h))

    def out_bytes(self, bits, layout):
        return int(lib().bsrng_out_bytes(self._h, int(bits), _layout(layout)))

    # -- operations -------------------------------------------------------
    def rekey(self, keys, ivs, stream=None):
        kp, kdev = _ptr(keys)
        if ivs is not None and getattr(ivs, "size", 1) == 0:
            ivs = None
        vp, vdev = _ptr(ivs)
        if ivs is not None and vdev != kdev:
            raise ValueError("keys and ivs must both be host or both be device buffers")
        self._keep = (keys, ivs)
        _check(lib().bsrng_rekey(self._h, kp, vp, INPUT_DEVICE if kdev else INPUT_HOST,
                                 _stream_ptr(stream)))

    def generate(self, out, bits, layout="row_major", stream=None):
        """Enqueue generation into device buffer `out` (torch CUDA tensor or pointer)."""
        op, dev = _ptr(out)
        if not dev:
            raise ValueError("generate() needs a device buffer; use generate_host()")
        if hasattr(out, "numel"):
            need = self.out_bytes(bits, layout)
            if out.numel() * out.element_size() < need:
                raise ValueError(f"out too small: need {need} bytes")
        _check(lib().bsrng_generate(self._h, op, int(bits), _layout(layout), _stream_ptr(stream)))

    def generate_host(self, bits, layout="row_major", stream=None) -> np.ndarray:
        """Generate and copy back to host.  Shapes: ROW_MAJOR uint8[n, bits/8],
        SLICED uint32[bits, G], CHECKSUM uint64 scalar array."""
        lay = _layout(layout)
        if lay == ROW_MAJOR:
            out = np.zeros((self.n, int(bits) // 8), dtype=np.uint8)
        elif lay == SLICED:
            out = np.zeros((int(bits), self.groups), dtype=np.uint32)
        else:
            out = np.zeros(1, dtype=np.uint64)
        _check(lib().bsrng_generate_host(self._h, out.ctypes.data, int(bits), lay, _stream_ptr(stream)))
        return out

    def copy_state(self) -> np.ndarray:
        ns = NSTATE[self.cipher]
        out = np.zeros((ns, self.groups), dtype=np.uint32)
        rc = lib().bsrng_copy_state(self._h, out.ctypes.data, out.size)
        if rc < 0:
            raise BsrngError(int(rc), last_error())
        return out

    def set_option(self, key, value):
        _check(lib().bsrng_set_option(self._h, key.encode(), int(value)))

    def close(self):
        if self._h:
            lib().bsrng_destroy(self._h)
            self._h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _layout(layout):
    return LAYOUTS[layout] if isinstance(layout, str) else int(layout)
