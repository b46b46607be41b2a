"""CPU-side checks of the C ABI boundary (no compute calls without a GPU):
libbsrng.so loads and exports every symbol include/bsrng.h declares, and
argument validation that happens before any device work."""
import ctypes
import os
import re

import pytest

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    txt = open(os.path.join(ROOT, "include", "bsrng.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(bsrng_\w+)\s*\(", txt)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_icppw_monfaredhkzrg20_b200 import build
    build.build()
    return bsrng.lib()


def test_header_declares_expected(L):
    assert set(_declared()) == set(bsrng.SYMBOLS)


def test_library_exports_every_declared_symbol(L):
    for name in _declared():
        assert hasattr(L, name), name
        assert ctypes.cast(getattr(L, name), ctypes.c_void_p).value


def test_create_validation(L):
    k = (ctypes.c_uint8 * 20)()
    assert L.bsrng_create(bsrng.MICKEY2, None, None, 1) is None
    assert "NULL" in bsrng.last_error()
    assert L.bsrng_create(bsrng.MICKEY2, ctypes.addressof(k), ctypes.addressof(k), 0) is None
    assert "n_instances" in bsrng.last_error()
    assert L.bsrng_create(99, ctypes.addressof(k), ctypes.addressof(k), 1) is None
    assert L.bsrng_create_ex(bsrng.MICKEY2, ctypes.addressof(k), ctypes.addressof(k), 81, 1, 0, 0, None) is None
    assert "iv_bits" in bsrng.last_error()
    assert L.bsrng_create_ex(bsrng.MICKEY2, ctypes.addressof(k), ctypes.addressof(k), 80, 1, 5, 0, None) is None
    assert "multiple of 32" in bsrng.last_error()


def test_null_handle_calls(L):
    assert L.bsrng_generate(None, None, 32, 0, None) == bsrng.EINVAL
    assert L.bsrng_generate_host(None, None, 32, 0, None) == bsrng.EINVAL
    assert L.bsrng_rekey(None, None, None, 0, None) == bsrng.EINVAL
    assert L.bsrng_out_bytes(None, 32, 0) == 0
    assert L.bsrng_num_instances(None) == 0
    assert L.bsrng_copy_state(None, None, 0) == bsrng.EINVAL
    assert L.bsrng_set_option(None, b"sched", 1) == bsrng.EINVAL
    L.bsrng_destroy(None)  # NULL-safe


def test_no_cpu_fallback_without_gpu(L):
    """On a box without a usable device, create fails loudly (ECUDA)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    k = (ctypes.c_uint8 * 20)()
    assert L.bsrng_create(bsrng.MICKEY2, ctypes.addressof(k), ctypes.addressof(k), 1) is None
    assert bsrng.last_error()
