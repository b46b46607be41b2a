"""GPU parity: bitsliced AES-128-CTR through the C
ABI vs the byte-oriented oracle (oracle/aes_ref.c).  Bar: bit-exact.

All instances share one key; instance i's keystream is
E_K(ctr_i) || E_K(ctr_i + 1) || ... (128-bit big-endian counter)."""
import numpy as np
import pytest

import oracle
from conftest import read_golden
from helpers import checksum, to_sliced

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng, inputs  # noqa: E402


def _gen(n, first=0, **kw):
    _, ctrs = inputs.make_inputs("aes128ctr", n, first)
    key = inputs.aes_key()
    return bsrng.Generator("aes128ctr", key, ctrs, first_instance=first, **kw), key, ctrs


def test_sp800_38a_f51_on_gpu():
    key = np.frombuffer(bytes.fromhex("2b7e151628aed2a6abf7158809cf4f3c"), np.uint8).copy()
    ctr = np.frombuffer(bytes.fromhex("f0f1f2f3f4f5f6f7f8f9fafbfcfdfeff"), np.uint8).reshape(1, 16).copy()
    row = [r for r in read_golden("aes128_vectors.txt") if r[0] == "ctr"][0]
    with bsrng.Generator("aes128ctr", key, ctr) as g:
        got = g.generate_host(256, "row_major")[0].tobytes().hex()
    assert got == row[3]


@pytest.mark.parametrize("seg", [0, 256, 512])
def test_ragged_all_layouts(seg):
    n, bits = 32 * 37 + 13, 1536
    g0, key, ctrs = _gen(n)
    want = oracle.aes128_ctr_keystream_batch(bytes(key), ctrs, bits)
    for layout in ("row_major", "sliced", "checksum"):
        g, _, _ = _gen(n)
        if seg:
            g.set_option("seg_clocks", seg)
        got = g.generate_host(bits, layout)
        if layout == "row_major":
            assert np.array_equal(got, want)
        elif layout == "sliced":
            assert np.array_equal(got, to_sliced(want))
        else:
            assert int(got[0]) == checksum(to_sliced(want))


def test_concatenation_and_counter_wrap():
    n = 64
    _, ctrs = inputs.make_inputs("aes128ctr", n)
    ctrs = ctrs.copy()
    ctrs[5] = np.frombuffer(bytes([0xFF] * 15 + [0xFD]), np.uint8)  # wraps after 3 blocks
    ctrs[6, 8:] = 0xFF                                              # carry out of the low 64 bits
    key = inputs.aes_key()
    g = bsrng.Generator("aes128ctr", key, ctrs)
    a = g.generate_host(384, "row_major")
    b = g.generate_host(640, "sliced")
    c = g.generate_host(256, "checksum")
    want = oracle.aes128_ctr_keystream_batch(bytes(key), ctrs, 384 + 640 + 256)
    assert np.array_equal(a, want[:, :48])
    assert np.array_equal(b, to_sliced(want[:, 48:128]))
    assert int(c[0]) == checksum(to_sliced(want[:, 128:]), t0=1024)


def test_device_inputs_and_errors():
    n = 96
    _, ctrs = inputs.make_inputs("aes128ctr", n)
    key = inputs.aes_key()
    g = bsrng.Generator("aes128ctr", torch.from_numpy(key).cuda(), torch.from_numpy(ctrs).cuda())
    want = oracle.aes128_ctr_keystream_batch(bytes(key), ctrs, 512)
    assert np.array_equal(g.generate_host(512, "row_major"), want)
    buf = torch.empty(1 << 16, dtype=torch.uint8, device="cuda")
    with pytest.raises(bsrng.BsrngError) as e:
        g.generate(buf, 96, "sliced")  # not a multiple of 128
    assert e.value.code == bsrng.EINVAL


def test_large_sampled():
    """2^22 counter streams x 2048 bits; sampled rows vs the oracle."""
    n, bits = 1 << 22, 2048
    g, key, ctrs = _gen(n)
    out = torch.empty(g.out_bytes(bits, "row_major"), dtype=torch.uint8, device="cuda")
    g.generate(out, bits, "row_major")
    torch.cuda.synchronize()
    rows = out.cpu().numpy().reshape(n, bits // 8)
    idx = np.unique(np.concatenate([np.random.default_rng(3).integers(0, n, 128), [0, 31, 32, n - 1]]))
    want = oracle.aes128_ctr_keystream_batch(bytes(key), ctrs[idx], bits)
    assert np.array_equal(rows[idx], want)


@pytest.mark.parametrize("bits,seg", [(4096, 0), (4096 * 3 + 1024, 0), (4096 * 5, 4096), (8192, 8192)])
def test_rowmajor_block_lanes(bits, seg):
    """ROW_MAJOR calls with >= 32 blocks per instance take the block-lane
    kernel (lanes = consecutive blocks of one instance); partial last
    encryptions, segments and a preceding call (block offset) included."""
    n = 32 * 5 + 3
    _, ctrs = inputs.make_inputs("aes128ctr", n)
    ctrs = ctrs.copy()
    ctrs[7] = np.frombuffer(bytes([0xFF] * 15 + [0xF0]), np.uint8)   # 128-bit wrap inside a 32-block tile
    ctrs[8, 8:] = 0xFF
    ctrs[8, 15] = 0xE1                                               # carry out of the low 64 bits
    key = inputs.aes_key()
    g = bsrng.Generator("aes128ctr", key, ctrs)
    if seg:
        g.set_option("seg_clocks", seg)
    pre = g.generate_host(384, "checksum")  # 3 blocks consumed first
    got = g.generate_host(bits, "row_major")
    want = oracle.aes128_ctr_keystream_batch(bytes(key), ctrs, bits, first_block=3)
    assert np.array_equal(got, want)
    assert int(pre[0]) == checksum(to_sliced(oracle.aes128_ctr_keystream_batch(bytes(key), ctrs, 384)))


@pytest.mark.parametrize("bits", [4480, 8192 + 128, 4096 + 31 * 128, 4096])
def test_rowmajor_lanes_plus_remainder(bits):
    """ROW_MAJOR calls of >= 32 blocks: whole 32-block encryptions in the
    block-lane kernel, the < 32-block remainder in the instance-sliced kernel
    writing the rows' last bytes (paper shape: 35 blocks = 4480 bits); two
    consecutive calls continue the counters."""
    n = 32 * 9 + 5
    g, key, ctrs = _gen(n)
    want = oracle.aes128_ctr_keystream_batch(bytes(key), ctrs, 2 * bits)
    got1 = g.generate_host(bits, "row_major")
    got2 = g.generate_host(bits, "row_major")
    assert np.array_equal(got1, want[:, :bits // 8])
    assert np.array_equal(got2, want[:, bits // 8:])


@pytest.mark.parametrize("device_inputs", [False, True])
@pytest.mark.parametrize("bits", [4096 + 384, 4096 + 31 * 128, 8192 + 128])
def test_rowmajor_remainder_pairs_carries(bits, device_inputs):
    """Block-lane ROW_MAJOR calls with a < 32-block remainder per row (the
    instance-sliced kernel writes the rows' last blocks): counters whose block
    index carries through the low 32 and 64 bits and wraps at 2^128 inside the
    remainder, a second call (block indices offset by the first call), ragged
    n, host and device-resident counters."""
    n = 32 * 7 + 19
    _, ctrs = inputs.make_inputs("aes128ctr", n, seed=77)
    ctrs = ctrs.copy()
    ctrs[3] = np.frombuffer(bytes([0xFF] * 16), np.uint8)                        # wraps at the first block
    ctrs[4, 12:] = 0xFF                                                          # low word carries
    ctrs[5, 8:] = 0xFF
    ctrs[5, 15] = 0xDF                                                           # carry out of 64 bits mid-row
    ctrs[33] = np.frombuffer(bytes([0xFF] * 15 + [0xD8]), np.uint8)              # 128-bit wrap inside the remainder
    key = inputs.aes_key(5)
    if device_inputs:
        g = bsrng.Generator("aes128ctr", torch.from_numpy(key).cuda(), torch.from_numpy(ctrs).cuda())
    else:
        g = bsrng.Generator("aes128ctr", key, ctrs)
    want = oracle.aes128_ctr_keystream_batch(bytes(key), ctrs, 2 * bits)
    for call in range(2):
        got = g.generate_host(bits, "row_major")
        assert np.array_equal(got, want[:, call * bits // 8:(call + 1) * bits // 8]), call
