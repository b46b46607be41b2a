"""GPU tests of the C-ABI contract (include/bsrng.h), called
through ctypes (paper_conf_icppw_monfaredhkzrg20_b200/bsrng.py marshals only):

* host inputs may be overwritten as soon as bsrng_rekey returns (handle-owned
  pinned staging), also when the caller's own buffers are pinned;
* bsrng_rekey never waits on the host (AES-128-CTR included: round keys reach
  the handle's constant slot by a stream-ordered copy);
* any MICKEY IV length 0..80 (the spec's range; sec. 2.3.1),
  bit-exact vs the oracle;
* a stream of another device is EINVAL;
* a device-input AES-128-CTR rekey followed by block-lane ROW_MAJOR calls
  (the counters come from the sliced state);
* a call of more than 2^32 bits per instance runs every clock (the kernels
  count an item's clocks in 32 bits; the launcher splits such calls).
"""
import ctypes

import numpy as np
import pytest

import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng, inputs  # noqa: E402


def _want(cipher, keys, ivs, bits, iv_bits=80):
    if cipher == "mickey2":
        return oracle.mickey2_keystream_batch(keys, ivs, iv_bits, bits)
    if cipher == "grain":
        return oracle.grain_keystream_batch(keys, ivs, bits)
    if cipher == "lfsr128":
        return oracle.lfsr128_keystream_batch(keys, bits)
    return oracle.aes128_ctr_keystream_batch(bytes(inputs.aes_key()), ivs, bits)


@pytest.mark.parametrize("cipher", ["mickey2", "grain", "aes128ctr", "lfsr128"])
@pytest.mark.parametrize("pinned", [False, True])
def test_host_inputs_reusable_on_return(cipher, pinned):
    """Overwrite the host key/IV arrays right after bsrng_rekey returns, while
    the stream is still busy (a sleep kernel queued first): the keystream
    still follows the ORIGINAL inputs."""
    n, bits = 32 * 9 + 5, 512
    keys, ivs = inputs.make_inputs(cipher, n, seed=31)
    if cipher == "aes128ctr":
        keys = inputs.aes_key(31)
    keys = np.ascontiguousarray(keys)
    want = (oracle.aes128_ctr_keystream_batch(bytes(keys), ivs, bits) if cipher == "aes128ctr"
            else _want(cipher, keys, ivs, bits))
    k0, v0 = inputs.make_inputs(cipher, n, seed=1)
    g = bsrng.Generator(cipher, inputs.aes_key(1) if cipher == "aes128ctr" else k0,
                        None if cipher == "lfsr128" else v0)
    kt = torch.from_numpy(keys.reshape(-1).copy())
    vt = torch.from_numpy(ivs.reshape(-1).copy()) if cipher != "lfsr128" else None
    if pinned:
        kt = kt.pin_memory()
        vt = vt.pin_memory() if vt is not None else None
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        torch.cuda._sleep(50_000_000)  # ~25 ms of GPU time ahead of the copy
    L = bsrng.lib()
    rc = L.bsrng_rekey(g.handle, kt.data_ptr(), vt.data_ptr() if vt is not None else None,
                       bsrng.INPUT_HOST, st.cuda_stream)
    assert rc == bsrng.OK, bsrng.last_error()
    kt.fill_(0xA5)
    if vt is not None:
        vt.fill_(0x5A)
    out = torch.empty(g.out_bytes(bits, "row_major"), dtype=torch.uint8, device="cuda")
    g.generate(out, bits, "row_major", stream=st)
    st.synchronize()
    assert np.array_equal(out.cpu().numpy().reshape(n, bits // 8), want)


@pytest.mark.parametrize("cipher", ["mickey2", "grain", "aes128ctr", "lfsr128"])
def test_rekey_is_asynchronous(cipher):
    """bsrng_rekey returns while the stream is still running an earlier
    kernel: no host synchronisation on the rekey path."""
    n = 32 * 64
    keys, ivs = inputs.make_inputs(cipher, n)
    k = inputs.aes_key() if cipher == "aes128ctr" else keys
    v = None if cipher == "lfsr128" else ivs
    g = bsrng.Generator(cipher, k, v)
    kd = torch.from_numpy(np.ascontiguousarray(k).reshape(-1).copy()).cuda()
    vd = torch.from_numpy(ivs.reshape(-1).copy()).cuda() if v is not None else None
    st = torch.cuda.Stream()
    torch.cuda.synchronize()
    with torch.cuda.stream(st):
        torch.cuda._sleep(200_000_000)  # ~100 ms
    g.rekey(kd, vd if vd is not None else None, stream=st)
    assert not st.query(), "rekey waited for the stream"
    st.synchronize()
    assert np.array_equal(g.generate_host(256, "row_major"), _want(cipher, keys, ivs, 256))


@pytest.mark.parametrize("iv_bits", [1, 7, 13, 79])
@pytest.mark.parametrize("init_fused", [1, 0])
def test_mickey_any_iv_length(iv_bits, init_fused):
    """IV lengths that are not whole bytes (and not multiples of the 4-clock
    init block): bit-exact keystream and post-init state vs the oracle."""
    n, bits = 70, 1024
    keys, ivs = inputs.make_inputs("mickey2", n, seed=9)
    want = _want("mickey2", keys, ivs, bits, iv_bits)
    g = bsrng.Generator("mickey2", keys, ivs, iv_bits=iv_bits)
    if not init_fused:
        g.set_option("init_fused", 0)
        g.rekey(keys, ivs)
    st = g.copy_state()
    for i in (0, 33, n - 1):
        r, s = oracle.mickey2_state(bytes(keys[i]), bytes(ivs[i]), iv_bits, 0)
        gi, j = divmod(i, 32)
        assert np.array_equal((st[:100, gi] >> np.uint32(j)) & 1, r.astype(np.uint32)), i
        assert np.array_equal((st[100:, gi] >> np.uint32(j)) & 1, s.astype(np.uint32)), i
    assert np.array_equal(g.generate_host(bits, "row_major"), want)


def test_mickey_iv_bits_out_of_range():
    keys, ivs = inputs.make_inputs("mickey2", 32)
    with pytest.raises(bsrng.BsrngError) as e:
        bsrng.Generator("mickey2", keys, ivs, iv_bits=81)
    assert e.value.code == bsrng.ECUDA  # create returns NULL; reason in last_error
    assert "iv_bits" in bsrng.last_error()


def test_stream_of_the_handles_device_is_accepted():
    keys, ivs = inputs.make_inputs("mickey2", 64)
    g = bsrng.Generator("mickey2", keys, ivs)
    st = torch.cuda.Stream(device=0)
    buf = torch.zeros(1, dtype=torch.int64, device="cuda:0")
    g.generate(buf, 256, "checksum", stream=st)
    st.synchronize()
    # the special handles cudaStreamLegacy (1) and cudaStreamPerThread (2)
    L = bsrng.lib()
    for special in (1, 2):
        assert L.bsrng_generate(g.handle, buf.data_ptr(), 256, bsrng.CHECKSUM, special) == bsrng.OK, bsrng.last_error()
    torch.cuda.synchronize()


@pytest.mark.skipif(not torch.cuda.is_available() or torch.cuda.device_count() < 2,
                    reason="needs a second GPU for a foreign stream")
def test_stream_of_another_device_is_einval():
    keys, ivs = inputs.make_inputs("mickey2", 64)
    with torch.cuda.device(0):
        g = bsrng.Generator("mickey2", keys, ivs)
    st1 = torch.cuda.Stream(device=1)
    buf = torch.zeros(1, dtype=torch.int64, device="cuda:0")
    L = bsrng.lib()
    assert L.bsrng_generate(g.handle, buf.data_ptr(), 256, bsrng.CHECKSUM, st1.cuda_stream) == bsrng.EINVAL
    assert "device" in bsrng.last_error()
    kd = torch.from_numpy(keys).cuda(0)
    vd = torch.from_numpy(ivs).cuda(0)
    assert L.bsrng_rekey(g.handle, kd.data_ptr(), vd.data_ptr(), bsrng.INPUT_DEVICE, st1.cuda_stream) == bsrng.EINVAL
    out = np.zeros(1, np.uint64)
    assert L.bsrng_generate_host(g.handle, out.ctypes.data, 256, bsrng.CHECKSUM, st1.cuda_stream) == bsrng.EINVAL


@pytest.mark.parametrize("bits", [4096, 4480, 8192 + 384])
def test_aes_device_input_rowmajor_lanes(bits):
    """Device-resident counters read in place by the init kernel, then
    ROW_MAJOR calls of >= 32 blocks (block-lane kernel + sliced remainder),
    two rekeys in a row and two calls each."""
    n = 32 * 40 + 9
    g = None
    for seed in (41, 42):
        _, ctr = inputs.make_inputs("aes128ctr", n, seed=seed)
        key = inputs.aes_key(seed)
        want = oracle.aes128_ctr_keystream_batch(bytes(key), ctr, 2 * bits)
        kd = torch.from_numpy(np.frombuffer(bytes(key), np.uint8).copy()).cuda()
        cd = torch.from_numpy(ctr.copy()).cuda()
        if g is None:
            g = bsrng.Generator("aes128ctr", kd, cd)
        else:
            g.rekey(kd, cd)
        for call in range(2):
            out = torch.empty(g.out_bytes(bits, "row_major"), dtype=torch.uint8, device="cuda")
            g.generate(out, bits, "row_major")
            torch.cuda.synchronize()
            got = out.cpu().numpy().reshape(n, bits // 8)
            assert np.array_equal(got, want[:, call * bits // 8:(call + 1) * bits // 8]), (seed, call)


def test_call_longer_than_2_32_bits():
    """One CHECKSUM call of 2^32 + 4096 bits per instance must run every clock:
    the state afterwards equals the state after the same bits in five
    shorter calls (the LFSR: 2.5 LOP3 per clock keeps this ~10 s)."""
    n = 64
    keys, _ = inputs.make_inputs("lfsr128", n)
    total = (1 << 32) + 4096
    one = bsrng.Generator("lfsr128", keys, None)
    cs = torch.zeros(1, dtype=torch.int64, device="cuda")
    one.generate(cs, total, "checksum")
    torch.cuda.synchronize()
    many = bsrng.Generator("lfsr128", keys, None)
    left = total
    while left:
        c = min(left, 1 << 30)
        many.generate(cs, c, "checksum")
        left -= c
    torch.cuda.synchronize()
    assert one.bits_done == many.bits_done == total
    assert np.array_equal(one.copy_state(), many.copy_state())
    # and the sliced call path (sched = 0) splits too
    g0 = bsrng.Generator("lfsr128", keys, None)
    g0.set_option("sched", 0)
    g0.generate(cs, total, "checksum")
    torch.cuda.synchronize()
    assert np.array_equal(g0.copy_state(), many.copy_state())
