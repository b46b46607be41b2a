"""GPU tests of the C ABI surface beyond single-cipher parity: edge sizes,
tuning options (every variant must stay bit-exact), concurrent handles on
separate streams, chunked host generation, and the 2^40 limit boundary."""
import numpy as np
import pytest

import oracle
from helpers import checksum, to_sliced

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng, inputs  # noqa: E402


def _want(cipher, keys, ivs, bits, first_block=0):
    if cipher == "mickey2":
        return oracle.mickey2_keystream_batch(keys, ivs, 80, bits)
    if cipher == "grain":
        return oracle.grain_keystream_batch(keys, ivs, bits)
    if cipher == "lfsr128":
        return oracle.lfsr128_keystream_batch(keys, bits)
    return oracle.aes128_ctr_keystream_batch(bytes(inputs.aes_key()), ivs, bits, first_block=first_block)


def _gen(cipher, keys, ivs, **kw):
    if cipher == "aes128ctr":
        return bsrng.Generator(cipher, inputs.aes_key(), ivs, **kw)
    return bsrng.Generator(cipher, keys, None if cipher == "lfsr128" else ivs, **kw)


@pytest.mark.parametrize("cipher", ["mickey2", "grain", "aes128ctr"])
def test_single_instance(cipher):
    keys, ivs = inputs.make_inputs(cipher, 1)
    want = _want(cipher, keys, ivs, 512)
    g = _gen(cipher, keys, ivs)
    assert np.array_equal(g.generate_host(512, "row_major"), want)
    sl = _gen(cipher, keys, ivs).generate_host(512, "sliced")
    assert np.array_equal(sl, to_sliced(want, msb_first=cipher != "grain"))
    assert np.all((sl >> np.uint32(1)) == 0)


@pytest.mark.parametrize("cipher", ["mickey2", "grain", "aes128ctr"])
def test_zero_bits_is_noop(cipher):
    keys, ivs = inputs.make_inputs(cipher, 40)
    g = _gen(cipher, keys, ivs)
    buf = torch.zeros(64, dtype=torch.uint8, device="cuda")
    g.generate(buf, 0, "row_major")
    assert g.bits_done == 0
    assert np.array_equal(g.generate_host(256, "row_major"), _want(cipher, keys, ivs, 256))


@pytest.mark.parametrize("cipher,opts", [
    ("mickey2", {"unroll": 4}), ("mickey2", {"sched": 0}),
    ("mickey2", {"ctas_per_sm": 2}), ("mickey2", {"rm_ws": 0}), ("mickey2", {"rm_ws": 1, "seg_clocks": 512}),
    ("mickey2", {"rm_ws": 1}), ("mickey2", {"rm_ws": 0, "rm_tmem": 0}),
    ("mickey2", {"rm_ws": 0, "rm_tmem": 1, "seg_clocks": 384}),
    ("grain", {"unroll": 16}), ("grain", {"rm_ws": 1}), ("grain", {"sched": 0}),
    ("grain", {"ctas_per_sm": 1, "seg_clocks": 256}), ("grain", {"rm_ws": 0, "ctas_per_sm": 1, "seg_clocks": 256}),
    ("grain", {"rm_ws": 0, "rm_tmem": 0}), ("grain", {"rm_ws": 0, "rm_tmem": 0, "unroll": 16}),
    ("grain", {"rm_ws": 0, "rm_tmem": 0, "ctas_per_sm": 2, "seg_clocks": 384}),
    ("mickey2", {"rm_ws": 0, "rm_tmem": 0}), ("mickey2", {"rm_ws": 0, "rm_tmem": 0, "seg_clocks": 160}),
    ("aes128ctr", {"ctas_per_sm": 1}), ("aes128ctr", {"rm_ws": 0}), ("aes128ctr", {"seg_clocks": 4096}),
    ("lfsr128", {}), ("lfsr128", {"rm_ws": 1, "seg_clocks": 512}), ("lfsr128", {"seg_clocks": 1536}),
    ("lfsr128", {"rm_ws": 2}), ("lfsr128", {"rm_ws": 2, "seg_clocks": 1024}), ("lfsr128", {"rm_ws": 2, "seg_clocks": 3072}),
    ("lfsr128", {"rm_ws": 2, "unroll": 16, "seg_clocks": 2048}),
])
def test_options_stay_bit_exact(cipher, opts):
    # 41 warp-units: MICKEY / Grain ROW_MAJOR default to the writer-warp kernel
    # here, rm_ws = 0 selects the plain kernel
    n, bits = 32 * 40 + 9, 8192
    keys, ivs = inputs.make_inputs(cipher, n)
    want = _want(cipher, keys, ivs, bits)
    for layout in ("row_major", "sliced", "checksum"):
        g = _gen(cipher, keys, ivs)
        for k, v in opts.items():
            g.set_option(k, v)
        got = g.generate_host(bits, layout)
        sl = to_sliced(want, msb_first=cipher != "grain")
        if layout == "row_major":
            assert np.array_equal(got, want), layout
        elif layout == "sliced":
            assert np.array_equal(got, sl), layout
        else:
            assert int(got[0]) == checksum(sl), layout


def test_option_validation():
    keys, ivs = inputs.make_inputs("grain", 32)
    g = bsrng.Generator("grain", keys, ivs)
    for k, v in (("unroll", 4), ("unroll", 8), ("sched", 2), ("seg_clocks", 33), ("ctas_per_sm", 99), ("rm_ws", 5), ("rm_ws", 3),
                 ("rm_slots", 4), ("rm_zreg", 0), ("rm_tmem", 2), ("rm_tma", 2), ("rm_dbl", 2), ("rm_phase", 2), ("rm_phase", -2), ("init_fused", 2)):
        with pytest.raises(bsrng.BsrngError) as e:
            g.set_option(k, v)
        assert e.value.code == bsrng.EINVAL


def test_concurrent_handles_on_streams():
    n, bits = 32 * 64, 2048
    handles, outs, wants = [], [], []
    streams = [torch.cuda.Stream() for _ in range(3)]
    for i, cipher in enumerate(("mickey2", "grain", "aes128ctr")):
        keys, ivs = inputs.make_inputs(cipher, n, seed=100 + i)
        if cipher == "aes128ctr":
            g = bsrng.Generator(cipher, inputs.aes_key(100 + i), ivs)
            want = oracle.aes128_ctr_keystream_batch(bytes(inputs.aes_key(100 + i)), ivs, bits)
        else:
            g = bsrng.Generator(cipher, keys, ivs)
            want = _want(cipher, keys, ivs, bits)
        out = torch.empty(g.out_bytes(bits, "row_major"), dtype=torch.uint8, device="cuda")
        handles.append(g)
        outs.append(out)
        wants.append(want)
    for g, out, st in zip(handles, outs, streams):
        g.generate(out, bits, "row_major", stream=st)
    torch.cuda.synchronize()
    for out, want in zip(outs, wants):
        assert np.array_equal(out.cpu().numpy().reshape(n, bits // 8), want)


def test_generate_host_chunks_rows():
    """ROW_MAJOR host output larger than the 1 GiB device bounce buffer is
    produced in column chunks (cudaMemcpy2D into the host rows)."""
    n, bits = 1 << 20, 1 << 14  # 2 GiB of keystream
    keys, ivs = inputs.make_inputs("grain", n)
    g = bsrng.Generator("grain", keys, ivs)
    rows = g.generate_host(bits, "row_major")
    idx = np.array([0, 1, 12345, n - 1])
    assert np.array_equal(rows[idx], oracle.grain_keystream_batch(keys[idx], ivs[idx], bits))


def test_mickey_2_40_limit_boundary():
    keys, ivs = inputs.make_inputs("mickey2", 32)
    g = bsrng.Generator("mickey2", keys, ivs)
    buf = torch.empty(8, dtype=torch.int64, device="cuda")
    with pytest.raises(bsrng.BsrngError) as e:
        g.generate(buf, (1 << 40) + 32, "checksum")
    assert e.value.code == bsrng.ERANGE
    assert g.bits_done == 0


@pytest.mark.parametrize("cipher,opts,bits", [
    ("grain", {"rm_ws": 0, "rm_tmem": 1}, 8192),
    ("grain", {"rm_ws": 0, "rm_tmem": 1}, 4416),                      # 552 B rows: 8 B-aligned flushes
    ("grain", {"rm_ws": 0, "rm_tmem": 1, "seg_clocks": 160}, 2080),   # partial slots at segment ends
    ("grain", {"rm_ws": 0, "rm_tmem": 1, "unroll": 16}, 4128),
    ("grain", {"rm_ws": 0, "rm_tmem": 1, "sched": 0}, 2048),
    ("grain", {"rm_ws": 0, "rm_tmem": 1, "ctas_per_sm": 2, "seg_clocks": 512}, 4096),
    ("mickey2", {"rm_ws": 0, "rm_tmem": 1}, 4416),
    ("mickey2", {"rm_ws": 0, "rm_tmem": 1, "seg_clocks": 96}, 1024),
    ("grain", {"rm_ws": 0, "rm_tmem": 1, "rm_tma": 0}, 8192),        # 8 B global-store flush instead of TMA
    ("mickey2", {"rm_ws": 0, "rm_tmem": 1}, 8192),        # TMA flush (1 KB rows) for warp 0, 8 B for warp 1
    ("grain", {"rm_ws": 0, "rm_tmem": 1, "rm_tma": 0}, 4416 + 256),  # double-buffered staging, progressive flush
    ("mickey2", {"rm_ws": 0, "rm_tmem": 1, "rm_tma": 0}, 2048 + 96),  # ... item ends mid-period
    ("grain", {"rm_ws": 0, "rm_tmem": 1, "rm_dbl": 0}, 4416),          # single buffer
    ("grain", {"rm_ws": 0, "rm_wide": 1}, 8192),                      # 64 B staging, whole 512-clock flushes
    ("grain", {"rm_ws": 0, "rm_wide": 1}, 4416),                      # 552 B rows: word-by-word flushes
    ("grain", {"rm_ws": 0, "rm_wide": 1, "seg_clocks": 160}, 2080),   # partial periods at segment ends
    ("mickey2", {"rm_ws": 0, "rm_wide": 1}, 1024 + 512 + 96),
    ("grain", {"rm_ws": 0, "rm_wide": 1, "unroll": 16, "seg_clocks": 1024}, 4096),
    ("grain", {"rm_ws": 0, "rm_l2last": 0}, 8192),                     # evict-first TMA flush
    ("grain", {"rm_ws": 0, "rm_l2last": 0, "rm_tma": 0}, 8192),        # evict-first 8 B sector flush
    ("grain", {"rm_ws": 1}, 4416),                         # writer warp, 552 B rows (STG.64 pieces)
    ("grain", {"rm_ws": 1, "seg_clocks": 512}, 4096 + 1024),
    ("grain", {"rm_ws": 1, "rm_phase": 0}, 4416),         # 552 B rows, all units flush in the same block
    ("grain", {"rm_ws": 1, "rm_phase": 1}, 8192),         # staggered flush periods on 16 B-aligned rows
    ("grain", {"rm_ws": 1, "rm_phase": 1, "seg_clocks": 1056}, 4416 + 96),  # ... and mid-period item starts
    ("mickey2", {"rm_ws": 1, "rm_phase": 1}, 2048 + 96),
    ("mickey2", {"rm_ws": 1}, 4416),
    # LFSR writer-warp kernel: 128-clock period bodies plus per-clock remainders
    ("lfsr128", {}, 8192),
    ("lfsr128", {}, 4416),                                # 34.5 periods; 552 B rows
    ("lfsr128", {"seg_clocks": 512}, 4096 + 1024 + 96),   # items of 4 periods, remainder block
    ("lfsr128", {"seg_clocks": 1056}, 3168 + 32),         # items of 33 blocks: mid-flush-period starts
])
def test_rm_tmem_staging_bit_exact(cipher, opts, bits):
    """ROW_MAJOR with the row segments staged in tensor memory (TMEM) instead
    of shared memory: every flush path (16 B, 8 B, partial words) bit-exact.
    n = 1289 is 41 warp-units, fewer than the SMSPs, where MICKEY and Grain
    default to the writer-warp kernel; rm_ws = 0 selects the plain kernel's
    staging variants."""
    n = 32 * 40 + 9
    keys, ivs = inputs.make_inputs(cipher, n)
    want = _want(cipher, keys, ivs, bits)
    g = _gen(cipher, keys, ivs)
    for k, v in opts.items():
        g.set_option(k, v)
    got = g.generate_host(bits, "row_major")
    assert np.array_equal(got, want)
    # a second call continues the streams (state carried through the handle)
    got2 = g.generate_host(256, "row_major")
    want2 = _want(cipher, keys, ivs, bits + 256)[:, bits // 8:]
    assert np.array_equal(got2, want2)


@pytest.mark.parametrize("cipher", ["mickey2", "grain", "aes128ctr", "lfsr128"])
@pytest.mark.parametrize("init_fused", [1, 0])
def test_init_paths_keystream(cipher, init_fused):
    """Both initialisation paths (slicing fused into the init kernel / the
    ballot slice kernels) give the oracle's keystream after a rekey, at a
    ragged n spanning several warp-units."""
    n, bits = 32 * 70 + 17, 512
    if cipher == "lfsr128":
        keys, _ = inputs.make_inputs(cipher, n)
        want = oracle.lfsr128_keystream_batch(keys, bits)
        g = bsrng.Generator(cipher, inputs.make_inputs(cipher, n, seed=5)[0], None)
        g.set_option("init_fused", init_fused)
        g.rekey(keys, None)
    else:
        keys, ivs = inputs.make_inputs(cipher, n)
        want = _want(cipher, keys, ivs, bits)
        k0, v0 = inputs.make_inputs(cipher, n, seed=5)
        g = _gen(cipher, k0, v0)
        g.set_option("init_fused", init_fused)
        g.rekey(inputs.aes_key() if cipher == "aes128ctr" else keys, ivs)
    assert np.array_equal(g.generate_host(bits, "row_major"), want)


@pytest.mark.parametrize("cipher", ["mickey2", "grain", "aes128ctr"])
@pytest.mark.parametrize("n", [32 * 70 + 17, 32 * 64, 5])
@pytest.mark.parametrize("misalign", [False, True])
def test_device_input_rekey(cipher, n, misalign):
    """Device-resident keys/IVs: 16 B aligned arrays are read in place by the
    init kernels (the partial last group through the tail buffer); a
    misaligned view takes the staged copy.  Two rekeys in a row, bit-exact."""
    import torch
    bits = 512
    g = None
    for seed in (7, 8):
        keys, ivs = inputs.make_inputs(cipher, n, seed=seed)
        want = _want(cipher, keys, ivs, bits)
        k = inputs.aes_key() if cipher == "aes128ctr" else keys
        if g is None:
            g = _gen(cipher, *inputs.make_inputs(cipher, n, seed=5))
        def dev(a):
            if isinstance(a, (bytes, bytearray)):
                a = np.frombuffer(bytes(a), dtype=np.uint8)
            flat = torch.from_numpy(np.ascontiguousarray(a).reshape(-1).copy())
            if not misalign:
                return flat.cuda()
            buf = torch.zeros(flat.numel() + 16, dtype=torch.uint8, device="cuda")
            buf[3:3 + flat.numel()] = flat.cuda()
            return buf[3:3 + flat.numel()]
        g.rekey(dev(k), dev(ivs))
        assert np.array_equal(g.generate_host(bits, "row_major"), want), seed


@pytest.mark.parametrize("cipher,bits,opts", [
    ("grain", 4096, {"rm_ws": 0}), ("grain", 2048, {"rm_ws": 0, "seg_clocks": 512}), ("mickey2", 2048, {"rm_ws": 0}),
    ("grain", 4096, {"rm_ws": 0, "rm_tma": 0}),
])
def test_rm_tma_flush_many_warps(cipher, bits, opts):
    """TMA tensor-store flushes (3-D view [q][group][byte] of the row-major
    output) from several warp-units at once plus a ragged tail unit that
    falls back to global stores: every row bit-exact.  (129 warp-units, fewer
    than the SMSPs: rm_ws = 0 keeps the plain kernel instead of the writer-warp
    default.)"""
    n = 32 * 32 * 4 + 17
    keys, ivs = inputs.make_inputs(cipher, n)
    want = _want(cipher, keys, ivs, bits)
    g = _gen(cipher, keys, ivs)
    for k, v in opts.items():
        g.set_option(k, v)
    assert np.array_equal(g.generate_host(bits, "row_major"), want)
