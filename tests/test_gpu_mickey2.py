"""GPU parity: bitsliced MICKEY 2.0 through the C ABI vs the bit-serial oracle.

Bar: bit-exact (GF(2) logic, no rounding, exactly one
keystream per (key, IV)).  Inputs: the seeded SplitMix64 recipe
(paper_conf_icppw_monfaredhkzrg20_b200/inputs.py, seed 0x5EED2020).
"""
import numpy as np
import pytest

import oracle
from conftest import read_golden
from helpers import checksum, state_to_sliced, to_sliced

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng, inputs  # noqa: E402


def _gen(n, first=0, **kw):
    keys, ivs = inputs.make_inputs("mickey2", n, first)
    return bsrng.Generator("mickey2", keys, ivs, first_instance=first, **kw), keys, ivs


def _dev_rows(g, bits):
    out = torch.empty(g.out_bytes(bits, "row_major"), dtype=torch.uint8, device="cuda")
    g.generate(out, bits, "row_major")
    torch.cuda.synchronize()
    return out.cpu().numpy().reshape(g.n, bits // 8)


# ----------------------------------------------------------------- spec vectors
@pytest.mark.parametrize("row", read_golden("mickey2_spec_vectors.txt"), ids=lambda r: r[0])
def test_spec_vectors_on_gpu(row):
    name, key, iv, iv_bits, prefix = row
    iv_bits = int(iv_bits)
    k = np.frombuffer(bytes.fromhex(key), np.uint8).reshape(1, 10)
    v = np.zeros((1, 10), np.uint8)
    if iv != "-":
        b = bytes.fromhex(iv)
        v[0, : len(b)] = np.frombuffer(b, np.uint8)
    with bsrng.Generator("mickey2", k, v, iv_bits=iv_bits) as g:
        got = g.generate_host(256, "row_major")[0].tobytes().hex()
    assert got.startswith(prefix)
    assert got == oracle.mickey2_keystream(bytes(k[0]), bytes(v[0]), iv_bits, 256).hex()


# ------------------------------------------------------------------ config 1
def test_config1_all_layouts():
    """C1: 32 instances x 2^16 bits, every bit of every layout vs the oracle."""
    n, bits = 32, 1 << 16
    keys, ivs = inputs.make_inputs("mickey2", n)
    want = oracle.mickey2_keystream_batch(keys, ivs, 80, bits)
    g = bsrng.Generator("mickey2", keys, ivs)
    assert np.array_equal(_dev_rows(g, bits), want)
    g = bsrng.Generator("mickey2", keys, ivs)
    sl = g.generate_host(bits, "sliced")
    assert np.array_equal(sl, to_sliced(want))
    g = bsrng.Generator("mickey2", keys, ivs)
    cs = g.generate_host(bits, "checksum")
    assert int(cs[0]) == checksum(to_sliced(want))


def test_preclock_state_parity():
    n = 70
    g, keys, ivs = _gen(n)
    # lanes >= n of the last group are padding instances (zero key/IV): their
    # state is defined but not part of the contract, so compare real lanes only
    real = np.full(g.groups, 0xFFFFFFFF, dtype=np.uint32)
    real[-1] = (1 << (n - 32 * (g.groups - 1))) - 1
    for clocks in (0, 96):
        if clocks:
            g.generate_host(clocks, "checksum")
        rs = [oracle.mickey2_state(bytes(keys[i]), bytes(ivs[i]), 80, clocks) for i in range(n)]
        want = state_to_sliced(np.stack([x[0] for x in rs]), np.stack([x[1] for x in rs]))
        assert np.array_equal(g.copy_state() & real, want)


@pytest.mark.parametrize("init_fused", [1, 0])
@pytest.mark.parametrize("n,iv_bits", [(70, 80), (32 * 37 + 13, 80), (1, 80), (33, 0), (100, 24), (4096 + 5, 72)])
def test_init_paths_state_parity(n, iv_bits, init_fused):
    """a-1 + a-2: the fused slicing + preclock kernel (default) and the
    separate slice / preclock kernels give the oracle's post-init state for
    every real instance, at ragged n and short IVs; rekey uses the same path."""
    keys, ivs = inputs.make_inputs("mickey2", n, seed=11)
    g = bsrng.Generator("mickey2", keys, ivs, iv_bits=iv_bits)
    g.set_option("init_fused", init_fused)
    k2, v2 = inputs.make_inputs("mickey2", n, seed=12)
    g.rekey(k2, v2)
    real = np.full(g.groups, 0xFFFFFFFF, dtype=np.uint32)
    if n % 32:
        real[-1] = (1 << (n % 32)) - 1
    idx = range(n) if n <= 256 else list(range(64)) + list(range(n - 64, n))
    rs = {i: oracle.mickey2_state(bytes(k2[i]), bytes(v2[i]), iv_bits, 0) for i in idx}
    st = g.copy_state()
    for i in idx:
        gi, j = divmod(i, 32)
        got_r = (st[:100, gi] >> np.uint32(j)) & 1
        got_s = (st[100:, gi] >> np.uint32(j)) & 1
        assert np.array_equal(got_r, np.asarray(rs[i][0], dtype=np.uint32)), i
        assert np.array_equal(got_s, np.asarray(rs[i][1], dtype=np.uint32)), i
    # and the keystream that follows
    want = oracle.mickey2_keystream_batch(k2[:40], v2[:40], iv_bits, 256)
    assert np.array_equal(g.generate_host(256, "row_major")[:40], want)


@pytest.mark.parametrize("iv_bits", [0, 32, 72])
def test_short_ivs(iv_bits):
    n, bits = 40, 512
    keys, ivs = inputs.make_inputs("mickey2", n)
    want = np.stack([np.frombuffer(oracle.mickey2_keystream(bytes(keys[i]), bytes(ivs[i]), iv_bits, bits),
                                   np.uint8) for i in range(n)])
    with bsrng.Generator("mickey2", keys, ivs, iv_bits=iv_bits) as g:
        assert np.array_equal(g.generate_host(bits, "row_major"), want)


# --------------------------------------------- several tiles + a ragged tail
@pytest.mark.parametrize("sched", [0, 1])
def test_ragged_multi_unit(sched):
    """n spans 2 warp-units (38 groups) with a 13-lane tail group."""
    n, bits = 32 * 37 + 13, 2048
    keys, ivs = inputs.make_inputs("mickey2", n)
    want = oracle.mickey2_keystream_batch(keys, ivs, 80, bits)
    for layout in ("row_major", "sliced", "checksum"):
        g = bsrng.Generator("mickey2", keys, ivs)
        g.set_option("sched", sched)
        got = g.generate_host(bits, layout)
        if layout == "row_major":
            assert np.array_equal(got, want)
        elif layout == "sliced":
            assert np.array_equal(got, to_sliced(want))
        else:
            assert int(got[0]) == checksum(to_sliced(want))


@pytest.mark.parametrize("seg", [32, 96, 256])
def test_persistent_segments(seg):
    """Time-segmented work items (flag hand-off between warps) == one pass."""
    n, bits = 32 * 32 * 5 + 7, 1024
    keys, ivs = inputs.make_inputs("mickey2", n)
    ref = bsrng.Generator("mickey2", keys, ivs)
    ref.set_option("sched", 0)
    want_rows = ref.generate_host(bits, "row_major")
    for layout in ("row_major", "sliced", "checksum"):
        g = bsrng.Generator("mickey2", keys, ivs)
        g.set_option("sched", 1)
        g.set_option("seg_clocks", seg)
        got = g.generate_host(bits, layout)
        if layout == "row_major":
            assert np.array_equal(got, want_rows)
        elif layout == "sliced":
            assert np.array_equal(got, to_sliced(want_rows))
        else:
            assert int(got[0]) == checksum(to_sliced(want_rows))
    idx = np.array([0, 1, 31, 32, 1000, 4000, n - 1])
    want = oracle.mickey2_keystream_batch(keys[idx], ivs[idx], 80, bits)
    assert np.array_equal(want_rows[idx], want)


# ------------------------------------------------------ statefulness, padding
@pytest.mark.parametrize("layout", ["row_major", "sliced", "checksum"])
def test_concatenation(layout):
    n, a, b = 96, 320, 704
    keys, ivs = inputs.make_inputs("mickey2", n)
    whole = bsrng.Generator("mickey2", keys, ivs).generate_host(a + b, "row_major")
    g = bsrng.Generator("mickey2", keys, ivs)
    x = g.generate_host(a, layout)
    y = g.generate_host(b, layout)
    assert g.bits_done == a + b
    if layout == "row_major":
        assert np.array_equal(np.concatenate([x, y], axis=1), whole)
    elif layout == "sliced":
        assert np.array_equal(np.concatenate([x, y], axis=0), to_sliced(whole))
    else:
        sl = to_sliced(whole)
        assert int(x[0]) == checksum(sl[:a], t0=0)
        assert int(y[0]) == checksum(sl[a:], t0=a)


def test_padding_instances_do_not_leak():
    keys, ivs = inputs.make_inputs("mickey2", 64)
    r64 = bsrng.Generator("mickey2", keys, ivs).generate_host(256, "row_major")
    g33 = bsrng.Generator("mickey2", keys[:33], ivs[:33])
    assert np.array_equal(g33.generate_host(256, "row_major"), r64[:33])
    s33 = bsrng.Generator("mickey2", keys[:33], ivs[:33]).generate_host(256, "sliced")
    assert np.all((s33[:, 1] >> np.uint32(1)) == 0)  # lanes >= 33 are zero
    assert np.array_equal(s33[:, 0], to_sliced(r64)[:, 0])


def test_layout_round_trip():
    keys, ivs = inputs.make_inputs("mickey2", 200)
    rows = bsrng.Generator("mickey2", keys, ivs).generate_host(640, "row_major")
    sl = bsrng.Generator("mickey2", keys, ivs).generate_host(640, "sliced")
    assert np.array_equal(to_sliced(rows), sl)


def test_device_inputs_and_rekey():
    n, bits = 128, 512
    keys, ivs = inputs.make_inputs("mickey2", n)
    want = oracle.mickey2_keystream_batch(keys, ivs, 80, bits)
    kd = torch.from_numpy(keys).cuda()
    vd = torch.from_numpy(ivs).cuda()
    g = bsrng.Generator("mickey2", kd, vd)
    assert np.array_equal(g.generate_host(bits, "row_major"), want)
    k2, v2 = inputs.make_inputs("mickey2", n, seed=7)
    g.rekey(k2, v2)
    assert g.bits_done == 0
    want2 = oracle.mickey2_keystream_batch(k2, v2, 80, bits)
    assert np.array_equal(g.generate_host(bits, "row_major"), want2)


# ------------------------------------------------------------- error paths
def test_errors():
    g, _, _ = _gen(64)
    buf = torch.empty(1 << 16, dtype=torch.uint8, device="cuda")
    with pytest.raises(bsrng.BsrngError) as e:
        g.generate(buf, 48, "sliced")
    assert e.value.code == bsrng.EINVAL
    with pytest.raises(bsrng.BsrngError) as e:
        g.generate(buf.data_ptr() + 4, 32, "sliced")
    assert e.value.code == bsrng.EINVAL
    with pytest.raises(bsrng.BsrngError) as e:
        g.generate(buf.data_ptr(), (1 << 40) + 32, "checksum")
    assert e.value.code == bsrng.ERANGE
    with pytest.raises(bsrng.BsrngError) as e:
        g.generate(buf, 32, 7)
    assert e.value.code == bsrng.EINVAL
    with pytest.raises(bsrng.BsrngError):
        g.set_option("nope", 1)


# ------------------------------------------- full-size (config 2) sampling
def test_config2_size_sampled():
    """n = 2^22 (the bench's instance count, its persistent launch): sampled
    instances vs the oracle, SLICED checksum vs the CHECKSUM layout, and shard
    invariance of the checksum."""
    n, bits = 1 << 22, 1024
    g, keys, ivs = _gen(n)
    sl = torch.empty(g.out_bytes(bits, "sliced") // 4, dtype=torch.int32, device="cuda")
    g.generate(sl, bits, "sliced")
    sl_h = sl.cpu().numpy().view(np.uint32).reshape(bits, n // 32)
    rng = np.random.default_rng(1)
    idx = np.unique(np.concatenate([rng.integers(0, n, 256), np.arange(32), np.arange(n - 32, n)]))
    want = oracle.mickey2_keystream_batch(keys[idx], ivs[idx], 80, bits)
    wbits = np.unpackbits(want, axis=1, bitorder="big")
    got = (sl_h[:, idx // 32] >> (idx % 32).astype(np.uint32)) & 1
    assert np.array_equal(got.T.astype(np.uint8), wbits)
    cs_full = bsrng.Generator("mickey2", keys, ivs).generate_host(bits, "checksum")[0]
    assert int(cs_full) == checksum(sl_h)
    half = n // 2
    parts = 0
    for r in range(2):
        gr = bsrng.Generator("mickey2", keys[r * half:(r + 1) * half], ivs[r * half:(r + 1) * half],
                             first_instance=r * half)
        parts = (parts + int(gr.generate_host(bits, "checksum")[0])) % (1 << 64)
    assert parts == int(cs_full)


def test_long_run_tail():
    """State carry at large t: bits [2^20, 2^20 + 1024) of sampled instances."""
    n = 32 * 40
    g, keys, ivs = _gen(n)
    g.generate_host(1 << 20, "checksum")
    tail = g.generate_host(1024, "row_major")
    idx = np.array([0, 5, 639, n - 1])
    full = oracle.mickey2_keystream_batch(keys[idx], ivs[idx], 80, (1 << 20) + 1024)
    assert np.array_equal(tail[idx], full[:, (1 << 20) // 8:])
