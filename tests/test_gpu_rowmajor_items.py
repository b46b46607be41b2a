"""GPU parity of ROW_MAJOR when warps run SEVERAL work items.

The persistent keystream kernel hands work items (warp-unit x time segment)
to resident warps by ticket.  A warp that finishes an item reuses its TMEM
staging columns, its TMA shared-memory box, the pending-flush slots
(s_pend_col / s_row0) and, with time segments, the segment flags for the
next item.  The bench's materialise line runs exactly that regime:
n = 2^22 MICKEY 2.0 instances (4096 warp-units) on 2 x 4 x 148 = 1184
resident warps, 2^15-bit calls, so warp-unit u is the (u // 1184 + 1)-th item
of some warp.  These tests compare rows from every item rank, plus random
rows, with the bit-serial oracle (sec. 4.5 output stage;
bit-exact), over two consecutive calls (the state carry
between calls), and force the multi-item regime at a small n for every
flush variant: TMA tensor stores, 8 B sector stores, double-buffered TMEM,
shared-memory staging and the warp-specialised kernel.
"""
import numpy as np
import pytest

import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng, inputs  # noqa: E402

RESIDENT_WARPS = 2 * 4 * 148  # whole_units policy: 2 CTAs/SM x 4 clock-loop warps


def _oracle_rows(cipher, keys, ivs, bits):
    if cipher == "mickey2":
        return oracle.mickey2_keystream_batch(keys, ivs, 80, bits)
    if cipher == "lfsr128":
        return oracle.lfsr128_keystream_batch(keys, bits)
    return oracle.grain_keystream_batch(keys, ivs, bits)


def _sample_rows(n, units_of_interest, rng, extra=256):
    rows = [1024 * u + r for u in units_of_interest for r in (0, 1, 31, 32, 517, 992, 1023)]
    rows += list(rng.integers(0, n, extra))
    rows += [n - 1]
    return np.unique(np.array([r for r in rows if 0 <= r < n], dtype=np.int64))


def _gather_rows(buf, idx, row_bytes):
    """rows idx of a device uint8 buffer of n x row_bytes (copy only those rows)."""
    t = torch.from_numpy(idx).to(buf.device)
    return buf.view(-1, row_bytes).index_select(0, t).cpu().numpy()


@pytest.mark.parametrize("cipher", ["mickey2", "grain"])
def test_bench_materialise_shape_two_calls(cipher):
    """n = 2^22, two consecutive 2^15-bit ROW_MAJOR calls in the bench's
    launch configuration (default options = what bench.py times)."""
    n, chunk = 1 << 22, 1 << 15
    keys, ivs = inputs.make_inputs(cipher, n)
    kd, vd = torch.from_numpy(keys).cuda(), torch.from_numpy(ivs).cuda()
    g = bsrng.Generator(cipher, kd, vd)
    buf = torch.empty(g.out_bytes(chunk, "row_major"), dtype=torch.uint8, device="cuda")
    units = n // 1024
    item_starts = [k * RESIDENT_WARPS for k in range(4) if k * RESIDENT_WARPS < units]
    rng = np.random.default_rng(20 if cipher == "mickey2" else 21)
    idx = _sample_rows(n, item_starts + [units - 1], rng)
    got = []
    for _ in range(2):
        g.generate(buf, chunk, "row_major")
        torch.cuda.synchronize()
        got.append(_gather_rows(buf, idx, chunk // 8))
    want = _oracle_rows(cipher, keys[idx], ivs[idx], 2 * chunk)
    assert np.array_equal(got[0], want[:, : chunk // 8]), "first call"
    assert np.array_equal(got[1], want[:, chunk // 8:]), "second call (state carried)"


# (cipher, options, bits per call): n ~ 2^20 = 1024 warp-units on one CTA per
# SM (592 warps), so most warps run two or more items
_FORCED = [
    ("grain", {"ctas_per_sm": 1, "seg_clocks": 256}, 2048),                   # TMA flush, time segments
    ("mickey2", {"ctas_per_sm": 1, "seg_clocks": 256}, 1024),                 # TMA flush, time segments
    ("grain", {"ctas_per_sm": 1, "seg_clocks": 256, "rm_tma": 0}, 2048),      # 8 B sector stores
    ("mickey2", {"ctas_per_sm": 1, "seg_clocks": 256, "rm_tma": 0}, 1024),    # 8 B sector stores
    ("grain", {"ctas_per_sm": 1, "seg_clocks": 2048, "rm_tma": 0}, 2048),     # double-buffered TMEM (1 segment)
    ("mickey2", {"ctas_per_sm": 1, "seg_clocks": 1024, "rm_tma": 0}, 1024),   # double-buffered TMEM (1 segment)
    ("grain", {"ctas_per_sm": 1, "seg_clocks": 256, "rm_tmem": 0}, 2048),     # shared-memory staging
    ("mickey2", {"ctas_per_sm": 1, "seg_clocks": 256, "rm_tmem": 0, "rm_ws": 0}, 1024),  # smem staging
    ("mickey2", {"seg_clocks": 256, "rm_ws": 1}, 1024),                        # warp-specialised
    ("grain", {"rm_wide": 1, "seg_clocks": 1024}, 2048),                      # 64 B staging, lone warps
    ("lfsr128", {"rm_ws": 0, "rm_wide": 1, "seg_clocks": 512}, 2048),         # 64 B staging
    ("lfsr128", {"ctas_per_sm": 1, "seg_clocks": 256}, 2048),                 # LFSR default (writer warp)
    ("lfsr128", {"seg_clocks": 512}, 2048 + 96),                              # period bodies + remainder
    ("lfsr128", {"rm_ws": 2, "seg_clocks": 1024}, 4096),                      # two writers per stream, 128 B
    ("lfsr128", {"rm_ws": 2}, 2048 + 256 + 96),                               # ragged last period: partial flushes
    ("lfsr128", {"rm_ws": 2, "seg_clocks": 256}, 768),                        # items start mid-period (k_lo > 0)
    ("lfsr128", {"rm_ws": 2, "seg_clocks": 160}, 480),                        # skip blocks at unaligned item starts
]


@pytest.mark.parametrize("cipher,opts,bits", _FORCED, ids=lambda x: str(x))
def test_forced_multi_item_per_warp(cipher, opts, bits):
    n = (1 << 20) + 37  # ragged tail unit
    keys, ivs = inputs.make_inputs(cipher, n, seed=77)
    kd = torch.from_numpy(keys).cuda()
    vd = torch.from_numpy(ivs).cuda() if cipher != "lfsr128" else None
    g = bsrng.Generator(cipher, kd, vd)
    for k, v in opts.items():
        g.set_option(k, v)
    buf = torch.empty(g.out_bytes(bits, "row_major"), dtype=torch.uint8, device="cuda")
    units = (n + 1023) // 1024
    rng = np.random.default_rng(5)
    idx = _sample_rows(n, [0, 1, 591, 592, 593, 1000, units - 2, units - 1], rng, extra=128)
    got = []
    for _ in range(2):
        g.generate(buf, bits, "row_major")
        torch.cuda.synchronize()
        got.append(_gather_rows(buf, idx, bits // 8))
    want = _oracle_rows(cipher, keys[idx], ivs[idx], 2 * bits)
    assert np.array_equal(got[0], want[:, : bits // 8])
    assert np.array_equal(got[1], want[:, bits // 8:])


@pytest.mark.parametrize("cipher", ["lfsr128", "aes128ctr"])
def test_bench_materialise_shape_other_ciphers(cipher):
    """The LFSR (writer-warp kernel, 64 B TMEM staging) and AES-128-CTR
    (block-lane kernel) at the bench's materialise shape: n = 2^22, two
    consecutive 2^15-bit ROW_MAJOR calls, sampled rows vs the oracle."""
    n, chunk = 1 << 22, 1 << 15
    keys, ivs = inputs.make_inputs(cipher, n)
    if cipher == "aes128ctr":
        key = inputs.aes_key()
        g = bsrng.Generator(cipher, torch.from_numpy(key).cuda(), torch.from_numpy(ivs).cuda())
    else:
        g = bsrng.Generator(cipher, torch.from_numpy(keys).cuda(), None)
    buf = torch.empty(g.out_bytes(chunk, "row_major"), dtype=torch.uint8, device="cuda")
    units = n // 1024
    rng = np.random.default_rng(22)
    idx = _sample_rows(n, [0, 1, 591, 592, 1183, 1184, 2368, units - 1], rng)
    got = []
    for _ in range(2):
        g.generate(buf, chunk, "row_major")
        torch.cuda.synchronize()
        got.append(_gather_rows(buf, idx, chunk // 8))
    if cipher == "aes128ctr":
        want = oracle.aes128_ctr_keystream_batch(bytes(inputs.aes_key()), ivs[idx], 2 * chunk)
    else:
        want = oracle.lfsr128_keystream_batch(keys[idx], 2 * chunk)
    assert np.array_equal(got[0], want[:, : chunk // 8])
    assert np.array_equal(got[1], want[:, chunk // 8:])


@pytest.mark.parametrize("cipher", ["grain", "mickey2", "lfsr128"])
def test_paper_shape_rowmajor_sampled(cipher):
    """configs[3]: 2^19 instances x 4416 clocks (552 B rows, 8 B aligned) in
    the launch configuration bench.py times (Grain and the LFSR: writer-warp
    kernel with two STG.64 per 16 B piece; MICKEY: double-buffered TMEM), two
    calls, sampled rows vs the oracle."""
    n, bits = 1 << 19, 4416
    keys, ivs = inputs.make_inputs(cipher, n, seed=3)
    g = bsrng.Generator(cipher, torch.from_numpy(keys).cuda(),
                        None if cipher == "lfsr128" else torch.from_numpy(ivs).cuda())
    buf = torch.empty(g.out_bytes(bits, "row_major"), dtype=torch.uint8, device="cuda")
    rng = np.random.default_rng(4)
    idx = _sample_rows(n, [0, 1, 255, 256, 511], rng, extra=160)
    got = []
    for _ in range(2):
        g.generate(buf, bits, "row_major")
        torch.cuda.synchronize()
        got.append(_gather_rows(buf, idx, bits // 8))
    want = _oracle_rows(cipher, keys[idx], ivs[idx], 2 * bits)
    assert np.array_equal(got[0], want[:, : bits // 8])
    assert np.array_equal(got[1], want[:, bits // 8:])
