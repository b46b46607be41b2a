"""Randomised parity sweep over the C ABI: seeded random (cipher, n, bits,
layout, option set, call split) cases, every output compared with the
bit-serial oracle (ROW_MAJOR / SLICED bit-exact, CHECKSUM = its definition on
the oracle keystream).  Complements the hand-picked cases: ragged n across
warp-unit boundaries, call lengths that are not whole staging periods, and
option combinations the other tests do not pair."""
import numpy as np
import pytest

import oracle
from helpers import checksum, to_sliced

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng, inputs  # noqa: E402

# n <= 7681 here is at most 241 warp-units, fewer than the SMSPs: MICKEY and
# Grain ROW_MAJOR default to the writer-warp kernel, rm_ws = 0 reaches the
# plain kernel's staging variants
W = {"rm_ws": 0}
OPTS = {
    "mickey2": [{}, {"sched": 0}, {**W, "rm_tmem": 0}, W, {**W, "rm_tma": 0}, {**W, "rm_wide": 1},
                {"seg_clocks": 96}, {**W, "ctas_per_sm": 1}, {**W, "rm_l2last": 0}, {"rm_ws": 1, "rm_phase": 1}],
    "grain": [{}, {"sched": 0}, {**W, "rm_tmem": 0}, {"rm_ws": 1}, W, {**W, "rm_tma": 0}, {**W, "rm_wide": 1},
              {"unroll": 16}, {"seg_clocks": 160}, {"ctas_per_sm": 1}, {**W, "rm_dbl": 0}, {"rm_ws": 1, "rm_phase": 1},
              {"rm_ws": 1, "rm_phase": 0}],
    "lfsr128": [{}, {"sched": 0}, {"rm_ws": 0}, {"rm_ws": 1}, {"rm_ws": 2}, {"rm_ws": 2, "seg_clocks": 96}, {**W, "rm_wide": 1},
                {"unroll": 16}, {"seg_clocks": 64}],
    "aes128ctr": [{}, {"rm_ws": 0}, {"ctas_per_sm": 1}, {"seg_clocks": 256}],
}


def _oracle(cipher, keys, ivs, bits):
    if cipher == "mickey2":
        return oracle.mickey2_keystream_batch(keys, ivs, 80, bits)
    if cipher == "grain":
        return oracle.grain_keystream_batch(keys, ivs, bits)
    if cipher == "lfsr128":
        return oracle.lfsr128_keystream_batch(keys, bits)
    return oracle.aes128_ctr_keystream_batch(bytes(inputs.aes_key()), ivs, bits)


@pytest.mark.parametrize("case", range(64))
def test_random_case(case):
    rng = np.random.default_rng(1000 + case)
    cipher = ["mickey2", "grain", "lfsr128", "aes128ctr"][case % 4]
    n = int(rng.choice([1, 31, 33, 1023, 1025, 2048 + 7, 4096 + 31, 7 * 1024 + 513]))
    q = 128 if cipher == "aes128ctr" else 32
    calls = [int(rng.integers(1, 24 if cipher != "mickey2" else 12)) * q for _ in range(int(rng.integers(1, 4)))]
    layout = ["row_major", "sliced", "checksum"][int(rng.integers(0, 3))]
    opts = OPTS[cipher][int(rng.integers(0, len(OPTS[cipher])))]
    keys, ivs = inputs.make_inputs(cipher, n, seed=int(rng.integers(1, 1 << 30)))
    if cipher == "aes128ctr":
        g = bsrng.Generator(cipher, inputs.aes_key(), ivs)
    else:
        g = bsrng.Generator(cipher, keys, None if cipher == "lfsr128" else ivs)
    for k, v in opts.items():
        g.set_option(k, v)
    want = _oracle(cipher, keys, ivs, sum(calls))
    msb = cipher != "grain"
    t0 = 0
    for c in calls:
        got = g.generate_host(c, layout)
        part = want[:, t0 // 8:(t0 + c) // 8]
        ctx = (cipher, n, calls, layout, opts)
        if layout == "row_major":
            assert np.array_equal(got, part), ctx
        elif layout == "sliced":
            assert np.array_equal(got, to_sliced(part, msb_first=msb)), ctx
        else:
            assert int(got[0]) == checksum(to_sliced(part, msb_first=msb), t0=t0), ctx
        t0 += c
