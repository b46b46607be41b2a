"""GPU parity: the bitsliced 128-bit LFSR
vs the bit-serial oracle (oracle/lfsr_ref.c).  Bar: bit-exact."""
import numpy as np
import pytest

import oracle
from helpers import checksum, to_sliced

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng, inputs  # noqa: E402


@pytest.mark.parametrize("unroll", [0, 16])
def test_all_layouts(unroll):
    n, bits = 32 * 37 + 13, 4096
    keys, _ = inputs.make_inputs("lfsr128", n)
    want = oracle.lfsr128_keystream_batch(keys, bits)
    for layout in ("row_major", "sliced", "checksum"):
        g = bsrng.Generator("lfsr128", keys, None)
        g.set_option("unroll", unroll)
        got = g.generate_host(bits, layout)
        if layout == "row_major":
            assert np.array_equal(got, want)
        elif layout == "sliced":
            assert np.array_equal(got, to_sliced(want))
        else:
            assert int(got[0]) == checksum(to_sliced(want))


def test_concatenation_and_state():
    n = 100
    keys, _ = inputs.make_inputs("lfsr128", n)
    g = bsrng.Generator("lfsr128", keys, None)
    assert np.array_equal(g.copy_state()[:, 0] & 1, np.unpackbits(keys[0], bitorder="big"))
    a = g.generate_host(1024, "row_major")
    b = g.generate_host(2048, "row_major")
    want = oracle.lfsr128_keystream_batch(keys, 3072)
    assert np.array_equal(np.concatenate([a, b], axis=1), want)


@pytest.mark.parametrize("seg", [0, 256, 384])
def test_checksum_period_body(seg):
    """CHECKSUM through the whole-period consume body (Lfsr128::consume_period:
    outputs folded from the entry state, clocks in place) and its < 128-clock
    remainder (whole 32-clock blocks, the API unit): clock counts off the
    128-clock period, segment boundaries inside and across
    periods, and a second call starting mid-period (t0 = first call's bits)."""
    n = 32 * 37 + 13
    keys, _ = inputs.make_inputs("lfsr128", n)
    for first, second in ((96, 160), (128 * 3 + 32, 992), (4096 + 32 * 3, 128 * 7), (32, 32)):
        want = to_sliced(oracle.lfsr128_keystream_batch(keys, first + second))
        g = bsrng.Generator("lfsr128", keys, None)
        if seg:
            g.set_option("seg_clocks", seg)
        a = g.generate_host(first, "checksum")
        b = g.generate_host(second, "checksum")
        assert int(a[0]) == checksum(want[:first])
        assert int(b[0]) == checksum(want[first:], t0=first)
