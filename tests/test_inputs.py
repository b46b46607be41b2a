"""The seeded input generator (paper_conf_icppw_monfaredhkzrg20_b200/inputs.py)."""
import numpy as np

import oracle
from conftest import read_golden
from paper_conf_icppw_monfaredhkzrg20_b200 import inputs


def test_splitmix64_known_answers():
    for kind, seed, idx, val in read_golden("splitmix64_vectors.txt"):
        seed, idx = int(seed, 16), int(idx)
        if kind == "out":
            assert int(inputs.splitmix64(seed, np.array([idx]))[0]) == int(val, 16)
        else:
            k, v = inputs.make_inputs("mickey2", 1, first_instance=idx, seed=seed)
            got = bytes(k[0] if kind.endswith("key") else v[0]).hex()
            assert got == val


def test_shard_invariance_of_inputs():
    k, v = inputs.make_inputs("mickey2", 1000)
    k2, v2 = inputs.make_inputs("mickey2", 300, first_instance=600)
    assert np.array_equal(k[600:900], k2) and np.array_equal(v[600:900], v2)


def test_shapes():
    for c in ("mickey2", "grain", "aes128ctr"):
        k, v = inputs.make_inputs(c, 5)
        assert k.shape == (5, inputs.KEY_BYTES[c]) and v.shape == (5, inputs.IV_BYTES[c])
        assert k.dtype == np.uint8


def test_keygen_instance0_keystream():
    """SURVEY.md sec. 8(c) item 5 lists instance 0's MICKEY keystream for seed
    0x5EED2020 (computed by an independent implementation there)."""
    k, v = inputs.make_inputs("mickey2", 1)
    ks = oracle.mickey2_keystream(bytes(k[0]), bytes(v[0]), 80, 128)
    assert ks.hex() == "8d2f0fdd85ffa8bd4aa685fb0df62b1d"
