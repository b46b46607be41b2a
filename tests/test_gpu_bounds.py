"""Out-of-bounds write checks for every output path (GPU).

compute-sanitizer is not available on the GPU pool for the final round-2
kernels (profiles/r2_sanitizer.md), so the output side gets its own bounds
check: each call writes into a view of a larger device buffer whose 64 KB
guard bands before and after are filled with a pattern; after the call the
guards must be untouched and the view must equal the oracle's keystream in the
requested layout (include/bsrng.h).  The cases cover every ROW_MAJOR staging
path (plain kernel with TMEM / TMA / 8 B sector / double-buffered / shared-
memory / 64 B staging, the writer-warp kernel with and without staggered flush
periods, the two-writer kernel with paired and unpaired blocks, the AES
block-lane kernel plus its remainder), SLICED and CHECKSUM, at ragged n, 8 B-
aligned rows (the paper's 552 B) and mid-period second calls.
"""
import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import oracle  # noqa: E402
from helpers import checksum, to_sliced  # noqa: E402

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng, inputs  # noqa: E402

GUARD = 1 << 16
PATTERN = 0xA5

W = {"rm_ws": 0}
CASES = [
    # cipher, n, calls (bits per call), options
    ("mickey2", 1289, [1024, 1536], {}),                                   # writer-warp kernel (lone units)
    ("mickey2", 1289, [4416], {}),                                         # ... 552 B rows, staggered flushes
    ("mickey2", 2048, [2048], W),                                          # TMEM staging + TMA flush
    ("mickey2", 1289, [1024, 96], {**W, "rm_tma": 0}),                     # 8 B sector flush, partial period
    ("mickey2", 1289, [1024], {**W, "rm_tmem": 0}),                        # shared-memory staging
    ("mickey2", 1289, [1024 + 512 + 96], {**W, "rm_wide": 1}),             # 64 B TMEM staging
    ("grain", 1289, [4416], {}),                                           # writer warp, 552 B rows
    ("grain", 1289, [4416], {"rm_ws": 1, "rm_phase": 0}),
    ("grain", 1289, [4096 + 1024], {"rm_ws": 1, "rm_phase": 1, "seg_clocks": 512}),
    ("grain", 2048 + 7, [4416 + 256], {**W, "rm_tma": 0}),                 # double-buffered TMEM
    ("grain", 2048 + 7, [8192], W),                                        # TMA flush, 1 KB rows
    ("grain", 1289, [2080], {**W, "rm_wide": 1, "seg_clocks": 160}),
    ("grain", 1289, [4416], {**W, "rm_tmem": 0}),
    ("lfsr128", 1289, [8192], {}),                                         # two-writer kernel, paired blocks
    ("lfsr128", 1289, [3200], {"seg_clocks": 160}),                        # ... odd item starts, unpaired blocks
    ("lfsr128", 1289, [4416, 96], {}),                                     # 552 B rows, mid-period second call
    ("lfsr128", 1289, [4096 + 1024 + 96], {"rm_ws": 1}),                   # one-writer kernel
    ("lfsr128", 1289, [2048], {"rm_ws": 0}),
    ("aes128ctr", 1289, [4480], {}),                                       # block-lane kernel + remainder
    ("aes128ctr", 1289, [4096, 512], {}),
    ("aes128ctr", 1289, [2048], {"rm_ws": 0}),                             # instance-sliced ROW_MAJOR
]


def _oracle(cipher, keys, ivs, bits):
    if cipher == "mickey2":
        return oracle.mickey2_keystream_batch(keys, ivs, 80, bits)
    if cipher == "grain":
        return oracle.grain_keystream_batch(keys, ivs, bits)
    if cipher == "lfsr128":
        return oracle.lfsr128_keystream_batch(keys, bits)
    return oracle.aes128_ctr_keystream_batch(bytes(inputs.aes_key()), ivs, bits)


def _generator(cipher, n, seed):
    keys, ivs = inputs.make_inputs(cipher, n, seed=seed)
    if cipher == "aes128ctr":
        return bsrng.Generator(cipher, inputs.aes_key(), ivs), keys, ivs
    return bsrng.Generator(cipher, keys, None if cipher == "lfsr128" else ivs), keys, ivs


# ROW_MAJOR staging options only matter for ROW_MAJOR
PARAMS = [(c, lay) for c in range(len(CASES)) for lay in ("row_major", "sliced", "checksum")
          if lay == "row_major" or not any(k.startswith("rm_") for k in CASES[c][3])]


@pytest.mark.parametrize("case,layout", PARAMS)
def test_guard_bands_untouched(case, layout):
    cipher, n, calls, opts = CASES[case]
    g, keys, ivs = _generator(cipher, n, seed=500 + case)
    for k, v in opts.items():
        g.set_option(k, v)
    want = _oracle(cipher, keys, ivs, sum(calls))
    msb = cipher != "grain"
    t0 = 0
    for c in calls:
        nbytes = g.out_bytes(c, layout)
        buf = torch.full((GUARD + nbytes + GUARD,), PATTERN, dtype=torch.uint8, device="cuda")
        view = buf[GUARD:GUARD + nbytes]
        g.generate(view, c, layout)
        torch.cuda.synchronize()
        host = buf.cpu().numpy()
        ctx = (cipher, n, calls, layout, opts)
        assert np.all(host[:GUARD] == PATTERN), ("write before the output", ctx)
        assert np.all(host[GUARD + nbytes:] == PATTERN), ("write past the output", ctx)
        got = host[GUARD:GUARD + nbytes]
        part = want[:, t0 // 8:(t0 + c) // 8]
        if layout == "row_major":
            assert np.array_equal(got.reshape(n, c // 8), part), ctx
        elif layout == "sliced":
            assert np.array_equal(got.view(np.uint32).reshape(c, -1), to_sliced(part, msb_first=msb)), ctx
        else:
            assert int(got.view(np.uint64)[0]) == checksum(to_sliced(part, msb_first=msb), t0=t0), ctx
        t0 += c
    g.close()
