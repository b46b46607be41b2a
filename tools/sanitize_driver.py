#!/usr/bin/env python3
"""Small generation runs of every cipher / layout / staging path, for
compute-sanitizer (memcheck, racecheck, synccheck).  Bit-exactness is the
tests' job; this only has to exercise every kernel once at ragged sizes."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng  # noqa: E402

cases = [
    ("mickey2", 32 * 40 + 9, 1024, {}), ("mickey2", 32 * 32 * 2, 2048, {}),            # TMEM staging, TMA flush
    ("mickey2", 32 * 40 + 9, 1024, {"rm_tma": 0}), ("mickey2", 32 * 40 + 9, 1024 + 512, {"rm_ws": 1}),
    ("mickey2", 32 * 40 + 9, 1024, {"rm_wide": 1}), ("mickey2", 32 * 40 + 9, 1024, {"rm_l2last": 0}),
    ("grain", 32 * 40 + 9, 1024, {}), ("grain", 32 * 32 * 2, 2048, {}), ("grain", 32 * 40, 552 * 8, {}),
    ("grain", 32 * 40 + 9, 2048, {"rm_ws": 1}), ("grain", 32 * 40, 552 * 8, {"rm_ws": 1}),
    ("grain", 32 * 40 + 9, 1024 + 512, {"rm_wide": 1}), ("grain", 32 * 40 + 9, 1024, {"rm_tma": 0}),
    ("aes128ctr", 32 * 9 + 5, 4480, {}), ("aes128ctr", 32 * 9 + 5, 4480, {"rm_ws": 0}),
    ("lfsr128", 32 * 37 + 13, 1024, {}), ("lfsr128", 32 * 37 + 13, 2048 + 96, {}),
    ("lfsr128", 32 * 37 + 13, 1024, {"rm_ws": 0}),
]
# SANITIZE_NO_TMEM=1: shared-memory staging instead of tensor memory (synccheck
# reports tcgen05.alloc's shared-memory result slot as an uninitialised barrier)
no_tmem = os.environ.get("SANITIZE_NO_TMEM") == "1"
for cipher, n, bits, opts in cases:
    g = bsrng.Generator.from_seed(cipher, n)
    if no_tmem:
        opts = dict(opts, rm_tmem=0)
    for k, v in opts.items():
        g.set_option(k, v)
    for layout in ("row_major", "sliced", "checksum"):
        out = torch.empty(max(g.out_bytes(bits, layout), 16), dtype=torch.uint8, device="cuda")
        g.generate(out, bits, layout)
    torch.cuda.synchronize()
    g.close()
    print("ok", cipher, n, bits, opts, flush=True)
