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

# n = 32 * 40 + 9 etc. are a few dozen warp-units, i.e. fewer than the SMSPs:
# there MICKEY and Grain default to the writer-warp ROW_MAJOR kernel, so the
# plain kernel's staging variants are reached with rm_ws = 0
W = {"rm_ws": 0}
cases = [
    ("mickey2", 32 * 40 + 9, 1024, {}), ("mickey2", 32 * 40 + 9, 1024 + 512, {}),      # writer warps (lone units)
    ("mickey2", 32 * 40 + 9, 1024, W), ("mickey2", 32 * 32 * 2, 2048, W),              # TMEM staging, TMA flush
    ("mickey2", 32 * 40 + 9, 1024, {**W, "rm_tma": 0}), ("mickey2", 32 * 40 + 9, 1024, {**W, "rm_wide": 1}),
    ("mickey2", 32 * 40 + 9, 1024, {**W, "rm_l2last": 0}), ("mickey2", 32 * 40 + 9, 1024, {**W, "rm_tmem": 0}),
    ("grain", 32 * 40 + 9, 1024, {}), ("grain", 32 * 40, 552 * 8, {}),                  # writer warps, 8 B rows
    ("grain", 32 * 40 + 9, 1024, W), ("grain", 32 * 32 * 2, 2048, W), ("grain", 32 * 40, 552 * 8, W),
    ("grain", 32 * 40 + 9, 1024 + 512, {**W, "rm_wide": 1}), ("grain", 32 * 40 + 9, 1024, {**W, "rm_tma": 0}),
    ("aes128ctr", 32 * 9 + 5, 4480, {}), ("aes128ctr", 32 * 9 + 5, 4480, {"rm_ws": 0}),
    ("lfsr128", 32 * 37 + 13, 1024, {}), ("lfsr128", 32 * 37 + 13, 2048 + 96, {}),    # period bodies + remainder
    ("lfsr128", 32 * 37 + 13, 1024, {"rm_ws": 0}), ("lfsr128", 32 * 37 + 13, 1024, {"rm_ws": 1}),
    ("lfsr128", 32 * 37 + 13, 3200, {"seg_clocks": 160}),   # two-writer kernel: odd item starts, unpaired blocks
]
# synccheck stops the process at the plain TMEM kernel ("Barrier error
# detected. Missing init" at shared address 0x0, PC outside the kernel; see
# profiles/r2_sanitizer.md), so gpu.sh runs it twice:
# SANITIZE_NO_TMEM=1: the plain kernel with shared-memory staging instead of
#   tensor memory (rm_tmem = 0 also disables the automatic writer-warp choice);
# SANITIZE_WS_ONLY=1: only the cases that keep the default kernel choice (the
#   writer-warp kernels, which allocate TMEM too, AES, LFSR).
no_tmem = os.environ.get("SANITIZE_NO_TMEM") == "1"
ws_only = os.environ.get("SANITIZE_WS_ONLY") == "1"
for cipher, n, bits, opts in cases:
    if ws_only and opts.get("rm_ws", -1) == 0 and cipher in ("mickey2", "grain"):
        continue
    g = bsrng.Generator.from_seed(cipher, n)
    if no_tmem:
        opts = dict({k: v for k, v in opts.items() if k != "rm_wide"}, rm_tmem=0)  # rm_wide implies TMEM
    for k, v in opts.items():
        g.set_option(k, v)
    for layout in ("row_major", "sliced", "checksum"):
        out = torch.empty(max(g.out_bytes(bits, layout), 16), dtype=torch.uint8, device="cuda")
        g.generate(out, bits, layout)
    torch.cuda.synchronize()
    g.close()
    print("ok", cipher, n, bits, opts, flush=True)
