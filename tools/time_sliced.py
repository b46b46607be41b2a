#!/usr/bin/env python3
"""CUDA-event time of SLICED generation (n = 2^22, 4096 bits per call = 2 GiB
of output) per cipher and option set: Tb/s and HBM write GB/s."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng  # noqa: E402

n = 1 << 22
for cipher, opts, bits in [("lfsr128", {}, 4096), ("lfsr128", {}, 32768), ("lfsr128", {"unroll": 16}, 32768),
                           ("mickey2", {}, 4096), ("grain", {}, 4096)]:
    g = bsrng.Generator.from_seed(cipher, n)
    for k, v in opts.items():
        g.set_option(k, v)
    out = torch.empty(g.out_bytes(bits, "sliced"), dtype=torch.uint8, device="cuda")
    for _ in range(3):
        g.generate(out, bits, "sliced")
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = 10
    e0.record()
    for _ in range(reps):
        g.generate(out, bits, "sliced")
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    print(cipher, opts, bits, f"{n * bits / ms / 1e9:.2f} Tb/s", f"{out.numel() / ms / 1e6:.0f} GB/s written", flush=True)
    g.close()
