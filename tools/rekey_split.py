#!/usr/bin/env python3
"""Time bsrng_rekey from device-resident keys (CUDA events) for each cipher;
run under ncu --metrics gpu__time_duration.sum to split copy vs init kernel."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng, inputs  # noqa: E402

n = 1 << 22
for cipher in sys.argv[1:] or ["mickey2", "grain", "aes128ctr"]:
    keys, ivs = inputs.make_inputs(cipher, n)
    g = bsrng.Generator(cipher, keys, ivs)
    kd = torch.from_numpy(keys).cuda()
    vd = torch.from_numpy(ivs).cuda()
    s = torch.cuda.current_stream()
    for _ in range(3):
        g.rekey(kd, vd, stream=s)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(10):
        g.rekey(kd, vd, stream=s)
    e1.record(s)
    torch.cuda.synchronize()
    print(cipher, "rekey ms", e0.elapsed_time(e1) / 10)
    g.close()
