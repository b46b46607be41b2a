#!/usr/bin/env python3
"""Small driver for ncu captures: one handle, a few generate() calls.

  python tools/prof_driver.py --layout checksum --n 4194304 --bits 4096 --reps 3
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--layout", default="checksum")
    p.add_argument("--cipher", default="mickey2")
    p.add_argument("--n", type=int, default=1 << 22)
    p.add_argument("--bits", type=int, default=4096)
    p.add_argument("--reps", type=int, default=3)
    p.add_argument("--sched", type=int, default=None)
    p.add_argument("--seg-clocks", type=int, default=None)
    p.add_argument("--rm-ws", type=int, default=None)
    p.add_argument("--unroll", type=int, default=None)
    p.add_argument("--opt", action="append", default=[], help="extra handle option key=value")
    a = p.parse_args()
    g = bsrng.Generator.from_seed(a.cipher, a.n)
    if a.sched is not None:
        g.set_option("sched", a.sched)
    if a.seg_clocks is not None:
        g.set_option("seg_clocks", a.seg_clocks)
    if a.rm_ws is not None:
        g.set_option("rm_ws", a.rm_ws)
    if a.unroll is not None:
        g.set_option("unroll", a.unroll)
    for kv in a.opt:
        k, v = kv.split("=")
        g.set_option(k, int(v))
    out = torch.empty(max(g.out_bytes(a.bits, a.layout), 16), dtype=torch.uint8, device="cuda")
    for _ in range(a.reps):
        g.generate(out, a.bits, a.layout)
    torch.cuda.synchronize()
    print("done", a)


if __name__ == "__main__":
    main()
