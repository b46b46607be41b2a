#!/usr/bin/env python3
"""Quick option sweep of bsrng_generate (CUDA-event timed, device-resident).

  python tools/sweep.py --layouts checksum,row_major --opts unroll=2 unroll=4 unroll=8
Each --opts entry is a comma-separated list of key=value handle options.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--cipher", default="mickey2")
    p.add_argument("--n", type=int, default=1 << 22)
    p.add_argument("--bits", type=int, default=1 << 16)
    p.add_argument("--chunk", type=int, default=1 << 15, help="row_major bits per call")
    p.add_argument("--layouts", default="checksum,row_major")
    p.add_argument("--reps", type=int, default=2)
    p.add_argument("--opts", nargs="*", default=[""])
    a = p.parse_args()
    g = bsrng.Generator.from_seed(a.cipher, a.n)
    nsm = torch.cuda.get_device_properties(0).multi_processor_count
    for layout in a.layouts.split(","):
        chunk = a.bits if layout == "checksum" else min(a.chunk, a.bits)
        out = torch.empty(max(g.out_bytes(chunk, layout), 16), dtype=torch.uint8, device="cuda")
        for o in a.opts:
            g2 = bsrng.Generator.from_seed(a.cipher, a.n)
            kv = {}
            for item in filter(None, o.split(",")):
                k, v = item.split("=")
                g2.set_option(k, int(v))
                kv[k] = int(v)
            for _ in range(1):
                g2.generate(out, chunk, layout)
            torch.cuda.synchronize()
            best = None
            for _ in range(a.reps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                for _ in range(a.bits // chunk):
                    g2.generate(out, chunk, layout)
                e1.record()
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1)
                best = ms if best is None else min(best, ms)
            tbps = a.n * a.bits / (best * 1e-3) / 1e12
            lop3 = 304 * (a.n // 32) * a.bits / (best * 1e-3)
            frac = lop3 / (nsm * 64 * 1965e6)
            print(json.dumps({"layout": layout, "opts": kv, "ms": round(best, 3), "tbps": round(tbps, 4),
                              "alu_frac_at_1965": round(frac, 4)}), flush=True)
            g2.close()


if __name__ == "__main__":
    main()
