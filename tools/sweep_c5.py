#!/usr/bin/env python3
"""BASELINE.json configs[4]: the paper-shaped sweep.

Sweeps, for bitsliced MICKEY 2.0 (and a slice for Grain v1 / AES-128-CTR):
  * schedule / occupancy: the paper's one-shot grid (one thread per 32-instance
    group, `sched=0`, PAPER.md:751-755 used 64 blocks x 256 threads) vs the
    persistent time-segmented queue at 1 or 2 resident clock-loop warps per
    SMSP (`ctas_per_sm` 1/2) vs the auto policy;
  * instances n in {2^19 (the paper's 64x256x32), 2^22, 2^25};
  * clocks per launch in {4416, 12992, 2^16, 2^20};
  * output layout (consume / SLICED / ROW_MAJOR) and the ROW_MAJOR staging
    variants (TMEM + TMA flush, TMEM + 8 B stores, shared memory, writer warps
    with 64 B TMEM staging, a lone warp with 64 B staging) for MICKEY, Grain
    and the LFSR.  (Round 1 also swept MICKEY's unroll U in {2, 4, 8}; only
    U = 4 is built since round 2: profiles/r1_sweep_c5.md.)
Every point is CUDA-event timed on a warmed stream (best of `--reps`), with the
algorithmic LOP3 rate against the ALU roofline at the SM clock sampled by
nvidia-smi during the run.  cuRAND on the same byte count is timed by
tools/microbench/curand_bench (context, run by tools/gpu_c5.sh).

Output: one JSON object per line (stdout).
"""
import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng  # noqa: E402

OPS = {"mickey2": 304.0,  # kernel count: deferred R reduction (327 in Galois form)
       "grain": 37.0, "aes128ctr": 16848.0 / 128.0, "lfsr128": 2.0}
ALG = {"mickey2": 327.0, "grain": 39.0, "aes128ctr": 17280.0 / 128.0, "lfsr128": 2.0}
PAPER_CLOCKS = (4416, 12992)  # multiples of 32 nearest the paper's 4,400 / 13,000


class ClockSampler:
    def __init__(self):
        self.samples, self._stop = [], threading.Event()
        self._t = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "--query-gpu=clocks.sm", "--format=csv,noheader,nounits",
                                      "-i", "0"], capture_output=True, text=True, timeout=5).stdout
                self.samples.append(int(out.strip().splitlines()[0]))
            except Exception:
                pass
            self._stop.wait(0.2)

    def __enter__(self):
        self._t.start()
        return self

    def __exit__(self, *exc):
        self._stop.set()
        self._t.join()

    def median(self):
        s = sorted(self.samples)
        return s[len(s) // 2] if s else None


def point(cipher, n, bits, layout, opts, reps, chunk=None, nsm=148):
    """Time `bits` clocks of `n` instances (in calls of `chunk` clocks)."""
    chunk = chunk or bits
    g = bsrng.Generator.from_seed(cipher, n)
    for k, v in opts.items():
        g.set_option(k, v)
    out = torch.empty(max(g.out_bytes(chunk, layout), 16), dtype=torch.uint8, device="cuda")
    g.generate(out, chunk, layout)  # warm-up (module load, first-touch)
    torch.cuda.synchronize()
    best = None
    with ClockSampler() as cs:
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(bits // chunk):
                g.generate(out, chunk, layout)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1)
            best = ms if best is None else min(best, ms)
    g.close()
    del out
    mhz = cs.median() or 1965
    tbps = n * bits / (best * 1e-3) / 1e12
    per_clock = OPS[cipher]
    if cipher == "mickey2" and "unroll" in opts:  # deferred-reduction block K follows U (bench.py)
        sys.path.insert(0, ROOT)
        import bench
        per_clock = bench.lop3_per_bit("mickey2", "consume", opts["unroll"])
    ops = per_clock * (n / 32) * bits / (best * 1e-3)
    peak = nsm * 64 * mhz * 1e6
    return {"cipher": cipher, "n": n, "clocks_per_call": chunk, "clocks": bits, "layout": layout, "opts": opts,
            "ms": round(best, 3), "tbps": round(tbps, 4), "sm_mhz": mhz, "alu_frac": round(ops / peak, 4),
            "alu_frac_alg": round(ALG[cipher] * (n / 32) * bits / (best * 1e-3) / peak, 4),
            "hbm_write_gbs": round(n * bits / 8 / (best * 1e-3) / 1e9, 1) if layout == "row_major" else None}


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--reps", type=int, default=3)
    p.add_argument("--quick", action="store_true", help="small subset (CI smoke of the tool)")
    a = p.parse_args()
    nsm = torch.cuda.get_device_properties(0).multi_processor_count
    emit = lambda d: print(json.dumps(d), flush=True)  # noqa: E731

    # 1. schedule x occupancy x n x clocks per launch (MICKEY consume)
    scheds = [("paper_oneshot", {"sched": 0}), ("persist_1w", {"ctas_per_sm": 1}),
              ("persist_2w", {"ctas_per_sm": 2}), ("auto", {})]
    ns = [1 << 19, 1 << 22] if a.quick else [1 << 19, 1 << 22, 1 << 25]
    clocks = [4416] if a.quick else [4416, 12992, 1 << 16, 1 << 20]
    for n in ns:
        for c in clocks:
            if n * c > (1 << 42):  # cap one point at ~2.5 s
                continue
            for name, o in scheds:
                d = point("mickey2", n, c, "checksum", o, a.reps, nsm=nsm)
                d["sweep"], d["schedule"] = "schedule", name
                emit(d)
    if a.quick:
        return
    # 2. output layouts (MICKEY, C2 shape, 2^16 clocks per instance)
    for lay, chunks in [("checksum", (1 << 16,)), ("sliced", (1 << 12, 1 << 15)), ("row_major", (1 << 12, 1 << 15))]:
        for chunk in chunks:
            d = point("mickey2", 1 << 22, 1 << 16, lay, {}, a.reps, chunk=chunk, nsm=nsm)
            d["sweep"] = "layout"
            emit(d)
    # 3. ROW_MAJOR staging variants (2^15-bit calls, 4 KB rows)
    variants = [("tmem_tma", {"rm_ws": 0, "rm_tmem": 1}), ("tmem_8B", {"rm_ws": 0, "rm_tmem": 1, "rm_tma": 0}),
                ("tmem_evict_first", {"rm_ws": 0, "rm_tmem": 1, "rm_l2last": 0}),
                ("smem", {"rm_ws": 0, "rm_tmem": 0}), ("writer_warps_64B", {"rm_ws": 1}),
                ("lone_warp_64B", {"rm_ws": 0, "rm_wide": 1})]
    for cipher, bits in (("mickey2", 1 << 16), ("grain", 1 << 17), ("lfsr128", 1 << 18)):
        for name, o in variants:
            d = point(cipher, 1 << 22, bits, "row_major", o, a.reps, chunk=1 << 15, nsm=nsm)
            d["sweep"], d["staging"] = "rm_staging", name
            emit(d)
    # 4. Grain v1 and AES-128-CTR: occupancy and unroll at the C2 shape
    for cipher, opts in [("grain", [{"ctas_per_sm": 1}, {"ctas_per_sm": 2}, {"unroll": 16}, {}]),
                         ("aes128ctr", [{"ctas_per_sm": 1}, {"ctas_per_sm": 2}, {}])]:
        for o in opts:
            for lay in ("checksum", "row_major"):
                d = point(cipher, 1 << 22, 1 << 16, lay, o, a.reps,
                          chunk=(1 << 14) if lay == "row_major" else None, nsm=nsm)
                d["sweep"] = "cipher"
                emit(d)


if __name__ == "__main__":
    main()
