#!/usr/bin/env python3
"""Benchmark: bitsliced MICKEY 2.0 keystream Tb/s on B200 (BASELINE.json).

Workload (BASELINE.json configs[1]): 2^22 MICKEY 2.0 instances x 2^20 keystream
bits per instance per GPU, keys/IVs from the seeded SplitMix64 recipe (seed
0x5EED2020), synthetic.  One "step" = the whole hot path over one batch:
  a-1 key/IV slicing + a-2 preclock (bsrng_rekey from device-resident keys),
  a-3 clock loop + a-4 output + a-5 state carry (bsrng_generate).
Headline mode "consume": CHECKSUM layout, every keystream bit is computed and
folded into a checksum read back at the end.  Mode "materialise": ROW_MAJOR
keystream written to HBM, 2^15 bits per call (16 GiB buffer, 32 calls/step).

Multi-GPU (torchrun, one process per GPU): rank r owns global instances
[r*n, (r+1)*n) -- weak scaling, no data-path collective; NCCL only carries the
max step time and the uint64 checksum sum (outside the timed region).

`--impl reference` times the CPU oracle (oracle/, bit-serial C) on this box's
host cores on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_DEFAULT = 1 << 22
BITS_DEFAULT = 1 << 20
# LOP3 per keystream bit position per 32-instance group (one clock of one
# thread).  Two counts per cipher:
#  * ALGORITHMIC -- SURVEY.md sec. 8(d)'s per-unit figure, the roofline
#    numerator the contract fixes: MICKEY 2.0 327 per clock (the spec's Galois
#    form, output op included), Grain v1 39 (App. D's
#    decomposition), AES-128-CTR 17280 per 32-block encryption (4096 bit
#    positions; DESIGN.md sec. 5 AES), the LFSR's Eq. 2 feedback 2 (k = 4 taps;
#    + 1 to accumulate the output word in consume mode, as MICKEY's 327
#    counts its output op).
#  * KERNEL -- what the shipped kernels need: MICKEY 304 with the R reduction
#    deferred over K = 4-clock blocks (315.5 at K = 2; mickey2.cuh clock_lazy,
#    DESIGN.md sec. 5 item 10), Grain 37 (+1 to fold into the checksum), AES
#    16848 (MixColumns + AddRoundKey as tools/mc_xor3.py's 84-LOP3 circuit per
#    column instead of 96; +64 for the checksum XOR tree), LFSR 2 (+0.5 for
#    the checksum).
# A kernel whose count is below the algorithmic one can exceed frac = 1.
MICKEY2_GALOIS_OPS = 327.0
MICKEY2_OPS_BY_BLOCK = {1: 327.0, 2: 315.5, 4: 304.0}
# AES kernel count per 32-block encryption: counter + round-0 key 256,
# SubBytes 10 x 16 x 84, MixColumns + AddRoundKey 9 x 4 x 84, final key 128
AES_KERNEL_OPS = 256.0 + 10 * 16 * 84 + 9 * 4 * 84 + 128
ALGORITHMIC_OPS = {"mickey2": 327.0, "grain": 39.0, "aes128ctr": 17280.0 / 128.0, "lfsr128": 2.0}


def algorithmic_ops(cipher, mode):
    """SURVEY.md sec. 8(d) per-clock LOP3 count per 32-instance group."""
    return 3.0 if (cipher == "lfsr128" and mode == "consume") else ALGORITHMIC_OPS[cipher]


def mickey2_block(unroll):
    """Deferred-reduction block K for a U-clock loop body (Mickey2::block_k)."""
    return 4 if unroll % 4 == 0 else 2 if unroll % 2 == 0 else 1


def lop3_per_bit(cipher, mode, unroll=None):
    """KERNEL count (see above) per clock per 32-instance group."""
    if cipher == "mickey2":
        return MICKEY2_OPS_BY_BLOCK[mickey2_block(unroll or 4)]
    if cipher == "grain":
        return 38.0 if mode == "consume" else 37.0
    if cipher == "lfsr128":
        # feedback XOR4 = 2 LOP3; consume folds the period's output words into
        # the accumulator (0.5 per clock; 128-clock loop body)
        return 2.5 if mode == "consume" else 2.0
    return (AES_KERNEL_OPS + (64.0 if mode == "consume" else 0.0)) / 128.0


CIPHER_NAME = {"mickey2": "MICKEY 2.0", "grain": "Grain v1", "aes128ctr": "AES-128-CTR",
               "lfsr128": "bitsliced LFSR-128 (Eq. 2)"}
ALU_LANES_PER_SM_CLK = 64      # 4 SMSP x 16 lanes (alu pipe rt = 2 cycles/warp-instr)
METRIC = "MICKEY 2.0 keystream Tb/s (1 and 8 B200); fraction of LOP3/HBM roofline"


def metric(args):
    """BASELINE.json's metric; with --cipher grain the same metric for Grain v1 (configs[3])."""
    return METRIC if args.cipher == "mickey2" else METRIC.replace("MICKEY 2.0", CIPHER_NAME[args.cipher])


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=3)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--workload", default="c2", choices=["c2", "c3", "c4", "rekey"],
                   help="c2 = BASELINE configs[1] per GPU (weak scaling); "
                        "c3 = configs[2]: 2^25 instances x 2^18 bits = 1 TiB total, split across GPUs (strong); "
                        "c4 = configs[3]: the paper's launch shape, 2^19 instances x 4416 clocks per GPU; "
                        "rekey = SURVEY NEXT-3: 2^22 short streams x 2^10 bits, key/IV setup dominates")
    p.add_argument("--cipher", default="mickey2", choices=["mickey2", "grain", "aes128ctr", "lfsr128"])
    p.add_argument("--instances", "--n", dest="n", type=int, default=None,
                   help="instances per GPU (c2/c4/rekey) / in total (c3); use --instances under torchrun "
                        "(its parser takes --n for one of its own options)")
    p.add_argument("--bits", type=int, default=None, help="keystream bits per instance per step")
    p.add_argument("--no-context", action="store_true", help="skip the ALU-peak / cuRAND microbenchmarks")
    p.add_argument("--mode", default="consume", choices=["consume", "materialise"],
                   help="headline mode")
    p.add_argument("--no-other-mode", action="store_true", help="skip timing the non-headline mode")
    p.add_argument("--chunk-bits", type=int, default=1 << 15, help="materialise bits per call")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--sched", type=int, default=None)
    p.add_argument("--seg-clocks", type=int, default=None)
    p.add_argument("--ctas-per-sm", type=int, default=None)
    p.add_argument("--opt", action="append", default=[], metavar="KEY=VALUE",
                   help="extra bsrng_set_option knob (A/B runs; defaults are the tuned ones)")
    p.add_argument("--test-delay-rank", type=int, default=-1, help=argparse.SUPPRESS)  # tests: MAX over ranks
    p.add_argument("--backend", default=os.environ.get("BSRNG_DIST_BACKEND", "nccl"), choices=["nccl", "gloo"],
                   help="process-group backend for N > 1 (gloo lets two ranks share one GPU in tests; "
                        "only the max step time and the checksum cross ranks)")
    return p.parse_args()


# ------------------------------------------------------------------ helpers
class ClockSampler:
    """nvidia-smi clocks/throttle sampling (every 50 ms) during the timed
    region: the sampler starts before the warm-up, waits for its first sample
    (nvidia-smi takes ~0.1-0.5 s to start), and only samples that arrive
    between begin() and end() (host clock) are reported."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []  # (arrival time, line)
        self.t0 = self.t1 = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "50"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            deadline = time.time() + 5.0
            while not self.lines and time.time() < deadline and self.proc.poll() is None:
                time.sleep(0.02)
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append((time.time(), line.strip()))

    def begin(self):
        self.t0 = time.time()

    def end(self):
        self.t1 = time.time()

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.06)  # let the last in-window sample arrive
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        t0 = self.t0 if self.t0 is not None else 0.0
        t1 = (self.t1 if self.t1 is not None else time.time()) + 0.05
        for ts, ln in self.lines:
            if not (t0 <= ts <= t1):
                continue
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx.append(float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm),
                "window_s": round(t1 - 0.05 - t0, 3) if self.t0 is not None else None}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except OSError:
        return {}


def profile_traffic():
    """dram bytes per launch of the keystream kernel from the committed ncu capture."""
    try:
        with open(os.path.join(ROOT, "profiles", "keystream_traffic.json")) as f:
            return json.load(f)
    except OSError:
        return None


# committed ncu --set full capture (tools/gpu_profile.sh) per cipher and mode
TRAFFIC_CAPTURE = {("mickey2", "consume"): "ks_consume", ("mickey2", "materialise"): "ks_rowmajor",
                   ("grain", "consume"): "grain_consume", ("grain", "materialise"): "grain_rowmajor",
                   ("aes128ctr", "consume"): "aes_consume", ("aes128ctr", "materialise"): "aes_rowmajor",
                   ("lfsr128", "consume"): "lfsr_consume", ("lfsr128", "materialise"): "lfsr_rowmajor"}


def traffic_for(cipher, mode, n, launch_bits):
    """(dram read + write bytes per launch, note) for the dominant kernel from
    the committed capture of the same kernel at n instances.  Consume launches
    move only the state carry (same per launch at any bit count); materialise
    writes scale with the bits per launch, so the capture's write bytes are
    scaled by launch_bits / captured bits when the two differ."""
    tr = profile_traffic()
    cap = (tr or {}).get("captures", {}).get(TRAFFIC_CAPTURE.get((cipher, mode), ""))
    if not cap or f"n={n}" not in cap.get("driver", ""):
        return None, None
    import re
    m = re.search(r"bits=(\d+)", cap.get("driver", ""))
    cap_bits = int(m.group(1)) if m else None
    rd, wr = cap["dram_read"], cap["dram_write"]
    note = f"ncu --set full capture '{TRAFFIC_CAPTURE[(cipher, mode)]}' (profiles/, n={n}, {cap_bits} bits per launch)"
    if mode == "materialise" and cap_bits and cap_bits != launch_bits:
        wr *= launch_bits / cap_bits
        note += f"; writes scaled to {launch_bits} bits per launch"
    return rd + wr, note


def state_words(cipher):
    """sliced state rows per 32-instance group (+1 checksum row)"""
    return {"mickey2": 201, "grain": 161, "aes128ctr": 129, "lfsr128": 129}[cipher]


def key_iv_bytes(cipher):
    """device-resident key/IV (counter) bytes per instance read by a rekey"""
    return {"mickey2": 20, "grain": 18, "aes128ctr": 16, "lfsr128": 16}[cipher]


def cpu_cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_sample(n_inst, bits, first=0, threads=None, cipher="mickey2"):
    """Time the oracle (unmodified, bit-serial) on host cores; returns bits/s."""
    import oracle
    from paper_conf_icppw_monfaredhkzrg20_b200 import inputs
    keys, ivs = inputs.make_inputs(cipher, n_inst, first)
    t = time.perf_counter()
    if cipher == "grain":
        oracle.grain_keystream_batch(keys, ivs, bits, threads=threads)
    elif cipher == "lfsr128":
        oracle.lfsr128_keystream_batch(keys, bits, threads=threads)
    elif cipher == "aes128ctr":
        oracle.aes128_ctr_keystream_batch(bytes(inputs.aes_key()), ivs, bits // 128 * 128, threads=threads)
    else:
        oracle.mickey2_keystream_batch(keys, ivs, 80, bits, threads=threads)
    dt = time.perf_counter() - t
    return n_inst * bits / dt, dt


def cpu_baseline(target_s=25.0, cipher="mickey2"):
    """The oracle as it stands, on all host cores, on a bounded sample of the
    workload (its first instances, 2^16 bits each) sized for ~target_s."""
    cores = cpu_cores()
    r0, _ = oracle_sample(2 * cores, 1 << 13, threads=cores, cipher=cipher)  # calibration
    n_s = int(max(cores, min(1 << 16, r0 * target_s / (1 << 16))))
    n_s = (n_s + cores - 1) // cores * cores
    r, dt = oracle_sample(n_s, 1 << 16, threads=cores, cipher=cipher)
    return {"value": r / 1e12, "unit": "Tb/s", "cores": cores, "kind": "oracle",
            "sample": f"instances 0..{n_s - 1} of the workload x 65536 bits ({dt:.1f} s), {cpu_model()}",
            "bits_per_s_per_core": r / cores}


def run_context(local_rank, names=("alu_peak", "curand", "write_peak")):
    """Live context numbers on this GPU: the measured LOP3 issue ceiling (the
    roofline denominator, measured before the timed region), cuRAND on the
    same B200 and the HBM write-only bandwidth (STG.128 / STG.32 streams;
    tools/microbench, built by __graft_entry__.build)."""
    out = {}
    mb = os.path.join(ROOT, "tools", "microbench")
    env = dict(os.environ, CUDA_VISIBLE_DEVICES=os.environ.get("CUDA_VISIBLE_DEVICES", str(local_rank)))
    exes = {"alu_peak": "alu_peak", "curand": "curand_bench", "write_peak": "write_peak"}
    argvs = {"alu_peak": ["200000"], "curand": ["4294967296"], "write_peak": []}
    for name in names:
        argv = argvs[name]
        exe = os.path.join(mb, exes[name])
        if not os.path.exists(exe):
            out[name] = "not built"
            continue
        try:
            r = subprocess.run([exe, *argv], capture_output=True, text=True, timeout=120, env=env)
            out[name] = [json.loads(ln) for ln in r.stdout.splitlines() if ln.startswith("{")]
        except Exception as e:  # pragma: no cover
            out[name] = f"failed: {e}"
    if isinstance(out.get("alu_peak"), list) and out["alu_peak"]:
        out["alu_peak_tlop3_per_s"] = max(x["tlop3_per_s"] for x in out["alu_peak"] if x["variant"] == "lop3")
    if isinstance(out.get("write_peak"), list) and out["write_peak"]:
        out["hbm_write_peak_gbs"] = max(x["write_gbs"] for x in out["write_peak"])
    return out


# ------------------------------------------------------------ reference arm
def workload(args, world):
    """(n_total, bits, scaling, description) of the benchmarked configuration."""
    name = CIPHER_NAME[args.cipher]
    if args.workload == "c2":
        bits = args.bits or BITS_DEFAULT
        n = args.n or N_DEFAULT
        return n * world, bits, "weak", f"configs[1]: {name}, {n} instances x {bits} bits per GPU per step"
    if args.workload == "rekey":
        bits = args.bits or 1024
        n = args.n or N_DEFAULT
        return n * world, bits, "weak", (f"NEXT-3 rekey: {name}, {n} fresh keys/IVs x {bits} bits per GPU per step "
                                         f"(slicing + initialisation clocks + keystream)")
    if args.workload == "c4":
        bits = args.bits or (4480 if args.cipher == "aes128ctr" else 4416)
        n = args.n or (1 << 19)
        return n * world, bits, "weak", (f"configs[3]: {name} at the paper's launch shape (64 x 256 threads x 32 "
                                         f"lanes = {n} instances) x {bits} clocks per GPU per step")
    bits = args.bits or (1 << 18)
    n_total = args.n or (1 << 25)
    return n_total, bits, "strong", (f"configs[2]: {name}, {n_total} instances x {bits} bits in total, "
                                     f"split over {world} GPU(s)")


def run_reference(args, rank, world):
    if rank != 0:
        return
    _, _, scaling, desc = workload(args, world)
    cores = cpu_cores()
    n_s, bits_s = 64 * cores, 1 << 15
    for _ in range(args.warmup):
        oracle_sample(n_s, bits_s, threads=cores, cipher=args.cipher)
    tot_bits, tot_t = 0, 0.0
    for _ in range(args.steps):
        r, dt = oracle_sample(n_s, bits_s, threads=cores, cipher=args.cipher)
        tot_bits += n_s * bits_s
        tot_t += dt
    v = tot_bits / tot_t / 1e12
    line = {
        "impl": "reference", "metric": metric(args), "value": v, "unit": "Tb/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_t / args.steps * 1e3,
        "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "u32",
        "data": "synthetic (SplitMix64 keys/IVs, seed 0x5EED2020)",
        "config": {"workload": f"{desc} ({args.mode})", "mode": args.mode,
                   "reference_step": f"bounded sample: first {n_s} instances x {bits_s} bits, bit-serial oracle"},
        "cpu_baseline": {"value": v, "unit": "Tb/s", "cores": cores, "kind": "oracle",
                         "sample": f"{n_s} instances x {bits_s} bits per step, {cpu_model()}"},
        "e2e": {"value": v, "unit": "Tb/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------- our arm
def run_ours(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist
    from paper_conf_icppw_monfaredhkzrg20_b200 import bsrng, inputs

    from paper_conf_icppw_monfaredhkzrg20_b200 import shard

    # one rank per GPU; with --backend gloo two ranks may share a GPU (tests)
    dev = torch.device("cuda", local_rank % torch.cuda.device_count())
    torch.cuda.set_device(dev)
    coll_dev = dev if (world > 1 and args.backend == "nccl") else None  # gloo reduces CPU tensors
    n_total, bits, scaling, desc = workload(args, world)
    if args.workload in ("c2", "c4", "rekey"):
        first, n = shard.weak_range(rank, n_total // world)
    else:
        first, n = shard.strong_range(rank, world, n_total)
    stream = torch.cuda.Stream(dev)

    # the measured LOP3 issue ceiling on this GPU (roofline denominator)
    peak_ctx = run_context(dev.index, ("alu_peak",)) if rank == 0 and not args.no_context else {}

    keys_h, ivs_h = inputs.make_inputs(args.cipher, n, first)
    if args.cipher == "aes128ctr":
        keys_h = inputs.aes_key()  # one key for every instance
    keys_pin = torch.from_numpy(keys_h).pin_memory()
    ivs_pin = torch.from_numpy(ivs_h).pin_memory()
    keys_d = keys_pin.to(dev)
    ivs_d = ivs_pin.to(dev)

    with torch.cuda.stream(stream):
        g = bsrng.Generator(args.cipher, keys_d, ivs_d, first_instance=first, stream=stream)
    for k, v in (("sched", args.sched), ("seg_clocks", args.seg_clocks), ("ctas_per_sm", args.ctas_per_sm)):
        if v is not None:
            g.set_option(k, v)
    for kv in args.opt:
        k, v = kv.split("=")
        g.set_option(k, int(v))
    cs_out = torch.zeros(1, dtype=torch.int64, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2

    def barrier():
        if world > 1:
            dist.barrier()

    def delay():  # test hook (--test-delay-rank): ~50 ms more on one rank
        if rank == args.test_delay_rank:
            with torch.cuda.stream(stream):
                torch.cuda._sleep(100_000_000)

    def step_consume(ev=None):
        if ev:
            ev[2].record(stream)
        delay()
        g.rekey(keys_d, ivs_d, stream=stream)
        if ev:
            ev[0].record(stream)
        g.generate(cs_out, bits, "checksum", stream=stream)
        if ev:
            ev[1].record(stream)

    chunk = min(args.chunk_bits, bits)
    rm_buf = None

    def step_materialise(ev=None):
        nonlocal rm_buf
        if rm_buf is None:
            rm_buf = torch.empty(g.out_bytes(chunk, "row_major"), dtype=torch.uint8, device=dev)
        if ev:
            ev[2].record(stream)
        g.rekey(keys_d, ivs_d, stream=stream)
        if ev:
            ev[0].record(stream)
        for _ in range(bits // chunk):
            g.generate(rm_buf, chunk, "row_major", stream=stream)
        if ev:
            ev[1].record(stream)

    def timed(step_fn, steps, warmup, sampler=None):
        if sampler:
            sampler.start()
        for _ in range(warmup):
            step_fn()
        torch.cuda.synchronize(dev)
        step_ms, kern_ms, rekey_ms = [], [], []
        l0 = bsrng.launch_count()
        if sampler:
            sampler.begin()
        for _ in range(steps):
            flush.zero_()  # L2 flush between timed steps (outside the timed region)
            torch.cuda.synchronize(dev)
            barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            k0, k1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            r0 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            step_fn((k0, k1, r0))
            e1.record(stream)
            torch.cuda.synchronize(dev)
            barrier()
            step_ms.append(e0.elapsed_time(e1))
            kern_ms.append(k0.elapsed_time(k1))
            rekey_ms.append(r0.elapsed_time(k0))
        if sampler:
            sampler.end()
        clocks = sampler.stop() if sampler else None
        launches = bsrng.launch_count() - l0
        # MAX over ranks of each rank's summed step / kernel / rekey times
        t = [shard.allreduce_max(sum(x), device=coll_dev) for x in (step_ms, kern_ms, rekey_ms)]
        timed.rekey_ms = t[2] / steps
        timed.rank_ms = sum(step_ms) / steps
        return t[0] / steps, t[1] / steps, launches, clocks

    peaks = measured_peaks()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    derived_peak = nsm * ALU_LANES_PER_SM_CLK * sm_max * 1e6 / 1e12
    measured_peak = peak_ctx.get("alu_peak_tlop3_per_s")

    def init_roofline(rk_ms):
        """a-1 + a-2 (bsrng_rekey) against the same ALU peak: initialisation
        clocks x ops per clock (MICKEY 260 x 306 with the deferred R reduction
        -- 328 in Galois form: 304 - 1 output + u = INPUT_BIT ^ s50 + its XOR
        into the pending word + FEEDBACK_S --, Grain 160 x 39; AES-CTR has no
        initialisation clocks, only slicing + a one-warp key expansion)."""
        ops = {"mickey2": 260 * 306.0, "grain": 160 * 39.0}.get(args.cipher)
        if not ops or rk_ms <= 0:
            return None
        achieved = ops * (n // 32) / (rk_ms * 1e-3) / 1e12
        return {"bound": "alu", "achieved": achieved, "peak": derived_peak, "unit": "TLOP3/s",
                "frac": achieved / derived_peak, "note": "rekey = fused slicing + initialisation kernel"}

    def roofline(kern_ms_per_step, clocks, mode):
        """achieved = ALGORITHMIC LOP3 (the sec. 8(d) per-clock
        count x groups x clocks) / the keystream kernel's CUDA-event time,
        against the LOP3 ceiling measured in this run (tools/microbench/alu_peak,
        before the timed region); the derived 148 x 64 lanes x sm_max peak and
        the kernel's own op count are reported beside it."""
        unroll = dict(kv.split("=", 1) for kv in args.opt).get("unroll")
        alg = algorithmic_ops(args.cipher, mode)
        kops = lop3_per_bit(args.cipher, mode, int(unroll) if unroll else None)
        units = (n // 32) * bits / (kern_ms_per_step * 1e-3) / 1e12  # group-clocks per s, x 1e12
        peak = measured_peak or derived_peak
        out = {"bound": "alu", "achieved": alg * units, "peak": peak, "unit": "TLOP3/s",
               "frac": alg * units / peak,
               "peak_basis": ("measured in this run: tools/microbench/alu_peak (independent lop3.b32 chains on "
                              "every SM)" if measured_peak else
                              f"derived: {nsm} SMs x {ALU_LANES_PER_SM_CLK} LOP3 lanes/clk x sm_max {sm_max:.0f} "
                              "MHz (alu_peak not run)"),
               "ops_per_clock_algorithmic": alg,
               "ops_per_clock_basis": "SURVEY.md sec. 8(d) / App. D per-clock LOP3 count",
               "ops_per_clock_kernel": kops,
               "frac_kernel_ops": kops * units / peak,
               "peak_derived": derived_peak,
               "frac_vs_derived_peak": alg * units / derived_peak,
               "traffic": None}
        if clocks and clocks.get("sm_mhz"):
            out["frac_at_sampled_clock"] = alg * units / (nsm * ALU_LANES_PER_SM_CLK * clocks["sm_mhz"] * 1e6 / 1e12)
        if mode == "materialise":
            # roofline choice by arithmetic intensity: LOP3 per byte written
            # (4 B per group-clock) against the ridge = LOP3 peak / HBM peak.
            # The LFSR's 2 LOP3 per 4 B sit far left of the ridge: its ROW_MAJOR
            # line is bound by HBM writes, the other ciphers' by the ALU.
            hbm = float(peaks.get("hbm_gbs", 6467.7))
            intensity = alg / 4.0
            ridge = peak * 1e12 / (hbm * 1e9)
            wr_gbs = units * 1e12 * 4 / 1e9  # bytes written per s
            out["lop3_per_byte"] = intensity
            out["ridge_lop3_per_byte"] = ridge
            out["hbm_write_gbs"] = wr_gbs
            out["hbm_frac"] = wr_gbs / hbm
            if intensity < ridge:
                out.update({"bound": "hbm", "achieved": wr_gbs, "peak": hbm, "unit": "GB/s",
                            "frac": wr_gbs / hbm,
                            "alu_frac": alg * units / peak,
                            "peak_basis": "MEASURED_PEAKS.json hbm_gbs (copy bandwidth, read + write)"})
        return out

    results = {}
    modes = [args.mode] + ([] if args.no_other_mode else [m for m in ("consume", "materialise") if m != args.mode])
    for mode in modes:
        fn = step_consume if mode == "consume" else step_materialise
        sampler = ClockSampler(dev.index) if rank == 0 else None
        ms, kms, launches, clocks = timed(fn, args.steps, args.warmup, sampler)
        tbps = n_total * bits / (ms * 1e-3) / 1e12
        rk_ms = timed.rekey_ms
        res = {"value": tbps, "ms_per_step": ms, "kernel_ms_per_step": kms,
               "rekey_ms_per_step": rk_ms, "keys_per_s": n_total / (rk_ms * 1e-3) if rk_ms > 0 else None,
               "preclock_roofline": init_roofline(rk_ms),
               "kernel_tbps_per_gpu": n * bits / (kms * 1e-3) / 1e12,
               "gpu_launches": launches, "roofline": roofline(kms, clocks, mode)}
        if world > 1:
            res["rank0_ms_per_step"] = timed.rank_ms
        if mode == "materialise":
            out_bytes = n * bits / 8
            res["hbm_write_gbs_per_gpu"] = out_bytes / (kms * 1e-3) / 1e9
            res["hbm_write_frac"] = res["hbm_write_gbs_per_gpu"] / float(peaks.get("hbm_gbs", 6650.0))
            res["calls_per_step"] = bits // chunk
        if clocks:
            res["clocks"] = clocks
        results[mode] = res

    # checksum of one consume step (sharding invariant), outside the timed region
    step_consume()
    torch.cuda.synchronize(dev)
    local_cs = int(cs_out.item()) & shard.MASK64
    checksum = shard.allreduce_checksum(local_cs, device=coll_dev)

    # e2e through the public API: host keys (pinned) -> bsrng_rekey (staged
    # H2D inside the call) -> bsrng_generate_host(CHECKSUM): the keystream
    # kernel plus the 8 B device->host read of the result, stream-synchronised
    e2e = None
    if not args.no_e2e:
        cs_host = np.zeros(1, dtype=np.uint64)
        kh, vh = keys_pin.numpy(), ivs_pin.numpy()

        def step_e2e(ev=None):
            if ev:
                ev[2].record(stream)
            g.rekey(kh, vh, stream=stream)
            if ev:
                ev[0].record(stream)
            cs_host[:] = g.generate_host(bits, "checksum", stream=stream)
            if ev:
                ev[1].record(stream)

        ms_e2e, _, _, _ = timed(step_e2e, max(1, args.steps), 1)
        e2e = {"value": n_total * bits / (ms_e2e * 1e-3) / 1e12, "unit": "Tb/s",
               "h2d_bytes_per_step": int(keys_h.nbytes + ivs_h.nbytes), "d2h_bytes_per_step": 8,
               "ms_per_step": ms_e2e, "mode": "consume",
               "api": "bsrng_rekey(host keys/IVs) + bsrng_generate_host(CHECKSUM)",
               "checksum_matches_device_path": bool(int(cs_host[0]) == local_cs)}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(cipher=args.cipher)
    context = None
    if rank == 0 and world == 1 and not args.no_context:
        context = dict(peak_ctx, **run_context(dev.index, ("curand", "write_peak")))

    if rank == 0:
        head = results[args.mode]
        rf = head["roofline"]
        for mode, res in results.items():
            lb = bits if mode == "consume" else min(bits, args.chunk_bits)
            t, note = traffic_for(args.cipher, mode, n, lb)
            if t is not None:
                res["roofline"]["traffic"] = t
                res["roofline"]["traffic_note"] = note
        line = {
            "metric": metric(args), "value": head["value"], "unit": "Tb/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": head["ms_per_step"],
            "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "u32",
            "data": "synthetic (SplitMix64 keys/IVs, seed 0x5EED2020)",
            "config": {"workload": f"{desc} ({args.mode})", "instances_total": n_total,
                       "instances_per_gpu": n, "bits_per_instance": bits,
                       "mode": args.mode, "parallelism": f"instance-range shards x{world}",
                       "backend": args.backend if world > 1 else None,
                       "l2": (f"flushed (256 MiB write) between timed steps; state "
                              f"{state_words(args.cipher) * (n // 32) * 4 / 2**20:.0f} MiB, keys/IVs "
                              f"{n * key_iv_bytes(args.cipher) / 2**20:.0f} MiB")},
            "roofline": rf, "clocks": head.get("clocks"), "gpu_launches": head["gpu_launches"],
            "e2e": e2e, "cpu_baseline": cpu, "checksum": f"{checksum:016x}", "context": context,
            "modes": {m: {k: v for k, v in r.items() if k != "clocks"} for m, r in results.items()},
            "clocks_by_mode": {m: r.get("clocks") for m, r in results.items()},
            "paper_context": "2.72 Tb/s RTX 2080 Ti, 2.90 Tb/s V100 (PAPER.md:46-50, 852-854); "
                             "exceeds the bit-exact LOP3 bound on those GPUs, see BASELINE.md",
        }
        print(json.dumps(line), flush=True)
    g.close()


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus and world == 1 and args.gpus > 1:
        print(f"--gpus {args.gpus} needs torchrun (WORLD_SIZE={world})", file=sys.stderr)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        dev = torch.device("cuda", local_rank % max(1, torch.cuda.device_count()))
        torch.cuda.set_device(dev)
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
    try:
        run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
