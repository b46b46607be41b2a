"""bench.py pieces that run without a GPU: the reference arm (the CPU oracle on
a bounded sample) prints one valid JSON line with the contract's keys, and
the workload table matches BASELINE.json's configs."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


@pytest.mark.parametrize("cipher", ["mickey2", "grain", "aes128ctr"])
def test_reference_arm_json(cipher):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--cipher", cipher,
                        "--steps", "1", "--warmup", "0"], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr
    line = json.loads(r.stdout.strip().splitlines()[-1])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "dtype", "config", "cpu_baseline", "e2e"):
        assert k in line, k
    assert line["impl"] == "reference" and line["value"] > 0 and line["unit"] == "Tb/s"
    assert line["cpu_baseline"]["kind"] == "oracle"
    assert line["e2e"]["h2d_bytes_per_step"] == 0


def test_workloads_match_baseline_configs():
    class A:
        cipher, n, bits = "mickey2", None, None
    a = A()
    a.workload = "c2"
    n_total, bits, scaling, desc = bench.workload(a, 1)
    assert (n_total, bits, scaling) == (1 << 22, 1 << 20, "weak")       # configs[1]
    a.workload = "c3"
    n_total, bits, scaling, _ = bench.workload(a, 8)
    assert n_total * bits == 1 << 43 and scaling == "strong"            # configs[2]: 1 TiB
    a.workload = "c4"
    n_total, bits, _, _ = bench.workload(a, 1)
    assert (n_total, bits) == (64 * 256 * 32, 4416)                     # configs[3]: paper shape


def test_op_counts():
    assert bench.lop3_per_bit("mickey2", "consume") == 304          # deferred R reduction, K = 4
    assert bench.lop3_per_bit("mickey2", "consume", unroll=2) == 315.5
    assert bench.MICKEY2_GALOIS_OPS == 327
    assert bench.lop3_per_bit("grain", "materialise") == 37
    assert abs(bench.lop3_per_bit("aes128ctr", "materialise") * 4096 / 32 - 16848) < 1e-9   # MC as 84 LOP3
    assert bench.algorithmic_ops("aes128ctr", "consume") * 128 == 17280                       # sec. 8(d) count
    assert bench.algorithmic_ops("mickey2", "materialise") == 327 and bench.algorithmic_ops("grain", "consume") == 39


# --- the deferred Galois reduction of MICKEY 2.0's R (mickey2.cuh clock_lazy) ---
# RTAPS of the MICKEY 2.0 specification (ref [5]), as tap positions.
_RTAPS = [0, 1, 3, 4, 5, 6, 9, 12, 13, 16, 19, 20, 21, 22, 25, 28, 37, 38, 41, 42, 45, 46, 50, 52, 54, 56, 58, 60,
          61, 63, 64, 65, 66, 67, 71, 72, 79, 80, 81, 82, 87, 88, 89, 90, 91, 92, 94, 95, 96, 97]


def _q_masks(k):
    """Q_m = x^(100+m) mod p(x) as 100-bit integers, m < k."""
    p_low = sum(1 << t for t in _RTAPS)
    out, cur = [], p_low
    for _ in range(k):
        out.append(cur)
        cur <<= 1
        if cur >> 100:
            cur = (cur & ((1 << 100) - 1)) ^ p_low
    return out


def _lazy_ops(k):
    """LOP3 per clock of the implemented schedule (pairs of overflow words)."""
    import math
    if k == 1:
        return 327.0
    Q = _q_masks(k)
    bit = lambda m, q: (Q[m] >> q) & 1
    shift = sum(100 + j for j in range(k))
    corr = 0
    for j in range(k):
        for q, base in ((67, 2), (33, 2), (0, 3)):
            t = sum(bit(m, q) for m in range(j))
            corr += math.ceil((base + t - 1) / 2) - math.ceil((base - 1) / 2)
    pairs = [[2 * p, 2 * p + 1] if 2 * p + 1 < k else [2 * p] for p in range((k + 1) // 2)]
    pre = sum(1 for g in pairs if len(g) == 2 and any(bit(g[0], q) and bit(g[1], q) for q in range(100)))
    red = sum(math.ceil(sum(1 for g in pairs if any(bit(m, q) for m in g)) / 2) for q in range(100))
    return 327 - 149 + (shift + corr + red + pre) / k


def test_mickey2_deferred_reduction_op_counts():
    for k in (1, 2, 4):
        assert _lazy_ops(k) == bench.MICKEY2_OPS_BY_BLOCK[k], k


def test_mickey2_deferred_reduction_equals_galois_clocking():
    """(x + c) * R mod p clocked K times unreduced, then folded with Q_m, equals
    K Galois clocks of the spec (r'_i = r_{i-1} ^ [i in RTAPS] (r99 ^ u) ^ c r_i,
    u = INPUT_BIT ^ s50 when mixing, else 0), with the taps r0 / r33 / r67 read
    mid-block through their pending terms."""
    import random
    rng = random.Random(2020)
    taps = set(_RTAPS)
    for k in (2, 4):
        Q = _q_masks(k)
        for _ in range(200):
            R = rng.getrandbits(100)
            ctl = [rng.getrandbits(1) for _ in range(k)]
            # MIXING (initialisation): u = INPUT_BIT ^ s50 joins the feedback
            mix = [rng.getrandbits(1) if k == 4 else 0 for _ in range(k)]
            # Galois (spec) clocks, recording r0/r33/r67 before each clock
            g, seen_g = R, []
            for c, u in zip(ctl, mix):
                seen_g.append(((g >> 0) & 1, (g >> 33) & 1, (g >> 67) & 1))
                r99 = ((g >> 99) & 1) ^ u
                nxt = 0
                for i in range(100):
                    v = ((g >> (i - 1)) & 1 if i else 0) ^ (r99 if i in taps else 0) ^ (c & (g >> i) & 1)
                    nxt |= v << i
                g = nxt
            # deferred: P' = (x + c) P, unreduced; taps read with pending terms
            P, seen_l = R, []
            for j, c in enumerate(ctl):
                pend = [(P >> (100 + m)) & 1 for m in range(j)]
                true = lambda q: ((P >> q) & 1) ^ (sum(pend[m] & ((Q[m] >> q) & 1) for m in range(j)) & 1)
                seen_l.append((true(0), true(33), true(67)))
                P = (P << 1) ^ (P if c else 0) ^ (mix[j] << 100)  # u * x^100 == u * sum RTAPS x^t
            low = P & ((1 << 100) - 1)
            for m in range(k):
                if (P >> (100 + m)) & 1:
                    low ^= Q[m]
            assert P >> (100 + k) == 0
            assert low == g and seen_l == seen_g


def test_reference_arm_under_torchrun_world2():
    """The driver launches the reference arm like ours for N > 1: rank 0 alone
    runs the oracle and prints the one JSON line, the other rank exits 0."""
    import socket
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                        "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(ROOT, "bench.py"),
                        "--impl", "reference", "--gpus", "2", "--steps", "1", "--warmup", "0"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    line = json.loads(lines[0])
    assert line["impl"] == "reference" and line["value"] > 0 and line["n_gpus"] == 2


def test_roofline_traffic_from_committed_captures():
    """roofline.traffic comes from the committed ncu capture of the same
    cipher and mode (profiles/keystream_traffic.json); materialise writes
    scale with the bits per launch."""
    for cipher, mode, bits in [("mickey2", "consume", 1 << 20), ("mickey2", "materialise", 1 << 15),
                               ("grain", "consume", 1 << 20), ("grain", "materialise", 1 << 15),
                               ("aes128ctr", "materialise", 1 << 15)]:
        t, note = bench.traffic_for(cipher, mode, 1 << 22, bits)
        assert t is not None and t > 0 and note, (cipher, mode)
        if mode == "materialise":
            alg = (1 << 22) * bits / 8
            assert 0.95 * alg < t < 1.2 * alg, (cipher, t / alg)   # ~1.0x the keystream bytes
    assert bench.traffic_for("mickey2", "consume", 1 << 19, 1 << 20) == (None, None)  # other n: no capture
