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
    assert bench.lop3_per_bit("mickey2", "consume") == 327
    assert bench.lop3_per_bit("grain", "materialise") == 37
    assert abs(bench.lop3_per_bit("aes128ctr", "materialise") * 4096 / 32 - 17280) < 1e-9
