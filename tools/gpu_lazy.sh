#!/bin/bash
# Deferred-reduction MICKEY: parity + bench
mkdir -p gpurun_out/lazy
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > gpurun_out/lazy/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/lazy/pytest_gpu.txt
timeout 900 python bench.py --no-cpu-baseline --no-context > gpurun_out/lazy/bench.json 2> gpurun_out/lazy/bench.err
timeout 600 python bench.py --no-cpu-baseline --no-context --no-e2e --opt unroll=8 --no-other-mode > gpurun_out/lazy/bench_u8.json 2>&1
