#!/bin/bash
mkdir -p gpurun_out/sel
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > gpurun_out/sel/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/sel/pytest_gpu.txt
timeout 900 python bench.py --cipher grain --no-cpu-baseline --no-context --no-e2e > gpurun_out/sel/c2_grain.json 2>&1
timeout 900 python bench.py --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode > gpurun_out/sel/c2_mickey_mat.json 2>&1
timeout 900 python bench.py --cipher aes128ctr --no-cpu-baseline --no-context --no-e2e > gpurun_out/sel/c2_aes.json 2>&1
