#!/bin/bash
D=gpurun_out/aesrem; mkdir -p $D
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $D/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> $D/pytest_gpu.txt
timeout 300 python bench.py --cipher aes128ctr --workload c4 --no-cpu-baseline --no-context --no-e2e > $D/c4_aes.json 2>&1
timeout 300 python bench.py --cipher grain --workload c4 --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode --opt rm_ws=1 > $D/c4_grain_ws.json 2>&1
timeout 300 python bench.py --workload c4 --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode --opt rm_ws=1 > $D/c4_mickey_ws.json 2>&1
