#!/bin/bash
D=gpurun_out/sect; mkdir -p $D
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $D/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> $D/pytest_gpu.txt
timeout 900 python bench.py --cipher grain --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode > $D/grain_mat.json 2>&1
timeout 900 python bench.py --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode > $D/mickey_mat.json 2>&1
timeout 900 python bench.py --cipher grain --workload c4 --no-cpu-baseline --no-context --no-e2e > $D/grain_c4.json 2>&1
