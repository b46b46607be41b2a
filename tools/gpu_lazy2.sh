#!/bin/bash
mkdir -p gpurun_out/lazy2
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > gpurun_out/lazy2/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/lazy2/pytest_gpu.txt
timeout 600 python bench.py --workload rekey --no-cpu-baseline --no-context --no-e2e --no-other-mode > gpurun_out/lazy2/rekey_mickey2.json 2>&1
