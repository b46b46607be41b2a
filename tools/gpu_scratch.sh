#!/bin/bash
# final tree: GPU tests + smoke + the driver's default bench command
set -u
bash tools/gpu.sh tests r2j
timeout 900 python bench.py > gpurun_out/r2j/bench_default.json 2> gpurun_out/r2j/bench_default.err
echo "bench exit $?" >> gpurun_out/r2j/pytest_gpu.txt
