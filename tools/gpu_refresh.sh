#!/bin/bash
# Round refresh: GPU tests, smoke, default bench line (+ reference arm).
mkdir -p gpurun_out/refresh
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/refresh/gpu.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/refresh/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/refresh/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/refresh/smoke.txt 2>&1
timeout 1200 python bench.py > gpurun_out/refresh/bench_default.json 2> gpurun_out/refresh/bench_default.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/refresh/bench_reference.json 2> gpurun_out/refresh/bench_reference.err
