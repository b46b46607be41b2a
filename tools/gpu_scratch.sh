#!/bin/bash
# lane-major z blocks (STS.128 / LDS.128) in the writer-warp kernels: parity, then A/B vs the
# previous build (tools/experiments/ab/old.so) on the writer-warp workloads
set -u
D=gpurun_out/g7; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_api.py tests/test_gpu_random.py tests/test_gpu_rowmajor_items.py tests/test_gpu_lfsr.py -m gpu -q -x -p no:cacheprovider > $D/pytest.txt 2>&1
echo "pytest exit $?" >> $D/pytest.txt
run() {  # name lib args...
  local name=$1 lib=$2; shift 2
  BSRNG_LIB=$lib timeout 300 python bench.py --mode materialise --no-other-mode --no-cpu-baseline --no-e2e --no-context "$@" > $D/$name.json 2> $D/$name.err
  python -c "import json; d=json.load(open('$D/$name.json')); print('$name', round(d['value'],3), d['modes']['materialise']['kernel_ms_per_step'])" >> $D/summary.txt 2>&1
}
for rep in 1 2; do
  for v in new old; do
    lib=""; [ $v = old ] && lib=tools/experiments/ab/old.so
    run c4_grain_$v "$lib" --cipher grain --workload c4 --steps 1000 --warmup 20
    run c4_mickey_$v "$lib" --cipher mickey2 --workload c4 --steps 300 --warmup 10
    run lfsr_ws2_$v "$lib" --cipher lfsr128 --steps 20 --warmup 3
    run lfsr_ws1_$v "$lib" --cipher lfsr128 --steps 20 --warmup 3 --opt rm_ws=1
  done
done
