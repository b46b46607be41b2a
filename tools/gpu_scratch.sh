#!/bin/bash
# two-writer kernel: stages 16 + 8 of the transposes in the clock-loop warp (WS2_PRE8 build).  Parity, A/B.
set -u
D=gpurun_out/g22; mkdir -p $D
BSRNG_LIB=tools/experiments/ab/pre8.so timeout 900 python -m pytest tests/test_gpu_lfsr.py tests/test_gpu_bounds.py tests/test_gpu_rowmajor_items.py tests/test_gpu_random.py tests/test_gpu_api.py -m gpu -q -p no:cacheprovider > $D/pytest_pre8.txt 2>&1
echo "pytest exit $?" >> $D/pytest_pre8.txt
timeout 600 python -m pytest tests/test_gpu_aes.py -m gpu -q -p no:cacheprovider > $D/pytest_aes.txt 2>&1
echo "pytest exit $?" >> $D/pytest_aes.txt
run() {  # name lib args...
  local name=$1 lib=$2; shift 2
  BSRNG_LIB=$lib timeout 300 python bench.py --no-other-mode --no-cpu-baseline --no-e2e --no-context "$@" > $D/$name.json 2> $D/$name.err
  python -c "import json; d=json.load(open('$D/$name.json')); print('$name', round(d['value'],3), [m['kernel_ms_per_step'] for m in d['modes'].values() if m])" >> $D/summary.txt 2>&1
}
for rep in 1 2; do
  for v in pre8 old; do
    run lfsr_$v tools/experiments/ab/$v.so --mode materialise --cipher lfsr128 --steps 20 --warmup 3
  done
done
