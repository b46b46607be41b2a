#!/bin/bash
# two-writer kernel: 16-byte meta records (one STS.128 / LDS.128).  Parity, A/B.
set -u
D=gpurun_out/g29; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_lfsr.py tests/test_gpu_api.py tests/test_gpu_random.py tests/test_gpu_rowmajor_items.py tests/test_gpu_bounds.py -m gpu -q -p no:cacheprovider > $D/pytest.txt 2>&1
echo "pytest exit $?" >> $D/pytest.txt
run() {  # name lib args...
  local name=$1 lib=$2; shift 2
  BSRNG_LIB=$lib timeout 300 python bench.py --no-other-mode --no-cpu-baseline --no-e2e --no-context "$@" > $D/$name.json 2> $D/$name.err
  python -c "import json; d=json.load(open('$D/$name.json')); print('$name', round(d['value'],3), [m['kernel_ms_per_step'] for m in d['modes'].values() if m])" >> $D/summary.txt 2>&1
}
for rep in 1 2; do
  for v in new old; do
    lib=""; [ $v = old ] && lib=tools/experiments/ab/old.so
    run lfsr_$v "$lib" --mode materialise --cipher lfsr128 --steps 20 --warmup 3
  done
done
