#!/bin/bash
# two-writer kernel: four blocks per writer step (WS2_QUAD build).  Parity with that build, then A/B.
set -u
D=gpurun_out/g17; mkdir -p $D
BSRNG_LIB=tools/experiments/ab/quad.so timeout 900 python -m pytest tests/test_gpu_api.py tests/test_gpu_random.py tests/test_gpu_rowmajor_items.py tests/test_gpu_lfsr.py -m gpu -q -p no:cacheprovider > $D/pytest.txt 2>&1
echo "pytest exit $?" >> $D/pytest.txt
run() {  # name lib args...
  local name=$1 lib=$2; shift 2
  BSRNG_LIB=$lib timeout 300 python bench.py --mode materialise --no-other-mode --no-cpu-baseline --no-e2e --no-context "$@" > $D/$name.json 2> $D/$name.err
  python -c "import json; d=json.load(open('$D/$name.json')); print('$name', round(d['value'],3), d['modes']['materialise']['kernel_ms_per_step'])" >> $D/summary.txt 2>&1
}
for rep in 1 2; do
  for v in quad old; do
    run lfsr_$v tools/experiments/ab/$v.so --cipher lfsr128 --steps 20 --warmup 3
  done
done
