#!/bin/bash
# L2 evict_last on a fraction of the addresses (createpolicy.fractional f): Grain C2 / paper shape, LFSR C2 ROW_MAJOR
set -u
D=gpurun_out/g30; mkdir -p $D
run() {  # name lib args...
  local name=$1 lib=$2; shift 2
  BSRNG_LIB=$lib timeout 300 python bench.py --no-other-mode --no-cpu-baseline --no-e2e --no-context "$@" > $D/$name.json 2> $D/$name.err
  python -c "import json; d=json.load(open('$D/$name.json')); print('$name', round(d['value'],3), [m['kernel_ms_per_step'] for m in d['modes'].values() if m])" >> $D/summary.txt 2>&1
}
for rep in 1 2; do
  for v in base f0.5 f0.75 f0.875; do
    lib=""; [ $v != base ] && lib=tools/experiments/ab/$v.so
    run c2_grain_$v "$lib" --mode materialise --cipher grain --steps 4 --warmup 3
    run lfsr_$v "$lib" --mode materialise --cipher lfsr128 --steps 20 --warmup 3
    run c4_grain_$v "$lib" --mode materialise --cipher grain --workload c4 --steps 1000 --warmup 20
  done
done
