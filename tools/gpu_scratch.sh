#!/bin/bash
# Grain at the paper shape (configs[3]) ROW_MAJOR: writer-warp kernel A/B
# (builds in tools/experiments/ab/, made with build.py -D... --out=...)
set -u
D=gpurun_out/g4; mkdir -p $D
B="python bench.py --cipher grain --workload c4 --mode materialise --no-other-mode --no-cpu-baseline --no-e2e --no-context --steps 1000 --warmup 20"
for v in base nw nf s0 s1000 g8 g2 base; do
  if [ $v = base ]; then lib=""; else lib=tools/experiments/ab/$v.so; fi
  BSRNG_LIB=$lib timeout 300 $B > $D/c4_$v.json 2> $D/c4_$v.err
  python -c "import json,sys; d=json.load(open('$D/c4_$v.json')); print('$v', round(d['value'],3), d['modes']['materialise']['kernel_ms_per_step'] if 'modes' in d else '')" >> $D/summary.txt 2>&1
done
# consume at the same shape for the lone-warp issue rate
BSRNG_LIB= timeout 300 python bench.py --cipher grain --workload c4 --no-other-mode --no-cpu-baseline --no-e2e --no-context --steps 1000 --warmup 20 > $D/c4_consume.json 2>&1
export SASS=1
bash tools/gpu.sh capture g4 grain_c4_ws keystream_rm_ws --cipher grain --layout row_major --n 524288 --bits 4416 --reps 2
