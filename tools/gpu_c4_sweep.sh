#!/bin/bash
D=gpurun_out/c4s; mkdir -p $D; rm -f $D/res.txt
run() {  # cipher opts...
  c=$1; shift
  echo "== $c $*" >> $D/res.txt
  timeout 300 python bench.py --cipher $c --workload c4 --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode "$@" 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); m=d['modes']['materialise']; print(round(m['value'],3), round(m['roofline']['frac'],3), round(m['ms_per_step'],3))" >> $D/res.txt 2>&1
}
run grain
run grain --opt seg_clocks=4608
run grain --opt seg_clocks=1024
run grain --opt ctas_per_sm=1
run grain --opt ctas_per_sm=1 --opt seg_clocks=4608
run grain --opt rm_tmem=0
run mickey2
run mickey2 --opt seg_clocks=1024
run mickey2 --opt ctas_per_sm=1
run aes128ctr
