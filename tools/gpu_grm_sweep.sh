#!/bin/bash
D=gpurun_out/grm_sweep; mkdir -p $D
timeout 600 python -m pytest tests/test_gpu_grain.py tests/test_gpu_mickey2.py -q -p no:cacheprovider -x > $D/pytest.txt 2>&1
for o in "" "--opt rm_zreg=0" "--opt unroll=16" "--opt rm_zreg=0 --opt unroll=16" "--opt rm_zreg=0 --opt unroll=8" "--opt seg_clocks=4096" "--opt seg_clocks=32768"; do
  echo "== $o" >> $D/res.txt
  timeout 600 python bench.py --cipher grain --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode --steps 3 --warmup 3 $o 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); m=d['modes']['materialise']; print(round(m['value'],3), round(m['roofline']['frac'],3))" >> $D/res.txt 2>&1
done
