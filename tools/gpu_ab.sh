#!/bin/bash
# A/B of the ROW_MAJOR kernel: current tree vs the worktree in _ab (same box)
D=gpurun_out/ab; mkdir -p $D; rm -f $D/res.txt
for rep in 1 2; do
for side in cur ab; do
  dir=.; [ $side = ab ] && dir=_ab
  echo "== $side rep $rep" >> $D/res.txt
  (cd $dir && timeout 600 python bench.py --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode --steps 3 --warmup 3) 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); m=d['modes']['materialise']; print(round(m['value'],4), round(m['roofline']['frac'],4))" >> $D/res.txt 2>&1
done; done
