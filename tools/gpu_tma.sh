#!/bin/bash
D=gpurun_out/tma; mkdir -p $D
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $D/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> $D/pytest_gpu.txt
for o in "" "--opt rm_tma=0"; do
  echo "== grain $o" >> $D/res.txt
  timeout 600 python bench.py --cipher grain --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode $o 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); m=d['modes']['materialise']; print(round(m['value'],3), round(m['roofline']['frac'],3))" >> $D/res.txt 2>&1
  echo "== mickey2 $o" >> $D/res.txt
  timeout 600 python bench.py --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode $o 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); m=d['modes']['materialise']; print(round(m['value'],3), round(m['roofline']['frac'],3))" >> $D/res.txt 2>&1
done
