#!/bin/bash
D=gpurun_out/dbl2; mkdir -p $D; rm -f $D/res.txt
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $D/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> $D/pytest_gpu.txt
for rep in 1 2; do
  echo "== c2 mickey materialise" >> $D/res.txt
  timeout 600 python bench.py --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); m=d['modes']['materialise']; print(round(m['value'],4), round(m['roofline']['frac'],4))" >> $D/res.txt 2>&1
done
for c in mickey2 grain; do
  echo "== c4 $c materialise" >> $D/res.txt
  timeout 300 python bench.py --cipher $c --workload c4 --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); m=d['modes']['materialise']; print(round(m['value'],4), round(m['roofline']['frac'],4))" >> $D/res.txt 2>&1
done
