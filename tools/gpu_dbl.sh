#!/bin/bash
D=gpurun_out/dbl; mkdir -p $D; rm -f $D/res.txt
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $D/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> $D/pytest_gpu.txt
run() {
  c=$1; shift
  echo "== $c $*" >> $D/res.txt
  timeout 300 python bench.py --cipher $c --workload c4 --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode "$@" 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); m=d['modes']['materialise']; print(round(m['value'],3), round(m['roofline']['frac'],3))" >> $D/res.txt 2>&1
}
run mickey2
run mickey2 --opt rm_dbl=0
run grain
run grain --opt rm_dbl=0
timeout 600 python bench.py --no-cpu-baseline --no-context --no-e2e --mode materialise --no-other-mode > $D/c2_mickey_mat.json 2>&1
