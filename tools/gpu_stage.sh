#!/bin/bash
D=gpurun_out/stage; mkdir -p $D
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $D/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> $D/pytest_gpu.txt
python tools/rekey_split.py > $D/rekey.txt 2>&1
ncu --metrics gpu__time_duration.sum,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active --clock-control none --csv --log-file $D/ncu.csv python tools/rekey_split.py > /dev/null 2>&1
for c in grain aes128ctr; do
timeout 600 python bench.py --cipher $c --workload rekey --no-cpu-baseline --no-context --no-e2e --no-other-mode > $D/rekey_$c.json 2>&1
done
