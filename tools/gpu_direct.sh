#!/bin/bash
D=gpurun_out/direct; mkdir -p $D
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $D/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> $D/pytest_gpu.txt
python tools/rekey_split.py > $D/rekey.txt 2>&1
for c in mickey2 grain aes128ctr; do
timeout 600 python bench.py --cipher $c --workload rekey --no-cpu-baseline --no-context --no-e2e --no-other-mode > $D/rekey_$c.json 2>&1
done
