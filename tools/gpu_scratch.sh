#!/bin/bash
# rm_phase (staggered 64 B flush periods in the writer-warp kernel): parity, then
# Grain / MICKEY paper shape ROW_MAJOR with and without it
set -u
D=gpurun_out/g6; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_api.py tests/test_gpu_random.py tests/test_gpu_rowmajor_items.py -m gpu -q -x -p no:cacheprovider > $D/pytest.txt 2>&1
echo "pytest exit $?" >> $D/pytest.txt
for c in grain mickey2; do
  B="python bench.py --cipher $c --workload c4 --mode materialise --no-other-mode --no-cpu-baseline --no-e2e --no-context --steps 1000 --warmup 20"
  for ph in 1 0 1 0; do
    timeout 300 $B --opt rm_phase=$ph > $D/c4_${c}_ph$ph.json 2> $D/c4_${c}_ph$ph.err
    python -c "import json; d=json.load(open('$D/c4_${c}_ph$ph.json')); print('$c phase=$ph', round(d['value'],3), d['modes']['materialise']['kernel_ms_per_step'])" >> $D/summary.txt 2>&1
  done
done
