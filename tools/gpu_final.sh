#!/bin/bash
# Final round record: GPU tests, smoke, default bench (+ reference arm), C4 lines
D=gpurun_out/final; mkdir -p $D
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > $D/gpu.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $D/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> $D/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $D/smoke.txt 2>&1
timeout 1200 python bench.py > $D/n1_default.json 2> $D/n1_default.err
timeout 600 python bench.py --impl reference > $D/n1_reference.json 2> $D/n1_reference.err
for c in mickey2 grain aes128ctr; do
  timeout 600 python bench.py --cipher $c --workload c4 --no-context --no-cpu-baseline --no-e2e > $D/c4_$c.json 2>&1
done
