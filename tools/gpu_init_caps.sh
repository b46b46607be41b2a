#!/bin/bash
# init-kernel captures (-s 0: one launch per process) + bench lines that read
# the regenerated keystream_traffic.json
mkdir -p gpurun_out/prof2 gpurun_out/bench2
cap() {
  name=$1; shift
  ncu --set full --clock-control none --import-source on -k regex:$1 -s 0 -c 1 -o /tmp/prof_$name "${@:2}" > gpurun_out/prof2/ncu_$name.log 2>&1
  ncu -i /tmp/prof_$name.ncu-rep --page raw --csv > gpurun_out/prof2/${name}_raw.csv 2>/dev/null
  ncu -i /tmp/prof_$name.ncu-rep --page details --csv > gpurun_out/prof2/${name}_details.csv 2>/dev/null
  rm -f /tmp/prof_$name.ncu-rep
}
cap preclock m2_init python tools/prof_driver.py --layout checksum --bits 32 --reps 1
cap grain_init grain_init python tools/prof_driver.py --cipher grain --layout checksum --bits 32 --reps 1
cp gpurun_out/prof2/../prof/gpu.txt gpurun_out/prof2/ 2>/dev/null
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > gpurun_out/prof2/gpu.txt
timeout 900 python bench.py > gpurun_out/bench2/n1_default.json 2> gpurun_out/bench2/n1_default.err
for c in grain aes128ctr; do
  timeout 600 python bench.py --cipher $c --no-context > gpurun_out/bench2/c2_$c.json 2>&1
done
