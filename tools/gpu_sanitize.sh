#!/bin/bash
# compute-sanitizer over every kernel path (SURVEY sec. 5 race detection)
D=gpurun_out/sanitize; mkdir -p $D
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_driver.py > $D/$tool.txt 2>&1
  echo "exit $?" >> $D/$tool.txt
done
