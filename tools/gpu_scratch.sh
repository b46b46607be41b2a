#!/bin/bash
# final check after the AES side-stream change: full GPU tests + smoke, AES paper-shape line as in the record
set -u
bash tools/gpu.sh tests r2i
bash tools/gpu.sh bench r2i c4_aes128ctr --cipher aes128ctr --workload c4 --no-cpu-baseline --no-e2e --steps 2000 --warmup 20
