#!/bin/bash
# ncu --set full + source of the Grain ROW_MAJOR (TMEM-staged) keystream kernel
mkdir -p gpurun_out/prof_grm
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 \
    -o gpurun_out/prof_grm/grain_rm_tmem python tools/prof_driver.py --cipher grain --layout row_major \
    --bits 32768 --reps 2 > gpurun_out/prof_grm/log.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 \
    -o gpurun_out/prof_grm/mickey_rm_tmem python tools/prof_driver.py --cipher mickey2 --layout row_major \
    --bits 32768 --reps 2 >> gpurun_out/prof_grm/log.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 \
    -o gpurun_out/prof_grm/mickey_consume python tools/prof_driver.py --cipher mickey2 --layout checksum \
    --bits 65536 --reps 2 >> gpurun_out/prof_grm/log.txt 2>&1
