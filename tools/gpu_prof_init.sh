#!/bin/bash
D=gpurun_out/prof1; mkdir -p $D
ncu --set full --clock-control none --import-source on -k regex:grain_init -s 0 -c 1 \
    -o /tmp/gi python tools/prof_driver.py --cipher grain --layout checksum --bits 32 --reps 1 > $D/gi_log.txt 2>&1
ncu -i /tmp/gi.ncu-rep --page raw --csv > $D/grain_init_raw.csv 2>>$D/gi_log.txt
ncu -i /tmp/gi.ncu-rep --page source --csv --print-source sass > $D/grain_init_sass.csv 2>>$D/gi_log.txt
