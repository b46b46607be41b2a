#!/bin/bash
# usage: gpu_prof_one.sh NAME <prof_driver args...>   (ncu --set full + SASS source CSVs)
D=gpurun_out/prof1; mkdir -p $D
name=$1; shift
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 \
    -o /tmp/$name python tools/prof_driver.py "$@" >> $D/log.txt 2>&1
ncu -i /tmp/$name.ncu-rep --page raw --csv > $D/${name}_raw.csv 2>>$D/log.txt
ncu -i /tmp/$name.ncu-rep --page source --csv --print-source sass > $D/${name}_sass.csv 2>>$D/log.txt
