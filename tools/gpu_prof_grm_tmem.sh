#!/bin/bash
# ncu --set full + source of the Grain / MICKEY ROW_MAJOR (TMEM-staged) and MICKEY consume
# keystream kernels; exports raw + SASS-source CSVs and keeps only the small reports.
D=gpurun_out/prof_grm; mkdir -p $D
run() {  # name, driver args
  local name=$1; shift
  ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 \
      -o /tmp/$name python tools/prof_driver.py "$@" >> $D/log.txt 2>&1
  ncu -i /tmp/$name.ncu-rep --page raw --csv > $D/${name}_raw.csv 2>>$D/log.txt
  ncu -i /tmp/$name.ncu-rep --page source --csv --print-source sass > $D/${name}_sass.csv 2>>$D/log.txt
  ncu -i /tmp/$name.ncu-rep --page details --csv > $D/${name}_details.csv 2>>$D/log.txt
}
run grain_rm_tmem --cipher grain --layout row_major --bits 32768 --reps 2
run mickey_rm_tmem --cipher mickey2 --layout row_major --bits 32768 --reps 2
run mickey_consume --cipher mickey2 --layout checksum --bits 65536 --reps 2
ls -la $D >> $D/log.txt
