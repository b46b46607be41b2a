mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:aes_ctr -s 1 -c 1 -o gpurun_out/aes_cs python tools/prof_driver.py --cipher aes128ctr --layout checksum --bits 16384 --reps 2 > /dev/null 2>&1
ls gpurun_out
