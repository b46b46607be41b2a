mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:rm_ws -s 1 -c 1 -o gpurun_out/grain_rmws python tools/prof_driver.py --cipher grain --layout row_major --bits 32768 --reps 2 > /dev/null 2>&1
ls gpurun_out
