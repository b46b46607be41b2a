mkdir -p gpurun_out
timeout 600 python tools/sweep.py --cipher grain --n 524288 --layouts row_major --bits 4416 --chunk 4416 --reps 3 --opts unroll=32
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 -o gpurun_out/grain_rm python tools/prof_driver.py --cipher grain --layout row_major --bits 32768 --reps 2 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 -o gpurun_out/grain_cs python tools/prof_driver.py --cipher grain --layout checksum --bits 65536 --reps 2 > /dev/null 2>&1
ls gpurun_out
