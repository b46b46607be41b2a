mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 -o gpurun_out/prof_consume python tools/prof_driver.py --layout checksum --bits 4096 --reps 2 > gpurun_out/ncu_consume.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 -o gpurun_out/prof_rowmajor python tools/prof_driver.py --layout row_major --bits 4096 --reps 2 > gpurun_out/ncu_rowmajor.log 2>&1
tail -3 gpurun_out/ncu_consume.log gpurun_out/ncu_rowmajor.log
ls -la gpurun_out
