# Round profile: launch list of the bench command + full captures of the
# dominant kernel (consume at the bench config, row-major at the bench chunk).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu.txt
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu.json 2> gpurun_out/bench_under_ncu.err
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -c 1 -o gpurun_out/ks_consume_full \
    python bench.py --steps 1 --warmup 0 --no-other-mode --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_consume.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 -o gpurun_out/ks_rowmajor_full \
    python tools/prof_driver.py --layout row_major --bits 32768 --reps 2 > gpurun_out/ncu_full_rowmajor.log 2>&1
ls -la gpurun_out
