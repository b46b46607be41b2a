# Round profile (see profiles/README.md): launch list of the default bench
# command + full ncu captures of the dominant kernel in both output modes.
mkdir -p gpurun_out/prof
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > gpurun_out/prof/gpu.txt
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/prof/launches.csv \
    python bench.py --no-cpu-baseline --no-context > gpurun_out/prof/bench_under_ncu.json 2> gpurun_out/prof/bench_under_ncu.err
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 -o gpurun_out/prof/ks_consume \
    python tools/prof_driver.py --layout checksum --bits 65536 --reps 2 > gpurun_out/prof/ncu_consume.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 -o gpurun_out/prof/ks_rowmajor \
    python tools/prof_driver.py --layout row_major --bits 32768 --reps 2 > gpurun_out/prof/ncu_rowmajor.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 -o gpurun_out/prof/ks_sliced \
    python tools/prof_driver.py --layout sliced --bits 4096 --reps 2 > gpurun_out/prof/ncu_sliced.log 2>&1
ncu --set full --clock-control none -k regex:preclock -c 1 -o gpurun_out/prof/preclock \
    python tools/prof_driver.py --layout checksum --bits 32 --reps 1 > gpurun_out/prof/ncu_preclock.log 2>&1
ls -la gpurun_out/prof
