# Round record (see profiles/README.md): tests, smoke, bench lines for every
# workload, the ncu launch list of the default bench command and full ncu
# captures of the dominant kernel per cipher/layout.
set -x
mkdir -p gpurun_out/prof gpurun_out/bench
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > gpurun_out/prof/gpu.txt
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/bench/pytest_gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/bench/smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/bench/n1_default.json 2> gpurun_out/bench/n1_default.err
timeout 600 python bench.py --impl reference > gpurun_out/bench/n1_reference.json 2>&1
for c in grain aes128ctr lfsr128; do
  timeout 600 python bench.py --cipher $c --no-context > gpurun_out/bench/c2_$c.json 2>&1
done
for c in mickey2 grain aes128ctr; do
  timeout 600 python bench.py --cipher $c --workload c4 --no-context --no-cpu-baseline --no-e2e > gpurun_out/bench/c4_$c.json 2>&1
  timeout 600 python bench.py --cipher $c --workload rekey --no-context --no-cpu-baseline --no-e2e --no-other-mode > gpurun_out/bench/rekey_$c.json 2>&1
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/prof/launches.csv \
    python bench.py --no-cpu-baseline --no-context > gpurun_out/prof/bench_under_ncu.json 2> gpurun_out/prof/bench_under_ncu.err
# full captures are exported to CSV on the box (the .ncu-rep files are ~18 MB
# each, over gpurun's 64 MiB copy-back limit) and the reports deleted
cap() {
  name=$1; shift
  ncu --set full --clock-control none --import-source on -k regex:$1 -s ${SKIP:-1} -c 1 -o /tmp/prof_$name "${@:2}" > gpurun_out/prof/ncu_$name.log 2>&1
  ncu -i /tmp/prof_$name.ncu-rep --page raw --csv > gpurun_out/prof/${name}_raw.csv 2>/dev/null
  ncu -i /tmp/prof_$name.ncu-rep --page details --csv > gpurun_out/prof/${name}_details.csv 2>/dev/null
  rm -f /tmp/prof_$name.ncu-rep
}
cap ks_consume keystream_kernel python tools/prof_driver.py --layout checksum --bits 65536 --reps 2
cap ks_rowmajor keystream_kernel python tools/prof_driver.py --layout row_major --bits 32768 --reps 2
cap ks_sliced keystream_kernel python tools/prof_driver.py --layout sliced --bits 4096 --reps 2
cap grain_consume keystream_kernel python tools/prof_driver.py --cipher grain --layout checksum --bits 65536 --reps 2
cap grain_rowmajor keystream_kernel python tools/prof_driver.py --cipher grain --layout row_major --bits 32768 --reps 2
cap aes_consume aes_ctr python tools/prof_driver.py --cipher aes128ctr --layout checksum --bits 16384 --reps 2
cap aes_rowmajor rowmajor_lanes python tools/prof_driver.py --cipher aes128ctr --layout row_major --bits 16384 --reps 2
cap lfsr_sliced keystream_kernel python tools/prof_driver.py --cipher lfsr128 --layout sliced --bits 65536 --reps 2
SKIP=0 cap preclock m2_init python tools/prof_driver.py --layout checksum --bits 32 --reps 1
SKIP=0 cap grain_init grain_init python tools/prof_driver.py --cipher grain --layout checksum --bits 32 --reps 1
ls -la gpurun_out/prof gpurun_out/bench
