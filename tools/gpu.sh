#!/bin/bash
# tools/gpu.sh -- the one driver for GPU-box work (run through gpurun from the
# repo root, e.g.  gpurun --timeout 1800 -- 'bash tools/gpu.sh record r2').
# Everything lands under gpurun_out/<tag>/ (merged back by gpurun); committed
# evidence is copied from there into profiles/ (see profiles/README.md).
#
#   tests   TAG [pytest args]   pytest -m gpu (+ smoke) -> TAG/pytest_gpu.txt, smoke.txt
#   bench   TAG NAME [args]     one bench.py line      -> TAG/NAME.json (+ .err)
#   record  TAG                 the round record: tests, smoke, default bench, reference arm,
#                               C2 line per cipher, C4 (paper shape) and rekey lines with >= 1 s
#                               timed regions (clock samples), C3 at N = 1
#   launches TAG [bench args]   ncu launch list (gpu__time_duration) of a bench command
#   capture TAG NAME REGEX [prof_driver args]
#                               ncu --set full (+ SASS source) of one kernel launch, exported to
#                               CSV on the box (reports are too big to copy back)
#   captures TAG                the standard capture set (dominant kernel per cipher x layout)
#   sanitize TAG                compute-sanitizer memcheck / racecheck / synccheck over every path
#   micro   TAG                 ALU issue ceiling, cuRAND same-bytes, HBM write peaks
#   sweep   TAG                 the configs[4] sweep (tools/sweep_c5.py)
set -u
cmd=$1; tag=$2; shift 2
D=gpurun_out/$tag; mkdir -p $D
gpuinfo() { nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > $D/gpu.txt 2>&1; }
bench() {  # NAME args...
  local name=$1; shift
  timeout ${BENCH_TIMEOUT:-1200} python bench.py "$@" > $D/$name.json 2> $D/$name.err
  echo "bench $name exit $?" >> $D/status.txt
}
capture() {  # NAME REGEX prof_driver-args...
  local name=$1 rx=$2; shift 2
  ncu --set full --clock-control none --import-source on -k regex:$rx -s ${SKIP:-1} -c 1 \
      -o /tmp/cap_$name python tools/prof_driver.py "$@" > $D/ncu_$name.log 2>&1
  ncu -i /tmp/cap_$name.ncu-rep --page raw --csv > $D/${name}_raw.csv 2>/dev/null
  ncu -i /tmp/cap_$name.ncu-rep --page details --csv > $D/${name}_details.csv 2>/dev/null
  [ -n "${SASS:-}" ] && ncu -i /tmp/cap_$name.ncu-rep --page source --csv --print-source sass > $D/${name}_sass.csv 2>/dev/null
  rm -f /tmp/cap_$name.ncu-rep
}
case $cmd in
tests)
  gpuinfo
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider --durations=20 "$@" > $D/pytest_gpu.txt 2>&1
  echo "pytest exit $?" >> $D/pytest_gpu.txt
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.txt 2>&1
  echo "smoke exit $?" >> $D/smoke.txt ;;
bench)
  gpuinfo; bench "$@" ;;
record)
  gpuinfo
  timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider --durations=20 > $D/pytest_gpu.txt 2>&1
  echo "pytest exit $?" >> $D/pytest_gpu.txt
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.txt 2>&1
  bench n1_default
  bench n1_reference --impl reference
  for c in grain aes128ctr; do bench c2_$c --cipher $c --steps 10; done
  bench c2_lfsr128 --cipher lfsr128 --steps 60
  # paper shape and rekey steps are a few ms: 400+ steps give >= 1 s timed regions
  for c in mickey2 grain aes128ctr; do
    bench c4_$c --cipher $c --workload c4 --no-cpu-baseline --no-e2e --steps 2000 --warmup 20
    bench rekey_$c --cipher $c --workload rekey --no-cpu-baseline --no-e2e --no-other-mode --steps 1000 --warmup 20
  done
  bench c3_n1 --workload c3 --steps 3 --warmup 3 --no-other-mode --no-context ;;
launches)
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $D/launches.csv \
      python bench.py --no-cpu-baseline --no-context "$@" > $D/bench_under_ncu.json 2> $D/bench_under_ncu.err ;;
capture)
  capture "$@" ;;
captures)
  capture ks_consume keystream_kernel --layout checksum --bits 65536 --reps 2
  capture ks_rowmajor keystream_kernel --layout row_major --bits 32768 --reps 2
  capture ks_sliced keystream_kernel --layout sliced --bits 4096 --reps 2
  capture grain_consume keystream_kernel --cipher grain --layout checksum --bits 65536 --reps 2
  capture grain_rowmajor keystream_kernel --cipher grain --layout row_major --bits 32768 --reps 2
  capture aes_consume aes_ctr --cipher aes128ctr --layout checksum --bits 16384 --reps 2
  capture aes_rowmajor rowmajor_lanes --cipher aes128ctr --layout row_major --bits 16384 --reps 2
  capture lfsr_consume keystream_kernel --cipher lfsr128 --layout checksum --bits 65536 --reps 2
  capture lfsr_rowmajor keystream_rm_ws --cipher lfsr128 --layout row_major --bits 32768 --reps 2
  capture lfsr_sliced keystream_kernel --cipher lfsr128 --layout sliced --bits 65536 --reps 2
  SKIP=0 capture preclock m2_init --layout checksum --bits 32 --reps 1
  SKIP=0 capture grain_init grain_init --cipher grain --layout checksum --bits 32 --reps 1 ;;
sanitize)
  for tool in memcheck racecheck; do
    timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_driver.py > $D/$tool.txt 2>&1
    echo "exit $?" >> $D/$tool.txt
  done
  for v in WS_ONLY NO_TMEM; do
    env SANITIZE_$v=1 timeout 1500 compute-sanitizer --tool synccheck --print-limit 20 \
      python tools/sanitize_driver.py > $D/synccheck_$v.txt 2>&1
    echo "exit $?" >> $D/synccheck_$v.txt
  done ;;
micro)
  (cd tools/microbench && ./alu_peak 200000 && ./curand_bench 4294967296 && ./write_peak) > $D/micro.log 2>&1 ;;
sweep)
  timeout 2400 python tools/sweep_c5.py > $D/sweep.jsonl 2> $D/sweep.err
  (cd tools/microbench && timeout 300 ./curand_bench 2147483648 && timeout 300 ./curand_bench 17179869184) > $D/curand.log 2>&1 ;;
*)
  echo "unknown command $cmd"; exit 2 ;;
esac
