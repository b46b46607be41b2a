# Fused MICKEY init kernel: parity, rekey A/B; TMEM Grain row-major occupancy check.
python -c "from paper_conf_icppw_monfaredhkzrg20_b200 import build as b; b.build()" || exit 1
mkdir -p gpurun_out/init
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/init/pytest.txt 2>&1; tail -3 gpurun_out/init/pytest.txt
for f in 1 0; do
  timeout 600 python bench.py --workload rekey --no-context --no-cpu-baseline --no-e2e --no-other-mode --opt init_fused=$f > gpurun_out/init/rekey_m2_f$f.json 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/init/rekey_m2_f$f.json').read().strip().splitlines()[-1]); print('fused=$f', d['value'], d['unit'], d['ms_per_step'], d['modes']['consume'].get('rekey_ms_per_step'), d['modes']['consume'].get('preclock_roofline'))"
done
BSRNG_DEBUG=1 timeout 300 python tools/prof_driver.py --cipher grain --layout row_major --bits 16384 --reps 1 --opt rm_tmem=1 2>&1 | tail -3
cap() {
  name=$1; shift
  ncu --set full --clock-control none --import-source on -k regex:$1 -s $SKIP -c 1 -o /tmp/prof_$name "${@:2}" > gpurun_out/init/ncu_$name.log 2>&1
  ncu -i /tmp/prof_$name.ncu-rep --page raw --csv > gpurun_out/init/${name}_raw.csv 2>/dev/null
  ncu -i /tmp/prof_$name.ncu-rep --page details --csv > gpurun_out/init/${name}_details.csv 2>/dev/null
  rm -f /tmp/prof_$name.ncu-rep
}
SKIP=0 cap m2_init m2_init python tools/prof_driver.py --layout checksum --bits 32 --reps 1
SKIP=1 cap grain_tmem keystream_kernel python tools/prof_driver.py --cipher grain --layout row_major --bits 16384 --reps 2 --opt rm_tmem=1
ls gpurun_out/init
