python -c "from paper_conf_icppw_monfaredhkzrg20_b200 import build as b; b.build()" || exit 1
mkdir -p gpurun_out/init2
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/init2/pytest.txt 2>&1; tail -3 gpurun_out/init2/pytest.txt
for c in mickey2 grain; do for f in 1 0; do
  timeout 600 python bench.py --cipher $c --workload rekey --no-context --no-cpu-baseline --no-e2e --no-other-mode --opt init_fused=$f > gpurun_out/init2/rekey_${c}_f$f.json 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/init2/rekey_${c}_f$f.json').read().strip().splitlines()[-1]); print('$c fused=$f', d['value'], d['unit'], d['ms_per_step'], d['modes']['consume'].get('rekey_ms_per_step'), d['modes']['consume'].get('preclock_roofline',{}).get('frac'))"
done; done
BSRNG_DEBUG=1 timeout 300 python tools/prof_driver.py --cipher grain --layout row_major --bits 16384 --reps 1 --opt rm_tmem=1 2>&1 | tail -2
BSRNG_DEBUG=1 timeout 300 python tools/prof_driver.py --cipher grain --layout row_major --bits 16384 --reps 1 --opt rm_tmem=1 --opt ctas_per_sm=2 2>&1 | tail -2
BSRNG_DEBUG=1 timeout 300 python tools/prof_driver.py --cipher grain --layout row_major --bits 16384 --reps 1 2>&1 | tail -2
