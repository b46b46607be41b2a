python -c "from paper_conf_icppw_monfaredhkzrg20_b200 import build as b; b.build()" || exit 1
mkdir -p gpurun_out/tm3
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/tm3/pytest.txt 2>&1; tail -2 gpurun_out/tm3/pytest.txt
BSRNG_DEBUG=1 timeout 300 python tools/prof_driver.py --cipher grain --layout row_major --bits 32768 --reps 1 2>&1 | tail -2
timeout 900 python tools/sweep.py --cipher grain --layouts row_major --bits 65536 --chunk 32768 --reps 3 --opts \
  "" rm_tmem=0 seg_clocks=4096 seg_clocks=2048 seg_clocks=8192 > gpurun_out/tm3/grain.jsonl 2>&1
cat gpurun_out/tm3/grain.jsonl
timeout 900 python bench.py --cipher grain --no-context --no-cpu-baseline > gpurun_out/tm3/c2_grain.json 2>&1
python -c "import json; d=json.loads(open('gpurun_out/tm3/c2_grain.json').read().strip().splitlines()[-1]); m=d['modes']; print('grain', d['value'], m['materialise']['value'], m['materialise']['roofline']['frac'])"
