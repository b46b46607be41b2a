python -c "from paper_conf_icppw_monfaredhkzrg20_b200 import build as b; b.build()" || exit 1
mkdir -p gpurun_out/tm2
timeout 600 python -m pytest tests/test_gpu_api.py -q -x > gpurun_out/tm2/pytest.txt 2>&1; tail -2 gpurun_out/tm2/pytest.txt
BSRNG_DEBUG=1 timeout 300 python tools/prof_driver.py --cipher grain --layout row_major --bits 16384 --reps 1 --opt rm_tmem=1 --opt ctas_per_sm=2 --opt seg_clocks=16384 2>&1 | tail -2
timeout 900 python tools/sweep.py --cipher grain --layouts row_major --bits 65536 --chunk 16384 --reps 3 --opts \
  "" rm_tmem=1,ctas_per_sm=2 rm_tmem=1,ctas_per_sm=2,seg_clocks=16384 rm_tmem=1,ctas_per_sm=2,seg_clocks=4096 > gpurun_out/tm2/grain.jsonl 2>&1
timeout 900 python tools/sweep.py --cipher mickey2 --layouts row_major --bits 65536 --chunk 32768 --reps 2 --opts \
  rm_ws=0,rm_tmem=1,ctas_per_sm=2,seg_clocks=32768 rm_ws=0,rm_slots=4 > gpurun_out/tm2/mickey.jsonl 2>&1
cat gpurun_out/tm2/*.jsonl
