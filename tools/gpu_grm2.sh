# TMEM staging for ROW_MAJOR: parity then speed.
python -c "from paper_conf_icppw_monfaredhkzrg20_b200 import build as b; b.build()" || exit 1
mkdir -p gpurun_out/grm2
timeout 600 python -m pytest tests/test_gpu_api.py -q -x -k "tmem or options" > gpurun_out/grm2/pytest.txt 2>&1; tail -5 gpurun_out/grm2/pytest.txt
timeout 900 python tools/sweep.py --cipher grain --layouts row_major --bits 65536 --chunk 16384 --reps 3 --opts \
  rm_slots=8 rm_tmem=1 rm_tmem=1,ctas_per_sm=1 rm_tmem=1,ctas_per_sm=2 rm_tmem=1,rm_zreg=0 rm_tmem=1,rm_zreg=0,ctas_per_sm=2 \
  rm_tmem=1,unroll=16,ctas_per_sm=2 > gpurun_out/grm2/grain.jsonl 2>&1
timeout 900 python tools/sweep.py --cipher lfsr128 --layouts row_major --bits 65536 --chunk 16384 --reps 3 --opts \
  rm_slots=8 rm_tmem=1 rm_tmem=1,ctas_per_sm=2 > gpurun_out/grm2/lfsr.jsonl 2>&1
timeout 900 python tools/sweep.py --cipher mickey2 --layouts row_major --bits 65536 --chunk 32768 --reps 2 --opts \
  rm_ws=0,rm_tmem=1 rm_ws=0,rm_tmem=1,ctas_per_sm=2 > gpurun_out/grm2/mickey.jsonl 2>&1
cat gpurun_out/grm2/*.jsonl
