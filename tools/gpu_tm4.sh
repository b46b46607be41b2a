python -c "from paper_conf_icppw_monfaredhkzrg20_b200 import build as b; b.build()" || exit 1
mkdir -p gpurun_out/tm4
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/tm4/pytest.txt 2>&1; tail -2 gpurun_out/tm4/pytest.txt
timeout 900 python tools/sweep.py --cipher grain --layouts row_major --bits 65536 --chunk 32768 --reps 3 --opts \
  "" rm_tmem=0 seg_clocks=8192 > gpurun_out/tm4/grain.jsonl 2>&1
timeout 900 python tools/sweep.py --cipher lfsr128 --layouts row_major --bits 65536 --chunk 32768 --reps 3 --opts \
  "" rm_tmem=1,ctas_per_sm=2 > gpurun_out/tm4/lfsr.jsonl 2>&1
timeout 900 python tools/sweep.py --cipher mickey2 --layouts row_major --bits 65536 --chunk 32768 --reps 2 --opts \
  "" rm_ws=0 rm_ws=0,rm_tmem=1 rm_ws=0,rm_tmem=1,seg_clocks=32768 rm_ws=0,rm_tmem=1,seg_clocks=8192 rm_ws=0,rm_slots=4 > gpurun_out/tm4/mickey.jsonl 2>&1
cat gpurun_out/tm4/*.jsonl
