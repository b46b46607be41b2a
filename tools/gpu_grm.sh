# Grain / MICKEY ROW_MAJOR staging variants (rm_slots, rm_zreg, occupancy).
python -c "from paper_conf_icppw_monfaredhkzrg20_b200 import build as b; b.build()" || exit 1
mkdir -p gpurun_out/grm
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/grm/pytest.txt 2>&1; tail -3 gpurun_out/grm/pytest.txt
timeout 900 python tools/sweep.py --cipher grain --layouts row_major --bits 65536 --chunk 16384 --reps 3 --opts \
  rm_slots=8 rm_slots=8,ctas_per_sm=1 rm_slots=4 rm_slots=4,ctas_per_sm=1 rm_zreg=0 rm_zreg=0,rm_slots=8 \
  rm_zreg=0,rm_slots=8,ctas_per_sm=1 unroll=16,rm_slots=4 unroll=16,rm_slots=4,ctas_per_sm=2 > gpurun_out/grm/grain.jsonl 2>&1
timeout 900 python tools/sweep.py --cipher grain --layouts checksum --bits 65536 --reps 3 --opts "" > gpurun_out/grm/grain_cs.jsonl 2>&1
timeout 900 python tools/sweep.py --cipher lfsr128 --layouts row_major --bits 65536 --chunk 16384 --reps 3 --opts \
  rm_slots=8 rm_slots=4 rm_zreg=0 > gpurun_out/grm/lfsr.jsonl 2>&1
timeout 900 python tools/sweep.py --cipher mickey2 --layouts row_major --bits 65536 --chunk 32768 --reps 2 --opts \
  "" rm_ws=0 rm_ws=0,rm_slots=4 rm_ws=0,rm_slots=4,ctas_per_sm=2 > gpurun_out/grm/mickey.jsonl 2>&1
cat gpurun_out/grm/*.jsonl
for c in mickey2 grain aes128ctr; do
  timeout 600 python bench.py --cipher $c --workload rekey --no-context --no-cpu-baseline --no-e2e --no-other-mode > gpurun_out/grm/rekey_$c.json 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/grm/rekey_$c.json').read().strip().splitlines()[-1]); print('$c', d['value'], d['unit'], d['ms_per_step'], d['modes']['consume'].get('rekey_ms_per_step'))"
done
