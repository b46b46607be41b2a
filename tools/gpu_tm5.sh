python -c "from paper_conf_icppw_monfaredhkzrg20_b200 import build as b; b.build()" || exit 1
mkdir -p gpurun_out/tm5
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/tm5/pytest.txt 2>&1; tail -2 gpurun_out/tm5/pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
for c in mickey2 grain; do BSRNG_DEBUG=1 timeout 300 python tools/prof_driver.py --cipher $c --layout row_major --bits 32768 --reps 1 2>&1 | grep occ; done
timeout 900 python tools/sweep.py --cipher grain --layouts row_major --bits 65536 --chunk 32768 --reps 3 --opts "" seg_clocks=8192 > gpurun_out/tm5/grain.jsonl 2>&1
timeout 900 python tools/sweep.py --cipher mickey2 --layouts row_major --bits 65536 --chunk 32768 --reps 2 --opts "" rm_ws=1 > gpurun_out/tm5/mickey.jsonl 2>&1
cat gpurun_out/tm5/*.jsonl
timeout 900 python bench.py --no-cpu-baseline --no-context > gpurun_out/tm5/n1.json 2>&1
python -c "import json; d=json.loads(open('gpurun_out/tm5/n1.json').read().strip().splitlines()[-1]); m=d['modes']; print('mickey', d['value'], d['roofline']['frac'], m['materialise']['value'], m['materialise']['roofline']['frac'], d['e2e']['value'])"
for c in grain aes128ctr lfsr128; do timeout 900 python bench.py --cipher $c --no-cpu-baseline --no-context --no-e2e > gpurun_out/tm5/c2_$c.json 2>&1
python -c "import json; d=json.loads(open('gpurun_out/tm5/c2_$c.json').read().strip().splitlines()[-1]); m=d['modes']; print('$c', d['value'], d['roofline']['frac'], m['materialise']['value'], m['materialise']['roofline']['frac'])"; done
for c in mickey2 grain aes128ctr; do
  timeout 600 python bench.py --cipher $c --workload rekey --no-context --no-cpu-baseline --no-e2e --no-other-mode > gpurun_out/tm5/rekey_$c.json 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/tm5/rekey_$c.json').read().strip().splitlines()[-1]); print('$c', d['value'], d['unit'], d['ms_per_step'], d['modes']['consume'].get('rekey_ms_per_step'))"
done
