D=gpurun_out/lp; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_api.py tests/test_gpu_rowmajor_items.py tests/test_gpu_lfsr.py tests/test_gpu_random.py tests/test_gpu_fullsize.py -x -q -m gpu > $D/pytest.txt 2>&1
tail -3 $D/pytest.txt
run() { n=$1; shift; timeout 300 python bench.py --no-context --no-cpu-baseline --no-e2e --no-other-mode "$@" > $D/$n.json 2>$D/$n.err; }
run lfsr_c2 --cipher lfsr128 --mode materialise --steps 20 --warmup 5
run lfsr_c4 --cipher lfsr128 --mode materialise --workload c4 --steps 2000 --warmup 20
run grain_c4 --cipher grain --mode materialise --workload c4 --steps 2000 --warmup 20
for f in $D/*.json; do echo $f; python -c "import json,sys; d=json.load(open('$f')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['clocks']['sm_mhz'])"; done
