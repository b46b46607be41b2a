D=gpurun_out/apol; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_aes.py tests/test_gpu_api.py -x -q -m gpu > $D/pytest.txt 2>&1
tail -3 $D/pytest.txt
run() { n=$1; shift; timeout 300 python bench.py --cipher aes128ctr --no-context --no-cpu-baseline --no-e2e --no-other-mode "$@" > $D/$n.json 2>$D/$n.err; }
run c2 --steps 10 --warmup 3
run c2_mat --steps 10 --warmup 3 --mode materialise
run rekey --workload rekey --steps 1000 --warmup 20
run c4 --workload c4 --steps 2000 --warmup 20
for f in $D/*.json; do echo $f; python -c "import json,sys; d=json.load(open('$f')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['clocks']['sm_mhz'])"; done
