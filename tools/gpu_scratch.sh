D=gpurun_out/wsv2; mkdir -p $D
run() { n=$1; shift; timeout 300 python bench.py --no-context --no-cpu-baseline --no-e2e --no-other-mode "$@" > $D/$n.json 2>$D/$n.err; }
run m2_c4_def --cipher mickey2 --mode materialise --workload c4 --steps 2000 --warmup 20
run m2_c4_ws --cipher mickey2 --mode materialise --workload c4 --steps 2000 --warmup 20 --opt rm_ws=1
run m2_c2_def --cipher mickey2 --mode materialise --steps 3 --warmup 3
run m2_c2_ws --cipher mickey2 --mode materialise --steps 3 --warmup 3 --opt rm_ws=1
run g_c2_def --cipher grain --mode materialise --steps 10 --warmup 3
run g_c2_ws --cipher grain --mode materialise --steps 10 --warmup 3 --opt rm_ws=1
for f in $D/*.json; do echo $f; python -c "import json,sys; d=json.load(open('$f')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['clocks']['sm_mhz'])"; done
