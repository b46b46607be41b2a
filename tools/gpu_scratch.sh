D=gpurun_out/pf1; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_api.py tests/test_gpu_rowmajor_items.py tests/test_gpu_lfsr.py tests/test_gpu_grain.py -q -x -p no:cacheprovider > $D/pytest.txt 2>&1
run() { name=$1; shift; timeout 300 python bench.py --no-context --no-cpu-baseline --no-e2e --warmup 10 --mode materialise --no-other-mode "$@" > $D/$name.json 2>$D/$name.err; }
run grain_c4 --cipher grain --workload c4 --steps 1000
run lfsr_c4 --cipher lfsr128 --workload c4 --steps 1000
run lfsr_c2 --cipher lfsr128 --steps 20
