D=gpurun_out/mx1; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_grain.py tests/test_gpu_rowmajor_items.py tests/test_gpu_api.py -q -x -p no:cacheprovider > $D/pytest.txt 2>&1
run() { name=$1; shift; timeout 300 python bench.py --cipher grain --no-context --no-cpu-baseline --no-e2e --steps 5 --warmup 3 --mode materialise --no-other-mode "$@" > $D/$name.json 2>$D/$name.err; }
run c2_mixed
run c2_base --opt rm_mixed=0
run c2_mixed_256k --bits 262144
