D=gpurun_out/ab_nofl; mkdir -p $D
timeout 900 python -m pytest -q -x -m gpu tests/test_gpu_rowmajor_items.py tests/test_gpu_random.py tests/test_gpu_grain.py tests/test_gpu_lfsr.py tests/test_gpu_api.py tests/test_gpu_mickey2.py tests/test_gpu_contract.py > $D/tests.txt 2>&1; tail -3 $D/tests.txt
B="python bench.py --no-cpu-baseline --no-e2e --no-context --no-other-mode --mode materialise"
for v in cur noflush; do
    export BSRNG_LIB=$PWD/build/lib_$v.so
    echo "== $v grain_c4";  timeout 300 $B --workload c4 --cipher grain --steps 400 --warmup 20
    echo "== $v lfsr_c2";   timeout 300 $B --cipher lfsr128 --steps 40
    echo "== $v lfsr_c2_wide";   timeout 300 $B --cipher lfsr128 --steps 40 --opt rm_ws=0 --opt rm_wide=1
done > $D/ab.txt 2>&1
grep -o '^== .*\|"value": [0-9.]*' $D/ab.txt | uniq
