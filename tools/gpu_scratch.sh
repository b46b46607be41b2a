# scratch A/B runs (overwritten freely; results that matter go to profiles/)
D=gpurun_out/ab_flush; mkdir -p $D
timeout 900 python -m pytest -q -x -m gpu tests/test_gpu_rowmajor_items.py tests/test_gpu_random.py tests/test_gpu_grain.py tests/test_gpu_lfsr.py tests/test_gpu_api.py tests/test_gpu_mickey2.py > $D/tests.txt 2>&1; tail -3 $D/tests.txt
B="python bench.py --no-cpu-baseline --no-e2e --no-context --no-other-mode --mode materialise"
for r in 1 2; do
  for v in prev cur; do
    if [ $v = cur ]; then unset BSRNG_LIB; else export BSRNG_LIB=$PWD/build/lib_$v.so; fi
    echo "== $v $r grain_c4";  timeout 300 $B --workload c4 --cipher grain --steps 400 --warmup 20
    echo "== $v $r mickey_c4"; timeout 300 $B --workload c4 --cipher mickey2 --steps 100 --warmup 5
    echo "== $v $r lfsr_c2";   timeout 300 $B --cipher lfsr128 --steps 40
  done
done > $D/ab.txt 2>&1
grep -o '^== .*\|"value": [0-9.]*' $D/ab.txt | uniq
