D=gpurun_out/ws2b; mkdir -p $D
timeout 600 python -m pytest -q -x -m gpu tests/test_gpu_api.py tests/test_gpu_rowmajor_items.py tests/test_gpu_random.py -k "lfsr" > $D/tests.txt 2>&1; tail -3 $D/tests.txt
B="python bench.py --no-cpu-baseline --no-e2e --no-context --no-other-mode --mode materialise"
for r in 1 2; do
for v in cur ws2nz16; do
if [ $v = cur ]; then unset BSRNG_LIB; else export BSRNG_LIB=$PWD/build/lib_$v.so; fi
echo "== $v ws2 lfsr_c2";   timeout 300 $B --cipher lfsr128 --steps 40 --opt rm_ws=2
done; done > $D/ab.txt 2>&1
grep -o '^== .*\|"value": [0-9.]*' $D/ab.txt | uniq
