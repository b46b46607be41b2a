D=gpurun_out/ab2; mkdir -p $D
timeout 600 python -m pytest tests/test_gpu_rowmajor_items.py tests/test_gpu_lfsr.py -q -x -p no:cacheprovider > $D/pytest.txt 2>&1
for v in s200 s50 s1000; do
  case $v in s200) unset BSRNG_LIB;; s50) export BSRNG_LIB=$PWD/build/libbsrng_ws50.so;; s1000) export BSRNG_LIB=$PWD/build/libbsrng_ws1000.so;; esac
  run() { name=$1; shift; timeout 300 python bench.py --no-context --no-cpu-baseline --no-e2e --steps 5 --warmup 3 --mode materialise --no-other-mode "$@" > $D/${v}_$name.json 2>$D/${v}_$name.err; }
  run grain_ws --cipher grain --opt rm_ws=1
  run grain_c4 --cipher grain --workload c4 --steps 1000 --warmup 10
  run lfsr --cipher lfsr128 --steps 20
  run mickey_ws --cipher mickey2 --opt rm_ws=1 --bits 65536
done
