D=gpurun_out/ab5; mkdir -p $D
for v in base fma16; do
  if [ $v = fma16 ]; then export BSRNG_LIB=$PWD/build/libbsrng_fma16.so; else unset BSRNG_LIB; fi
  run() { name=$1; shift; timeout 300 python bench.py --no-context --no-cpu-baseline --no-e2e --warmup 3 --mode materialise --no-other-mode "$@" > $D/${v}_$name.json 2>$D/${v}_$name.err; }
  run grain_c2 --cipher grain --steps 8
  run mickey_c2 --cipher mickey2 --steps 3 --bits 131072
  run grain_c4 --cipher grain --workload c4 --steps 1000
  run mickey_c4 --cipher mickey2 --workload c4 --steps 300
done
