D=gpurun_out/gip2; mkdir -p $D
run() { n=$1; shift; timeout 300 python bench.py --no-context --no-cpu-baseline --no-e2e --no-other-mode "$@" > $D/$n.json 2>$D/$n.err; }
for v in default nopf oneshot oneshot_nopf; do
  if [ $v = default ]; then unset BSRNG_LIB; else export BSRNG_LIB=$PWD/build/libgi_$v.so; fi
  run $v --cipher grain --workload rekey --steps 1000 --warmup 20
done
unset BSRNG_LIB
git -C . log -1 --format=%h 2>/dev/null
for f in $D/*.json; do echo $f; python -c "import json,sys; d=json.load(open('$f')); m=list(d['modes'].values())[0]; print(d['value'], d['ms_per_step'], m['kernel_ms_per_step'], m['rekey_ms_per_step'], m['preclock_roofline']['frac'])"; done
