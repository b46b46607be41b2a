D=gpurun_out/ab2; mkdir -p $D
for r in 1 2; do
  for v in prev cur; do
    if [ $v = cur ]; then unset BSRNG_LIB; else export BSRNG_LIB=$PWD/build/lib_prev.so; fi
    echo "== $v $r"; timeout 300 python tools/time_sliced.py
  done
done > $D/sliced.txt 2>&1
cat $D/sliced.txt
