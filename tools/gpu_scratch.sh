D=gpurun_out/sw7; mkdir -p $D
bash tools/gpu.sh tests sw7
run() { c=$1; name=$2; shift 2; timeout 300 python bench.py --cipher $c --mode materialise --no-other-mode --no-context --no-cpu-baseline --no-e2e --steps 5 --warmup 3 "$@" > $D/${c}_$name.json 2>$D/${c}_$name.err; }
run lfsr128 c2 --steps 40
run grain c2 --bits 262144
run grain c4 --workload c4 --steps 300 --warmup 10
run lfsr128 c4 --workload c4 --steps 300 --warmup 10
run mickey2 c2 --bits 65536
