mkdir -p gpurun_out/bench
for c in aes128ctr grain; do
timeout 900 python bench.py --cipher $c --no-cpu-baseline --no-context > gpurun_out/bench/c2_$c.json 2>&1
timeout 600 python bench.py --cipher $c --workload c4 --no-cpu-baseline --no-context --no-e2e > gpurun_out/bench/c4_$c.json 2>&1
done
timeout 600 python bench.py --workload c4 --no-cpu-baseline --no-context --no-e2e > gpurun_out/bench/c4_mickey2.json 2>&1
for f in gpurun_out/bench/*.json; do python -c "
import json,sys
d=json.loads(open('$f').read().strip().splitlines()[-1])
m=d['modes']
print('$f', round(d['value'],3), 'frac', round(d['roofline']['frac'],3), 'mat', round(m['materialise']['value'],3), round(m['materialise']['roofline']['frac'],3), 'e2e', d['e2e'] and round(d['e2e']['value'],3))
"; done
