for c in grain mickey2; do for b in 4416 12992; do
timeout 600 python bench.py --cipher $c --workload c4 --bits $b --no-cpu-baseline --no-context --no-e2e | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'], 'consume', round(d['value'],3), 'frac', round(d['roofline']['frac'],4), 'materialise', round(d['modes']['materialise']['value'],3), round(d['modes']['materialise']['roofline']['frac'],4))"
done; done
