for c in mickey2 grain aes128ctr; do
timeout 600 python bench.py --cipher $c --workload rekey --no-cpu-baseline --no-context --no-e2e --no-other-mode | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); m=d['modes']['consume']
print('$c', 'Tb/s', round(d['value'],3), 'step ms', round(d['ms_per_step'],3), 'rekey ms', round(m['rekey_ms_per_step'],3), 'keys/s %.3g' % m['keys_per_s'], 'preclock frac', m['preclock_roofline'] and round(m['preclock_roofline']['frac'],3), 'ks frac', round(d['roofline']['frac'],3))"
done
