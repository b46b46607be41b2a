#!/usr/bin/env python3
"""Warp-stall samples from an ncu --page source --csv --print-source sass export:
totals per stall reason and per opcode.  Usage: ncu_stalls.py <sass.csv> [lo-hi ...]"""
import csv, sys, re
from collections import Counter, defaultdict
f = sys.argv[1]
rows = list(csv.reader(open(f)))
hdr = rows[1]; data = rows[2:]
ix = {h: i for i, h in enumerate(hdr)}
stall_cols = [h for h in hdr if h.startswith('stall_') and 'Not Issued' not in h]
tot = Counter(); byop = defaultdict(Counter); nsamp = 0
ranges = [tuple(int(x, 16) for x in r.split('-')) for r in sys.argv[2:]]
for r in data:
    try: addr = int(r[ix['Address']], 16)
    except: continue
    if ranges and not any(lo <= addr <= hi for lo, hi in ranges): continue
    op = r[ix['Source']].strip()
    op = re.sub(r'^@!?U?P\w+\s+', '', op).split()[0] if op else '?'
    for h in stall_cols:
        v = float(r[ix[h]] or 0)
        tot[h] += v; byop[op][h] += v
    nsamp += float(r[ix['# Samples']] or 0)
print('samples', nsamp)
S = sum(tot.values())
for h, v in tot.most_common(12): print(f'{h:28s} {v:10.0f} {100*v/S:5.1f}%')
print('--- by opcode (top)')
opt = sorted(byop.items(), key=lambda kv: -sum(kv[1].values()))[:14]
for op, c in opt:
    s = sum(c.values()); top = ', '.join(f'{k[6:]}={100*v/s:.0f}%' for k, v in c.most_common(3))
    print(f'{op:22s} {100*s/S:5.1f}%  {top}')
