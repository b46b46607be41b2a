timeout 600 python tools/sweep.py --layouts checksum,sliced,row_major --bits 65536 --opts unroll=1 unroll=2 unroll=4 unroll=8 unroll=4,sched=0 unroll=2,ctas_per_sm=1
