timeout 600 python tools/sweep.py --layouts checksum,sliced,row_major --bits 65536 --opts unroll=2 unroll=4 unroll=8 unroll=4,seg_clocks=65536 unroll=4,ctas_per_sm=2,sched=0
timeout 600 python tools/sweep.py --layouts checksum --n 524288 --bits 65536 --opts unroll=4 unroll=4,ctas_per_sm=2,sched=0
