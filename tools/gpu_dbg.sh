BSRNG_DEBUG=1 timeout 600 python tools/sweep.py --layouts checksum --bits 16384 --reps 1 --opts unroll=4,seg_clocks=2048 unroll=4,seg_clocks=8192 unroll=4,ctas_per_sm=1,seg_clocks=2048
