#!/bin/bash
# configs[2] at N = 1 (1 TiB of MICKEY keystream in one step; strong scaling
# baseline for the driver's N = 2/4/8 runs)
D=gpurun_out/c3; mkdir -p $D
timeout 1200 python bench.py --workload c3 --steps 3 --warmup 3 --no-other-mode --no-context > $D/c3_n1.json 2> $D/c3_n1.err
