timeout 600 python -m pytest tests/test_gpu_mickey2.py -q -x 2>&1 | tail -3
timeout 600 python tools/sweep.py --layouts row_major,checksum --bits 65536 --opts unroll=4 unroll=2
timeout 600 python tools/sweep.py --layouts row_major --bits 65536 --chunk 4096 --opts unroll=4
