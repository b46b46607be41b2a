timeout 600 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
timeout 300 python tools/sweep.py --layouts row_major --bits 65536 --opts rm_ws=1 rm_ws=0
timeout 300 python tools/sweep.py --cipher grain --layouts row_major,checksum --bits 65536 --opts rm_ws=1 rm_ws=0
timeout 300 python tools/sweep.py --cipher grain --n 524288 --layouts row_major --bits 4416 --chunk 4416 --reps 3 --opts rm_ws=1 rm_ws=0
