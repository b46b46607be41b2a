#!/bin/bash
D=gpurun_out/sanitize; mkdir -p $D
timeout 300 compute-sanitizer --tool synccheck ./tools/microbench/tmem_layout > $D/synccheck_tmem_layout.txt 2>&1; echo "exit $?" >> $D/synccheck_tmem_layout.txt
SANITIZE_NO_TMEM=1 timeout 1500 compute-sanitizer --tool synccheck --print-limit 20 python tools/sanitize_driver.py > $D/synccheck_no_tmem.txt 2>&1; echo "exit $?" >> $D/synccheck_no_tmem.txt
