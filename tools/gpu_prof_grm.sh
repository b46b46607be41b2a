mkdir -p gpurun_out
python - <<'PY'
import re
src=open('tools/prof_driver.py').read()
PY
ncu --set full --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 -o gpurun_out/grain_rm2 python tools/prof_driver.py --cipher grain --layout row_major --bits 32768 --reps 2 --rm-ws 0 > gpurun_out/grm.log 2>&1
tail -2 gpurun_out/grm.log
