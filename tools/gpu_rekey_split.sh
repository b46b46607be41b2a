#!/bin/bash
D=gpurun_out/rekey_split; mkdir -p $D
python tools/rekey_split.py > $D/events.txt 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $D/ncu.csv python tools/rekey_split.py > $D/ncu_stdout.txt 2>&1
