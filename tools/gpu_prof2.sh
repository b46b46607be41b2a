mkdir -p gpurun_out
for v in "seg 2048" "noseg 16384"; do set -- $v
ncu --section WarpStateStats --section SchedulerStats --section ComputeWorkloadAnalysis --section SpeedOfLight --section SourceCounters --metrics smsp__pcsamp_warps_issue_stalled_no_instructions,smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio --clock-control none --import-source on -k regex:keystream_kernel -s 1 -c 1 -o gpurun_out/prof_$1 python tools/prof_driver.py --layout checksum --bits 16384 --reps 2 --seg-clocks $2 > gpurun_out/ncu_$1.log 2>&1
done
ls gpurun_out
