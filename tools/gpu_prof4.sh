# Grain ROW_MAJOR: ncu full + SASS source stalls for the smem (default) and TMEM 2-CTA variants.
python -c "from paper_conf_icppw_monfaredhkzrg20_b200 import build as b; b.build()" || exit 1
mkdir -p gpurun_out/prof4
cap() {
  name=$1; shift
  ncu --set full --clock-control none --import-source on -k regex:$1 -s 1 -c 1 -o /tmp/prof_$name "${@:2}" > gpurun_out/prof4/ncu_$name.log 2>&1
  ncu -i /tmp/prof_$name.ncu-rep --page raw --csv > gpurun_out/prof4/${name}_raw.csv 2>/dev/null
  ncu -i /tmp/prof_$name.ncu-rep --page source --csv --print-source sass > gpurun_out/prof4/${name}_sass.csv 2>/dev/null
  rm -f /tmp/prof_$name.ncu-rep
}
cap grain_rm_smem keystream_kernel python tools/prof_driver.py --cipher grain --layout row_major --bits 16384 --reps 2
cap grain_rm_tmem2 keystream_kernel python tools/prof_driver.py --cipher grain --layout row_major --bits 16384 --reps 2 --opt rm_tmem=1 --opt ctas_per_sm=2 --opt seg_clocks=4096
cap grain_cs keystream_kernel python tools/prof_driver.py --cipher grain --layout checksum --bits 16384 --reps 2
timeout 900 python tools/sweep.py --cipher grain --layouts row_major --bits 65536 --chunk 16384 --reps 3 --opts \
  rm_tmem=1,rm_zreg=0,ctas_per_sm=2,seg_clocks=4096 rm_tmem=1,ctas_per_sm=2,seg_clocks=2048 rm_tmem=1,unroll=16,ctas_per_sm=2,seg_clocks=4096 > gpurun_out/prof4/grain.jsonl 2>&1
cat gpurun_out/prof4/grain.jsonl
ls -la gpurun_out/prof4
