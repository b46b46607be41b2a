# ncu captures for the ROW_MAJOR staging variants and the init kernels.
python -c "from paper_conf_icppw_monfaredhkzrg20_b200 import build as b; b.build()" || exit 1
mkdir -p gpurun_out/prof3
cap() {
  name=$1; shift
  ncu --set full --clock-control none --import-source on -k regex:$1 -s 1 -c 1 -o /tmp/prof_$name "${@:2}" > gpurun_out/prof3/ncu_$name.log 2>&1
  ncu -i /tmp/prof_$name.ncu-rep --page raw --csv > gpurun_out/prof3/${name}_raw.csv 2>/dev/null
  ncu -i /tmp/prof_$name.ncu-rep --page details --csv > gpurun_out/prof3/${name}_details.csv 2>/dev/null
  ncu -i /tmp/prof_$name.ncu-rep --page source --csv --print-source sass > gpurun_out/prof3/${name}_source.csv 2>/dev/null
  rm -f /tmp/prof_$name.ncu-rep
}
cap grain_rm4 keystream_kernel python tools/prof_driver.py --cipher grain --layout row_major --bits 16384 --reps 2 --opt rm_slots=4
cap grain_rm8 keystream_kernel python tools/prof_driver.py --cipher grain --layout row_major --bits 16384 --reps 2 --opt rm_slots=8
cap m2_rm4 keystream_kernel python tools/prof_driver.py --layout row_major --bits 16384 --reps 2 --rm-ws 0 --opt rm_slots=4
cap preclock m2_preclock python tools/prof_driver.py --layout checksum --bits 32 --reps 1
cap slice slice_bits python tools/prof_driver.py --layout checksum --bits 32 --reps 1
ls -la gpurun_out/prof3
