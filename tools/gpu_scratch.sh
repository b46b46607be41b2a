export SASS=1
bash tools/gpu.sh capture ws2d lfsr_ws2 keystream_rm_ws2 --cipher lfsr128 --layout row_major --bits 32768 --reps 2 --opt rm_ws=2
