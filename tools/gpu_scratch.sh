D=gpurun_out/sw8; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_aes.py tests/test_gpu_contract.py tests/test_gpu_api.py -q -x -p no:cacheprovider > $D/pytest.txt 2>&1
timeout 600 python bench.py --cipher aes128ctr --no-context --no-cpu-baseline --no-e2e --steps 10 > $D/aes_c2.json 2>$D/aes_c2.err
timeout 600 python bench.py --cipher aes128ctr --workload c4 --no-context --no-cpu-baseline --no-e2e --steps 2000 --warmup 20 > $D/aes_c4.json 2>$D/aes_c4.err
SASS=1 bash tools/gpu.sh capture sw8 aes_consume aes_ctr --cipher aes128ctr --layout checksum --bits 16384 --reps 2
SASS=1 bash tools/gpu.sh capture sw8 aes_rowmajor rowmajor_lanes --cipher aes128ctr --layout row_major --bits 16384 --reps 2
