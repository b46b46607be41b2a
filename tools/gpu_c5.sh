# Re-verify the round's state on a fresh box, then the configs[4] sweep.
mkdir -p gpurun_out/c5
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > gpurun_out/c5/gpu.txt
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/c5/pytest_gpu.txt 2>&1; tail -3 gpurun_out/c5/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c5/smoke.txt 2>&1; tail -2 gpurun_out/c5/smoke.txt
timeout 900 python bench.py > gpurun_out/c5/n1_default.json 2> gpurun_out/c5/n1_default.err; cat gpurun_out/c5/n1_default.json
timeout 1500 python tools/sweep_c5.py > gpurun_out/c5/sweep.jsonl 2> gpurun_out/c5/sweep.err; wc -l gpurun_out/c5/sweep.jsonl; tail -3 gpurun_out/c5/sweep.err
# cuRAND on the byte counts of the materialise calls (2^22 x 2^12 and 2^22 x 2^15 bits)
(cd tools/microbench && timeout 300 ./curand_bench 2147483648 && timeout 300 ./curand_bench 17179869184) > gpurun_out/c5/curand.log 2>&1; tail -12 gpurun_out/c5/curand.log
