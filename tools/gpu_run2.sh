mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_mickey2.py -m gpu -q -rf -k preclock 2>&1 | tail -5
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
cat gpurun_out/bench.json; tail -5 gpurun_out/bench.err
