set -x
nvidia-smi -L
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -rf 2>&1 | tail -40 > gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
cat gpurun_out/pytest_gpu.log gpurun_out/smoke.log gpurun_out/bench.json; tail -5 gpurun_out/bench.err
