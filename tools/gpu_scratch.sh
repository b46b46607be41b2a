#!/bin/bash
# guard-band bounds tests
set -u
D=gpurun_out/g19; mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_bounds.py -m gpu -q -p no:cacheprovider --durations=5 > $D/pytest.txt 2>&1
echo "pytest exit $?" >> $D/pytest.txt
