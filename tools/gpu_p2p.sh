#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_p2p_bands.py -x -q > gpurun_out/p2p_tests.log 2>&1; echo "p2p rc=$?" >> gpurun_out/p2p_tests.log
nvidia-smi --query-gpu=name,utilization.gpu --format=csv >> gpurun_out/p2p_tests.log 2>&1
if grep -q "p2p rc=0" gpurun_out/p2p_tests.log; then
  timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
fi
echo done
