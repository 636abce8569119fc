#!/bin/bash
# GPU parity tests of the current build, then A/B timing of build/variants/*.so.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
ls build/variants/*.so > /tmp/vlist
timeout 1200 bash tools/exp_libs.sh $(cat /tmp/vlist) > gpurun_out/exp.txt 2>&1
echo done
