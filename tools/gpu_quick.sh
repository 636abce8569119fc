#!/bin/bash
# Smoke + GPU tests (short timeouts), then A/B of build/variants/*.so.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
if grep -q "smoke ok" gpurun_out/smoke.log; then
  timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
  ls build/variants/*.so > /tmp/vlist
  timeout 900 bash tools/exp_libs.sh $(cat /tmp/vlist) > gpurun_out/exp.txt 2>&1
fi
echo done
