#!/bin/bash
# One gpurun call: build check, GPU tests, bench line, ncu launch list and one
# full capture of the step kernel.  Outputs land in gpurun_out/.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
cat MEASURED_PEAKS.json > gpurun_out/peaks.json 2>/dev/null
if [ "${SKIP_TESTS:-0}" != 1 ]; then
  timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
fi
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
if [ "${SKIP_NCU:-0}" != 1 ]; then
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
     python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > /dev/null 2>&1
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:step_kernel --launch-skip 3 -c 1 \
     -f -o gpurun_out/prof_step python bench.py --steps 1 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/ncu_full.log 2>&1
fi
echo done
