#!/bin/bash
# One full ncu capture of the step kernel (bench workload, 1 launch).
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:step_kernel --launch-skip 3 -c 1 \
   -f -o gpurun_out/${NCU_NAME:-prof_new} python bench.py --steps 1 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/ncu_full.log 2>&1
echo done
