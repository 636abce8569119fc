#!/bin/bash
# ncu launch list of every kernel (duration + DRAM bytes) for tools/all_kernels_workload.py.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  --csv --log-file gpurun_out/all_kernels.csv python tools/all_kernels_workload.py > gpurun_out/all_kernels.log 2>&1
echo done
