#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_workload.py > gpurun_out/racecheck.txt 2>&1
echo "rc=$?" >> gpurun_out/racecheck.txt
