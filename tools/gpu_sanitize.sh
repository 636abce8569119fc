#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  echo "=== $tool" >> gpurun_out/sanitizer.txt
  timeout 600 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_workload.py >> gpurun_out/sanitizer.txt 2>&1
  echo "rc=$?" >> gpurun_out/sanitizer.txt
done
echo done
