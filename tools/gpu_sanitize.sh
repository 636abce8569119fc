#!/bin/bash
# compute-sanitizer over every path (tools/sanitize_workload.py); the summary
# goes to gpurun_out/sanitizer.txt.  initcheck serialises kernels, so the
# band modes whose kernels wait on each other (peer-memory exchange) are
# skipped under it (they would wait forever and trap).
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
rm -f gpurun_out/sanitizer.txt
for tool in memcheck racecheck synccheck initcheck; do
  echo "=== $tool" >> gpurun_out/sanitizer.txt
  SANITIZE_TOOL=$tool timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_workload.py \
    >> gpurun_out/sanitizer.txt 2>&1
  echo "rc=$?" >> gpurun_out/sanitizer.txt
done
echo done
