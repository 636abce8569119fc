#!/bin/bash
# A/B timing of build/variants/*.so only.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
ls build/variants/*.so > /tmp/vlist
timeout 1500 bash tools/exp_libs.sh $(cat /tmp/vlist) > gpurun_out/exp.txt 2>&1
echo done
