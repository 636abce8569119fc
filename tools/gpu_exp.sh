#!/bin/bash
# A/B variants + wait statistics in one gpurun call.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
lib=paper_conf_icpp_fanjzac15_b200/libsharp.so
cp $lib build/libsharp.orig.so
if [ -f build/variants/waitstat.so ]; then
  cp build/variants/waitstat.so $lib
  timeout 120 python tools/waitstat.py > gpurun_out/waitstat.txt 2>&1
  cp build/libsharp.orig.so $lib
fi
ls build/variants/*.so | grep -v waitstat > /tmp/vlist
timeout 1200 bash tools/exp_libs.sh $(cat /tmp/vlist) > gpurun_out/exp.txt 2>&1
echo done
