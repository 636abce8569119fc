#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
cp paper_conf_icpp_fanjzac15_b200/libsharp.so build/libsharp.cur.so
cp build/libsharp_tl.so paper_conf_icpp_fanjzac15_b200/libsharp.so
timeout 300 python tools/timeline.py > gpurun_out/timeline.txt 2>&1
cp build/libsharp.cur.so paper_conf_icpp_fanjzac15_b200/libsharp.so
timeout 900 bash tools/exp_lat.sh $(ls build/variants/*.so) > gpurun_out/lat.txt 2>&1
timeout 900 bash tools/exp_libs.sh $(ls build/variants/*.so) > gpurun_out/exp.txt 2>&1
echo done
