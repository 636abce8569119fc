#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
timeout 300 python bench.py --frames 1 --steps 200 --warmup 10 --e2e-steps 20 --no-cpu > gpurun_out/single_1080p.json 2> gpurun_out/single.err
timeout 300 python bench.py --frames 1 --width 3840 --height 2160 --steps 200 --warmup 10 --e2e-steps 20 --no-cpu > gpurun_out/single_4k.json 2>> gpurun_out/single.err
timeout 300 python bench.py --frames 1 --width 512 --height 512 --steps 200 --warmup 10 --e2e-steps 20 --no-cpu > gpurun_out/single_512.json 2>> gpurun_out/single.err
timeout 300 python bench.py --workload bands --steps 50 --warmup 5 --no-cpu > gpurun_out/bands_nccl_8k.json 2>> gpurun_out/single.err
ls build/variants/*.so > /tmp/vlist
timeout 900 bash tools/exp_libs.sh $(cat /tmp/vlist) > gpurun_out/exp.txt 2>&1
echo done
