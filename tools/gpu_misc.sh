#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 300 python bench.py --workload bands --steps 50 --warmup 5 > gpurun_out/bands_nccl_8k.json 2> gpurun_out/bands.err
timeout 300 python bench.py --workload bands --exchange p2p --steps 50 --warmup 5 > gpurun_out/bands_p2p_8k.json 2>> gpurun_out/bands.err
timeout 300 python bench.py --workload bands --exchange p2p --width 16384 --height 16384 --steps 20 --warmup 3 > gpurun_out/bands_p2p_16k.json 2>> gpurun_out/bands.err
timeout 300 python bench.py --frames 1 --steps 200 --warmup 10 --e2e-steps 20 > gpurun_out/single_1080p.json 2> gpurun_out/single.err
timeout 300 python bench.py --frames 1 --width 512 --height 512 --steps 200 --warmup 10 --e2e-steps 20 > gpurun_out/single_512.json 2>> gpurun_out/single.err
echo done
