#!/bin/bash
# Every committed profile artefact of profiles/<round>/ in one gpurun call:
# GPU tests, smoke, the default bench line, single-image lines (512^2, 1080p,
# 4K, 8K), the optimisation ladder (4K), row bands (8K / 16384^2: NCCL, p2p,
# one launch), the ncu launch list of the bench command, one full capture of
# the step kernel and one of the resident kernel.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
for wh in 512x512 1920x1080 3840x2160 7680x4320; do
  w=${wh%x*}; h=${wh#*x}
  timeout 300 python bench.py --frames 1 --width $w --height $h --steps 200 --warmup 10 --e2e-steps 20 \
    > gpurun_out/single_$wh.json 2>> gpurun_out/single.err
done
timeout 300 python bench.py --frames 32 --width 3840 --height 2160 --steps 20 --warmup 3 --e2e-steps 3 --no-cpu \
  > gpurun_out/batch_4k.json 2>> gpurun_out/single.err
timeout 900 python bench.py --workload ladder --steps 10 --warmup 3 > gpurun_out/ladder_4k.json 2> gpurun_out/ladder.err
for ex in nccl p2p one; do
  timeout 300 python bench.py --workload bands --exchange $ex --steps 50 --warmup 5 > gpurun_out/bands_${ex}_8k.json 2>> gpurun_out/bands.err
done
timeout 300 python bench.py --workload bands --exchange one --width 16384 --height 16384 --steps 20 --warmup 3 \
  > gpurun_out/bands_one_16k.json 2>> gpurun_out/bands.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
   python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:step_kernel --launch-skip 3 -c 1 \
   -f -o gpurun_out/prof_step python bench.py --steps 1 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:res_kernel --launch-skip 3 -c 1 \
   -f -o gpurun_out/prof_res python tools/step_time.py 4 1024 1920 1080 > gpurun_out/ncu_res.log 2>&1
echo done
