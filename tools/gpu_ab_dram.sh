#!/bin/bash
# A/B timing of build/variants/*.so plus DRAM bytes of one step-kernel launch per variant.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
ls build/variants/*.so > /tmp/vlist
timeout 900 bash tools/exp_libs.sh $(cat /tmp/vlist) > gpurun_out/exp.txt 2>&1
lib=paper_conf_icpp_fanjzac15_b200/libsharp.so
cp $lib build/libsharp.orig2.so
for v in $(cat /tmp/vlist); do
  cp $v $lib
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:step_kernel --launch-skip 3 -c 1 --csv python bench.py --steps 1 --warmup 3 --no-cpu --e2e-steps 0 2>/dev/null | grep -E "dram__|gpu__time" | awk -F'","' -v n=$(basename $v) '{print n, $(NF-2), $(NF-1), $NF}' >> gpurun_out/exp.txt
done
cp build/libsharp.orig2.so $lib
echo done
