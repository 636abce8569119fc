#!/bin/bash
# Timing experiments: rebuild libsharp.so with each flag set and run the bench
# (device-resident value only).  Usage: tools/exp.sh "" "-DSHARP_EXP_NO_BORDER" ...
cd "$(dirname "$0")/.."
for flags in "$@"; do
  rm -f paper_conf_icpp_fanjzac15_b200/libsharp.so
  make -s paper_conf_icpp_fanjzac15_b200/libsharp.so EXTRA_NVCC_FLAGS="$flags" > /dev/null 2>&1 || { echo "build failed: $flags"; continue; }
  v=$(python bench.py --steps 30 --warmup 3 --no-cpu --e2e-steps 0 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('%.0f Mpix/s  %.3f ms/step' % (d['value'], d['ms_per_step']))")
  echo "[$flags] $v"
done
rm -f paper_conf_icpp_fanjzac15_b200/libsharp.so
make -s paper_conf_icpp_fanjzac15_b200/libsharp.so > /dev/null 2>&1
