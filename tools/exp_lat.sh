#!/bin/bash
# A/B of single-image latency (bench --frames 1, device-resident) for prebuilt libraries.
cd "$(dirname "$0")/.."
lib=paper_conf_icpp_fanjzac15_b200/libsharp.so
cp $lib build/libsharp.orig.so
for pass in 1 2; do
  for v in "$@"; do
    cp "$v" $lib
    for wh in 512x512 1920x1080 3840x2160; do
      w=${wh%x*}; h=${wh#*x}
      r=$(python bench.py --frames 1 --width $w --height $h --steps 200 --warmup 20 --no-cpu --e2e-steps 0 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('%.1f us' % (d['ms_per_step']*1e3))")
      echo "[$pass $(basename $v)] ${wh}: $r"
    done
  done
done
cp build/libsharp.orig.so $lib
