#!/bin/bash
# A/B timing of prebuilt libraries: tools/exp_libs.sh build/variants/a.so build/variants/b.so ...
# Each is copied over libsharp.so and timed (device-resident value only);
# runs the list twice (interleaved) to expose drift.
cd "$(dirname "$0")/.."
lib=paper_conf_icpp_fanjzac15_b200/libsharp.so
cp $lib build/libsharp.orig.so
for pass in 1 2; do
  for v in "$@"; do
    cp "$v" $lib
    r=$(python bench.py --steps 30 --warmup 3 --no-cpu --e2e-steps 0 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('%.0f Mpix/s  %.3f ms/step' % (d['value'], d['ms_per_step']))")
    echo "[$pass $(basename $v)] $r"
  done
done
cp build/libsharp.orig.so $lib
