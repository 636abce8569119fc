#!/bin/bash
# A/B of the e2e leg (pinned 1024 x 1080p through sharp_run_batch) for prebuilt libraries.
cd "$(dirname "$0")/.."
lib=paper_conf_icpp_fanjzac15_b200/libsharp.so
cp $lib build/libsharp.orig.so
for pass in 1 2 3; do
  for v in "$@"; do
    cp "$v" $lib
    r=$(python tools/e2e_sweep.py 3 0 2>/dev/null | tail -1)
    echo "[$pass $(basename $v)] $r"
  done
done
cp build/libsharp.orig.so $lib
