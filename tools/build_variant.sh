#!/bin/bash
# Builds a variant of libsharp.so with extra nvcc flags into build/variants/NAME.so
# (the in-tree libsharp.so is rebuilt normally afterwards).
# usage: tools/build_variant.sh NAME "-DFLAG ..."
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
touch paper_conf_icpp_fanjzac15_b200/csrc/*.cu
make -s EXTRA_NVCC_FLAGS="$2" paper_conf_icpp_fanjzac15_b200/libsharp.so
cp paper_conf_icpp_fanjzac15_b200/libsharp.so build/variants/$1.so
touch paper_conf_icpp_fanjzac15_b200/csrc/*.cu
make -s paper_conf_icpp_fanjzac15_b200/libsharp.so
