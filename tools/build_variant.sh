#!/bin/bash
# Build a variant of libapointer.so with extra -D flags into build/variants/lib_<name>.so
# (same flags as the Makefile's product build, plus $2).
# usage: tools/build_variant.sh <name> "<-DFLAG ...>"
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
/usr/local/cuda/bin/nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo \
  -Xcompiler -fPIC -Iinclude -Ipaper_conf_isca_shaharbs16_b200/csrc --expt-relaxed-constexpr \
  -rdc=true -maxrregcount=${MAXRREG:-64} $2 \
  -shared paper_conf_isca_shaharbs16_b200/csrc/*.cu -o build/variants/lib_$1.so -lcuda
echo built build/variants/lib_$1.so
