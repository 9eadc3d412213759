#!/bin/bash
# Build libstokesfo.so of the CURRENT tree with extra nvcc flags into build/libstokesfo_<name>.so
# (same-box A/B of compile-time design switches).  Usage: bash scripts/build_variant.sh NAME "-DSFO_X=1 ..."
set -e
ROOT=$(cd "$(dirname "$0")/.." && pwd)
mkdir -p "$ROOT/build"
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2 -shared \
  $2 -I "$ROOT/include" -o "$ROOT/build/libstokesfo_$1.so" "$ROOT/paper_conf_sc_antepara0cw24_b200/csrc/sfo_capi.cu" \
  "$ROOT/paper_conf_sc_antepara0cw24_b200/csrc/sfo_mesh.cpp"
echo "$ROOT/build/libstokesfo_$1.so"
