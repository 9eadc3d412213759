#!/bin/bash
# Build libstokesfo.so of a git revision into build/libstokesfo_<rev>.so (same-box A/B baselines).
set -e
# Usage: bash scripts/build_rev.sh REV
REV=$1
ROOT=$(cd "$(dirname "$0")/.." && pwd)
T=$(mktemp -d)
git -C "$ROOT" archive "$REV" include paper_conf_sc_antepara0cw24_b200/csrc | tar -x -C "$T"
mkdir -p "$ROOT/build"
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2 -shared \
  -I "$T/include" -o "$ROOT/build/libstokesfo_$REV.so" "$T/paper_conf_sc_antepara0cw24_b200/csrc/sfo_capi.cu" \
  "$T/paper_conf_sc_antepara0cw24_b200/csrc/sfo_mesh.cpp"
rm -rf "$T"
echo "$ROOT/build/libstokesfo_$REV.so"
