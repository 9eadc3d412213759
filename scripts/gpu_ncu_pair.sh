#!/bin/bash
# ncu --set full of the eval kernel for the in-tree library and another build.
# Usage: bash scripts/gpu_ncu_pair.sh TAG OTHER_LIB "bench args"
TAG=$1; OTHER=$2; ARGS=$3
OUT=gpurun_out; mkdir -p $OUT
for L in new old; do
  if [ $L = new ]; then E=""; else E="STOKESFO_LIB=$OTHER"; fi
  env $E timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval -s 3 -c 1 -o $OUT/prof_${TAG}_$L \
     python bench.py $ARGS --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_${TAG}_$L.log 2>&1
done
