#!/bin/bash
# ncu --set full of the eval kernel for several bench arg sets.  Usage: bash scripts/gpu_ncu_ops.sh TAG "ARGS1" "ARGS2" ...
TAG=$1; shift
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
i=0
for A in "$@"; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval -s 3 -c 1 -o $OUT/prof_${TAG}_$i \
     python bench.py $A --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_${TAG}_$i.log 2>&1
  i=$((i+1))
done
echo done
