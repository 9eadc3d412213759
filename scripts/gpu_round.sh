#!/bin/bash
# Round measurement pass: gpu_check (tests, smoke, C4 bench + reference arm, ncu launch list + full capture)
# then bench lines for the other configs/ops.  Usage: bash scripts/gpu_round.sh TAG
TAG=$1
OUT=gpurun_out; mkdir -p $OUT
bash scripts/gpu_check.sh $TAG C4
for A in "--config C3" "--config C5" "--config C4 --op resid" "--config C5 --op resid" "--config C4 --op jvp" "--config C4 --op jac_csr" "--config C4p"; do
  timeout 900 python bench.py $A --no-cpu-baseline >> $OUT/bench_${TAG}_lines.jsonl 2>> $OUT/bench_${TAG}_lines.err
done
echo done
