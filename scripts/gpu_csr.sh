#!/bin/bash
# NEXT-2 round: GPU tests (csr subset), aux measurements, bench jac_csr vs jacobian lines, ncu of the fused kernel.
TAG=$1
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu_$TAG.log
timeout 900 python scripts/bench_aux.py --config C3 --ops scatter_r,csr --out $OUT/aux_${TAG}_C3.jsonl > $OUT/aux_${TAG}_C3.log 2>&1
for A in "--config C3 --op jac_csr" "--config C3" "--config C4 --op jac_csr" "--config C5 --op jac_csr"; do
  timeout 900 python bench.py $A --no-cpu-baseline --no-e2e >> $OUT/bench_$TAG.jsonl 2>> $OUT/bench_$TAG.err
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval -s 3 -c 1 -o $OUT/prof_${TAG}_csr \
   python bench.py --config C3 --op jac_csr --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_full_$TAG.log 2>&1
echo done
