#!/bin/bash
# NEXT-2 round: GPU tests, aux measurements (pull vs atomic CSR), bench jac_csr vs jacobian lines, ncu.
TAG=$1
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu_$TAG.log
timeout 900 python scripts/bench_aux.py --config C3 --ops csr --out $OUT/aux_${TAG}_C3.jsonl > $OUT/aux_${TAG}_C3.log 2>&1
STOKESFO_CSR_ATOMIC=1 timeout 900 python scripts/bench_aux.py --config C3 --ops csr --out $OUT/aux_${TAG}_C3_atomic.jsonl > $OUT/aux_${TAG}_C3_atomic.log 2>&1
timeout 1200 python scripts/bench_aux.py --config C4 --ops csr --out $OUT/aux_${TAG}_C4.jsonl > $OUT/aux_${TAG}_C4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:csr_gather -s 3 -c 1 -o $OUT/prof_${TAG}_gather \
   python scripts/bench_aux.py --config C3 --ops csr > $OUT/ncu_gather_$TAG.log 2>&1
echo done
