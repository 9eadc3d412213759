#!/bin/bash
# GPU tests + auxiliary-op measurements (scripts/bench_aux.py).
# Usage (under gpurun): bash scripts/gpu_aux.sh TAG [pytest -k expr]
TAG=$1; K=${2:-}
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
if [ -n "$K" ]; then
  timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "$K" > $OUT/pytest_gpu_$TAG.log 2>&1
else
  timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu_$TAG.log 2>&1
fi
echo "pytest exit $?" >> $OUT/pytest_gpu_$TAG.log
timeout 900 python scripts/bench_aux.py --config C3 --out $OUT/aux_${TAG}_C3.jsonl > $OUT/aux_${TAG}_C3.log 2>&1
timeout 900 python scripts/bench_aux.py --config C4 --ops basal,lateral --out $OUT/aux_${TAG}_C4.jsonl > $OUT/aux_${TAG}_C4.log 2>&1
echo done
