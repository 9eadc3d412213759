#!/bin/bash
# Quick A/B on the GPU: parity tests + bench-only lines for each env setting.
# Usage: bash scripts/gpu_variants.sh TAG CFG "ENV1" "ENV2" ...
TAG=$1; CFG=$2; shift 2
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
i=0
for V in "$@"; do
  env $V timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider > $OUT/pytest_${TAG}_$i.log 2>&1; echo "[$V] pytest exit $?" >> $OUT/pytest_${TAG}_$i.log
  env $V timeout 600 python bench.py --config $CFG --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > $OUT/bench_${TAG}_$i.json 2> $OUT/bench_${TAG}_$i.err
  echo "[$V] $(cat $OUT/bench_${TAG}_$i.json | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["roofline"]["frac"], d["clocks"])')" >> $OUT/variants_$TAG.txt
  i=$((i+1))
done
cat $OUT/variants_$TAG.txt
