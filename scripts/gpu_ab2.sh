#!/bin/bash
# GPU tests then same-box A/B (bench lines) against an older build, for several bench arg sets.
# Usage: bash scripts/gpu_ab2.sh TAG OTHER_LIB "ARGS1" "ARGS2" ...
TAG=$1; OTHER=$2; shift 2
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu_$TAG.log
for A in "$@"; do
  for r in 1 2 3; do
    for L in new old; do
      if [ $L = new ]; then E=""; else E="STOKESFO_LIB=$OTHER"; fi
      env $E timeout 600 python bench.py $A --no-cpu-baseline --no-e2e > $OUT/ab_tmp.json 2>/dev/null
      echo "[$A] $L run$r $(python -c 'import json,sys; d=json.loads(open(sys.argv[1]).read()); print(round(d["value"]/1e9,4), round(d["roofline"]["kernel_ms"],4), round(d["roofline"]["frac"],4), d["clocks"]["sm_mhz"], d["clocks"]["reasons"])' $OUT/ab_tmp.json)" >> $OUT/samebox_$TAG.txt
    done
  done
done
cat $OUT/samebox_$TAG.txt
