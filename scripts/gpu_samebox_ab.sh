#!/bin/bash
# Same-box A/B of two library builds: bash scripts/gpu_samebox_ab.sh TAG OTHER_LIB "bench args"
TAG=$1; OTHER=$2; ARGS=$3
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
for r in 1 2 3; do
  for L in new old; do
    if [ $L = new ]; then E=""; else E="STOKESFO_LIB=$OTHER"; fi
    env $E timeout 600 python bench.py $ARGS --no-cpu-baseline --no-e2e > $OUT/ab_${TAG}_${L}_$r.json 2>/dev/null
    echo "$L run$r $(python -c 'import json,sys; d=json.loads(open(sys.argv[1]).read()); print(round(d["value"]/1e9,4), round(d["roofline"]["kernel_ms"],3), round(d["roofline"]["frac"],3))' $OUT/ab_${TAG}_${L}_$r.json)" >> $OUT/samebox_$TAG.txt
  done
done
cat $OUT/samebox_$TAG.txt
