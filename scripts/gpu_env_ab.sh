#!/bin/bash
# Same-box A/B/n of environment settings of one build, interleaved, 3 rounds each.
# Usage (under gpurun): bash scripts/gpu_env_ab.sh TAG "BENCH ARGS" "ENV1" "ENV2" ...   ("-" = no extra env)
TAG=$1; ARGS=$2; shift 2
OUT=gpurun_out; mkdir -p $OUT
[ -f paper_conf_sc_antepara0cw24_b200/libstokesfo.so ] || python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
for r in 1 2 3; do
  for V in "$@"; do
    if [ "$V" = "-" ]; then E=""; else E="$V"; fi
    env $E timeout 600 python bench.py $ARGS --no-cpu-baseline --no-e2e > $OUT/ab_tmp.json 2>$OUT/ab_tmp.err
    echo "[$ARGS] [$V] run$r $(python -c 'import json,sys; d=json.loads(open(sys.argv[1]).read()); print(round(d["value"]/1e9,4), round(d["roofline"]["kernel_ms"],4), round(d["roofline"]["frac"],4), d["clocks"]["sm_mhz"], d["clocks"]["reasons"])' $OUT/ab_tmp.json 2>&1 | tail -1)" >> $OUT/samebox_$TAG.txt
  done
done
cat $OUT/samebox_$TAG.txt
