#!/bin/bash
# Full GPU tests, then bench lines for several argument sets, ncu full capture of the last.
# Usage: bash scripts/gpu_ab.sh TAG "BENCH ARGS 1" "BENCH ARGS 2" ...
TAG=$1; shift
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu_$TAG.log
i=0
for A in "$@"; do
  timeout 600 python bench.py $A --no-cpu-baseline --no-e2e > $OUT/bench_${TAG}_$i.json 2> $OUT/bench_${TAG}_$i.err
  echo "[$A] $(python -c 'import json,sys; d=json.loads(open(sys.argv[1]).read()); print(round(d["value"]/1e9,4), "Gcells/s", round(d["roofline"]["kernel_ms"],3), "ms", round(d["roofline"]["frac"],3), d["clocks"])' $OUT/bench_${TAG}_$i.json)" >> $OUT/ab_$TAG.txt
  i=$((i+1))
done
if [ -n "$NCU_ARGS" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval -s 3 -c 1 -o $OUT/prof_$TAG \
     python bench.py $NCU_ARGS --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_full_$TAG.log 2>&1
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$TAG.csv \
     python bench.py $NCU_ARGS --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_launch_$TAG.log 2>&1
fi
cat $OUT/ab_$TAG.txt
