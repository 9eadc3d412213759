#!/bin/bash
# ncu --set full of the evaluation kernel for several workloads, summarised ON THE BOX (the .ncu-rep
# files stay there; only text comes back): per workload profiles/<TAG>_<name>_ncu_summary.md, the
# shared-memory wavefront breakdown, and the traffic.json entry keyed by this build's source revision.
# Usage (under gpurun): bash scripts/gpu_prof.sh TAG "name|key|bench args" ...
TAG=$1; shift
OUT=gpurun_out/prof_$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for spec in "$@"; do
  IFS='|' read -r NAME KEY ARGS <<< "$spec"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval -s 3 -c 1 -o /tmp/prof_${TAG}_$NAME \
     python bench.py $ARGS --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/ncu_$NAME.log 2>&1
  python scripts/ncu_summary.py --tag ${TAG}_$NAME --rep /tmp/prof_${TAG}_$NAME.ncu-rep --key "$KEY" \
     --note "ncu --set full --clock-control none of: python bench.py $ARGS" > /dev/null 2> $OUT/summary_$NAME.err
  UNITS=$(python -c "import sys; sys.path.insert(0,'.'); import bench; print(bench.units_per_launch('$KEY'))")
  python scripts/ncu_smem_breakdown.py /tmp/prof_${TAG}_$NAME.ncu-rep $UNITS > $OUT/smem_$NAME.txt 2>&1
  ncu -i /tmp/prof_${TAG}_$NAME.ncu-rep --page raw --csv > $OUT/raw_$NAME.csv 2>/dev/null
  cp profiles/${TAG}_${NAME}_ncu_summary.md $OUT/
done
cp profiles/traffic.json $OUT/traffic.json
echo done
