#!/bin/bash
# ncu captures of the main workloads on the current sources (re-keys profiles/traffic.json to this build's source
# revision) + the default bench line and smoke. Usage: bash scripts/gpu_rekey.sh TAG
TAG=$1
OUT=gpurun_out/rekey_$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke exit $?" >> $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench_C4.json 2> $OUT/bench_C4.err
bash scripts/gpu_prof.sh $TAG "c4jac|C4:hex8:jacobian:stored|--config C4" "c5jac|C5:wedge6:jacobian:stored|--config C5" \
   "c4cmp|C4:hex8:jacobian:compact|--config C4 --geometry compact" "c4res|C4:hex8:resid:stored|--config C4 --op resid" \
   "c4jvpy|C4:hex8:jvp_y:stored|--config C4 --op jvp_y" "c4otf|C4:hex8:jacobian:on_the_fly|--config C4 --geometry on_the_fly" \
   "c3jac|C3:hex8:jacobian:stored|--config C3" > $OUT/prof.log 2>&1
python scripts/bench_table.py $OUT/bench_C4.json > $OUT/table.md
cat $OUT/table.md; tail -1 $OUT/smoke.log
