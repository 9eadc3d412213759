#!/bin/bash
# Short round-end pass on the final sources: -m gpu suite, smoke, default bench + reference arm, the global-fill
# lines, launch list, and ncu captures re-keying profiles/traffic.json to this build. Usage: bash scripts/gpu_final2.sh TAG
TAG=$1
OUT=gpurun_out/final_$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -rf > $OUT/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke exit $?" >> $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench_C4.json 2> $OUT/bench_C4.err
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $OUT/bench_reference.json 2> $OUT/bench_reference.err
for A in "--config C3" "--config C4p" "--config C5" "--config C4 --geometry compact" "--config C4 --geometry on_the_fly" \
         "--config C4 --op jac_packed" "--config C4 --op jac_global" "--config C4 --op jac_global --global-format packed" \
         "--config C3 --op jac_global" "--config C5 --op jac_global" "--config C4 --op resid" "--config C4 --op jvp_y"; do
  timeout 900 python bench.py $A --no-cpu-baseline >> $OUT/bench_lines.jsonl 2>> $OUT/bench_lines.err
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
   python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --sustain 0 > $OUT/ncu_launch.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_c5global.csv \
   python bench.py --config C5 --op jac_global --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --sustain 0 > $OUT/ncu_launch2.log 2>&1
bash scripts/gpu_prof.sh $TAG "c4jac|C4:hex8:jacobian:stored|--config C4" "c5jac|C5:wedge6:jacobian:stored|--config C5" \
   "c4cmp|C4:hex8:jacobian:compact|--config C4 --geometry compact" "c4res|C4:hex8:resid:stored|--config C4 --op resid" \
   "c4jvpy|C4:hex8:jvp_y:stored|--config C4 --op jvp_y" "c4otf|C4:hex8:jacobian:on_the_fly|--config C4 --geometry on_the_fly" \
   "c3jac|C3:hex8:jacobian:stored|--config C3" > $OUT/prof.log 2>&1
python scripts/bench_table.py $OUT/bench_C4.json $OUT/bench_lines.jsonl > $OUT/table.md
cat $OUT/table.md; tail -3 $OUT/pytest_gpu.log; tail -1 $OUT/smoke.log
