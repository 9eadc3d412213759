#!/bin/bash
# Round-end measurement pass (under gpurun): build, full -m gpu suite, smoke, the default bench line, the reference
# arm, bench lines of every workload / op / geometry mode, the ncu launch list of the default bench, and ncu --set full
# captures summarised on the box (profiles/<TAG>_*_ncu_summary.md, traffic.json keyed by this build's revision).
# Usage: bash scripts/gpu_final.sh TAG
TAG=$1
OUT=gpurun_out/final_$TAG; mkdir -p $OUT
nvidia-smi -L > $OUT/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -rf > $OUT/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke exit $?" >> $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench_C4.json 2> $OUT/bench_C4.err
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $OUT/bench_reference.json 2> $OUT/bench_reference.err
for A in "--config C3" "--config C5" "--config C4p" "--config C4 --op resid" "--config C5 --op resid" \
         "--config C4 --op jvp" "--config C4 --geometry compact" "--config C4 --op jvp --geometry compact" \
         "--config C5 --geometry compact" "--config C4 --geometry on_the_fly" "--config C4 --op jac_global" \
         "--config C4 --op jac_csr" "--config C4 --op jvp_y" "--config C4 --op jvp_y --geometry compact" "--config C1" \
         "--config C4 --op jac_global --global-format full" "--config C3 --op jac_global" \
         "--config C5 --op jac_global --global-format full" "--config C5 --op jvp" "--config C4 --op jvp --geometry compact"; do
  timeout 900 python bench.py $A --no-cpu-baseline >> $OUT/bench_lines.jsonl 2>> $OUT/bench_lines.err
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
   python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --sustain 0 > $OUT/ncu_launch.log 2>&1
bash scripts/gpu_prof.sh $TAG "c4jac|C4:hex8:jacobian:stored|--config C4" "c5jac|C5:wedge6:jacobian:stored|--config C5" \
   "c4jvp|C4:hex8:jvp:stored|--config C4 --op jvp" "c4res|C4:hex8:resid:stored|--config C4 --op resid" \
   "c5res|C5:wedge6:resid:stored|--config C5 --op resid" "c4cmp|C4:hex8:jacobian:compact|--config C4 --geometry compact" \
   "c4otf|C4:hex8:jacobian:on_the_fly|--config C4 --geometry on_the_fly" "c3jac|C3:hex8:jacobian:stored|--config C3" \
   "c4pjac|C4p:hex8:jacobian:stored|--config C4p" "c4jvpy|C4:hex8:jvp_y:stored|--config C4 --op jvp_y" \
   "c5cmp|C5:wedge6:jacobian:compact|--config C5 --geometry compact" > $OUT/prof.log 2>&1
python - <<PY > $OUT/summary.txt
import json
for f in ["$OUT/bench_C4.json", "$OUT/bench_reference.json", "$OUT/bench_lines.jsonl"]:
    for ln in open(f):
        if not ln.startswith("{"): continue
        d = json.loads(ln)
        c = d.get("config", {})
        r = d.get("roofline", {})
        print(d.get("impl", "ours"), c.get("workload", "")[:30], c.get("op"), c.get("geometry"), "%.4g" % d["value"],
              "ms %.3f" % d["ms_per_step"], "frac %.3f" % r.get("frac", 0), "sus %.4g" % d.get("sustained", {}).get("value", 0))
PY
cat $OUT/summary.txt; tail -3 $OUT/pytest_gpu.log; tail -1 $OUT/smoke.log
