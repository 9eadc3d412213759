#!/bin/bash
# Quick measurement pass (under gpurun): build, -m gpu suite, smoke, default bench line, a few workload lines and
# ncu --set full of the named workloads. Usage: bash scripts/gpu_quick.sh TAG "bench args;bench args" [prof specs...]
TAG=$1; LINES=$2; shift 2
OUT=gpurun_out/quick_$TAG; mkdir -p $OUT
nvidia-smi -L > $OUT/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -rf -x > $OUT/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke exit $?" >> $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench_C4.json 2> $OUT/bench_C4.err
IFS=';' read -ra ARR <<< "$LINES"
for A in "${ARR[@]}"; do
  timeout 900 python bench.py $A --no-cpu-baseline >> $OUT/bench_lines.jsonl 2>> $OUT/bench_lines.err
done
if [ $# -gt 0 ]; then bash scripts/gpu_prof.sh $TAG "$@" > $OUT/prof.log 2>&1; fi
python - <<PY > $OUT/summary.txt
import json
for f in ["$OUT/bench_C4.json", "$OUT/bench_lines.jsonl"]:
    try: lines = open(f).readlines()
    except OSError: continue
    for ln in lines:
        if not ln.startswith("{"): continue
        d = json.loads(ln)
        c = d.get("config", {})
        r = d.get("roofline", {})
        print(d.get("impl", "ours"), c.get("workload", "")[:30], c.get("op"), c.get("geometry"), "%.4g" % d["value"],
              "ms %.3f" % d["ms_per_step"], "frac %.3f" % r.get("frac", 0), "sus %.4g" % d.get("sustained", {}).get("value", 0))
PY
cat $OUT/summary.txt; tail -3 $OUT/pytest_gpu.log; tail -1 $OUT/smoke.log
