#!/bin/bash
# GPU tests, the Fig. 2 experiment (timing + ncu dram bytes), resid-op bench line.
TAG=${1:-r09}
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu_$TAG.log
timeout 900 python scripts/bench_fig2.py --config C4p --out $OUT/fig2_$TAG.json > $OUT/fig2_$TAG.log 2>&1
timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
   --log-file $OUT/fig2_ncu_$TAG.csv python scripts/bench_fig2.py --config C4p --ncu > $OUT/fig2_ncu_$TAG.log 2>&1
timeout 600 python bench.py --config C4 --op resid --steps 20 --warmup 5 > $OUT/bench_resid_$TAG.json 2> $OUT/bench_resid_$TAG.err
echo done
