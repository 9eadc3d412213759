#!/bin/bash
# One gpurun call, several steps: build, -m gpu suite, then each argument as a command line (run in order).
# Usage (under gpurun): bash scripts/gpu_batch.sh TAG "cmd1" "cmd2" ...
TAG=$1; shift
OUT=gpurun_out/batch_$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider -rf -x > $OUT/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
i=0
for C in "$@"; do
  i=$((i+1)); echo "== $C" >> $OUT/cmds.log
  bash -c "$C" >> $OUT/cmds.log 2>&1
done
tail -60 $OUT/cmds.log
