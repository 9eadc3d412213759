#!/bin/bash
# Exercise bench.py's N>1 path on a 1-GPU box: 2 and 4 ranks sharing cuda:0 over gloo (debug backend).
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_mr.log 2>&1
for NP in 2 4; do
  STOKESFO_BENCH_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $NP \
     --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus $NP --config C1 --steps 5 --warmup 3 \
     > $OUT/bench_mr_$NP.json 2> $OUT/bench_mr_$NP.err; echo "np=$NP exit $?" >> $OUT/bench_mr.txt
done
cat $OUT/bench_mr.txt
