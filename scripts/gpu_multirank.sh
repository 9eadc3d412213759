#!/bin/bash
# Exercise bench.py's N>1 path on a 1-GPU box: ranks share cuda:0 over gloo (debug backend);
# halo via the fused peer-memory path (CUDA IPC between processes) and via the pack/exchange path.
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_mr.log 2>&1
for H in p2p nccl; do
for NP in 2 4; do
  STOKESFO_BENCH_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $NP \
     --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus $NP --config C1 --steps 5 --warmup 3 --halo $H --check --no-e2e \
     > $OUT/bench_mr_${H}_$NP.json 2> $OUT/bench_mr_${H}_$NP.err; echo "halo=$H np=$NP exit $? $(head -c 300 $OUT/bench_mr_${H}_$NP.json | tr -d '\n' | cut -c1-120) check=$(grep -o 'halo_check[^,]*' $OUT/bench_mr_${H}_$NP.json)" >> $OUT/bench_mr.txt
done
done
cat $OUT/bench_mr.txt
