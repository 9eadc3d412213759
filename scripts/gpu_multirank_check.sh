#!/bin/bash
# bench.py N>1 path at full size on ONE GPU (ranks share it over gloo; CUDA IPC between the rank processes):
# every line's halo_check_max_rel_err compares each rank's halo-summed R (and Y for jvp) with a one-GPU
# evaluation of the whole mesh.  Usage (under gpurun): bash scripts/gpu_multirank_check.sh TAG
TAG=$1; OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for A in "--config C4 --halo p2p" "--config C4 --halo nccl" "--config C5 --halo p2p" "--config C4 --op jvp --halo p2p" \
         "--config C4 --op jvp --halo nccl"; do
  STOKESFO_BENCH_BACKEND=gloo timeout 1200 python bench.py --gpus 2 --check --steps 5 --warmup 3 --no-e2e --sustain 0 $A \
     > $OUT/mr_tmp.json 2> $OUT/mr_tmp.err
  python -c "
import json,sys
try:
    d=json.loads(open('$OUT/mr_tmp.json').read().strip().splitlines()[-1])
    print('[$A]', 'n_gpus', d['n_gpus'], 'halo', d['halo'][:30], 'check', d.get('halo_check_max_rel_err'), 'per_rank_cells', [r['cells'] for r in d['per_rank']])
except Exception as e:
    print('[$A] FAILED', e, open('$OUT/mr_tmp.err').read()[-800:])
" >> $OUT/multirank_$TAG.txt
done
cat $OUT/multirank_$TAG.txt
