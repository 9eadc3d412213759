#!/bin/bash
# Under gpurun: DFMA vs DMMA throughput and power (nvidia-smi every 50 ms during each run).
OUT=gpurun_out; mkdir -p $OUT
[ -x build/micro_fp64 ] || /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/micro_fp64 scripts/micro_fp64.cu
for M in dfma dmma dfma dmma; do
  for W in 8 16; do
    nvidia-smi --id=0 --query-gpu=clocks.sm,power.draw,clocks_event_reasons.sw_power_cap --format=csv,noheader,nounits -lms 50 > $OUT/micro_smi.csv &
    P=$!
    R=$(./build/micro_fp64 $M 3 $W)
    kill $P; wait $P 2>/dev/null
    S=$(python -c "
import sys
rows=[l.split(', ') for l in open('$OUT/micro_smi.csv') if l.strip()]
busy=[(float(r[0]),float(r[1])) for r in rows if float(r[1])>250]
busy=busy[len(busy)//4:]
m=lambda v: sorted(v)[len(v)//2] if v else -1
print('\"sm_mhz\": %s, \"power_w\": %s, \"samples\": %d' % (m([b[0] for b in busy]), m([b[1] for b in busy]), len(busy)))")
    echo "${R%\}}, $S}" >> $OUT/micro_fp64.jsonl
  done
done
cat $OUT/micro_fp64.jsonl
