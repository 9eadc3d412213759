#!/bin/bash
# ncu --set full of one eval launch + the per-instruction source page (SASS with CUDA line correlation) as CSV,
# for attributing stall samples to phases of the kernel.  Usage (under gpurun): bash scripts/gpu_prof_src.sh TAG "bench args"
TAG=$1; ARGS=$2
OUT=gpurun_out/src_$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval -s 3 -c 1 -o /tmp/src_$TAG \
   python bench.py $ARGS --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --sustain 0 > $OUT/ncu.log 2>&1
ncu -i /tmp/src_$TAG.ncu-rep --page source --csv --print-source cuda,sass > $OUT/source_cuda_sass.csv 2> $OUT/src.err
ncu -i /tmp/src_$TAG.ncu-rep --page source --csv --print-source sass > $OUT/source_sass.csv 2>> $OUT/src.err
gzip -f $OUT/source_cuda_sass.csv $OUT/source_sass.csv
ls -la $OUT
