#!/bin/bash
# NEXT-1 Table II analogue: StokesFOResid (Fig. 2) times under each __launch_bounds__ variant library
# (scripts/build_variant.sh lb<MAXT>_<MINB> "-DSFO_ALBANY_MAXT=.. -DSFO_ALBANY_MINB=..").
# Usage (under gpurun): bash scripts/gpu_fig2_lb.sh TAG LIB...   ("cur" = the in-tree build)
TAG=$1; shift
OUT=gpurun_out/fig2lb_$TAG; mkdir -p $OUT
for L in "$@"; do
  if [ $L = cur ]; then E=""; N=default; else E="STOKESFO_LIB=$L"; N=$(basename $L .so); fi
  env $E timeout 900 python scripts/bench_fig2.py --config C4p --reps 10 --out $OUT/$N.json > /dev/null 2> $OUT/$N.err
done
ls $OUT
