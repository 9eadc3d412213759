set -x
OUT=gpurun_out/r2g; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
B="python bench.py --config C4 --op jac_global --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --sustain 0"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launch_packed.csv $B > $OUT/l1.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launch_full.csv $B --global-format full > $OUT/l2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:csr_gather -s 3 -c 1 -o /tmp/gpack $B > $OUT/n1.log 2>&1
python scripts/ncu_summary.py --tag r2g_gpack --rep /tmp/gpack.ncu-rep --key C4:hex8:csr_gather_packed:stored --note "ncu --set full of csr_gather_kernel<8,false,true> in: $B" > /dev/null 2>$OUT/s1.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:csr_gather -s 3 -c 1 -o /tmp/gfull $B --global-format full > $OUT/n2.log 2>&1
python scripts/ncu_summary.py --tag r2g_gfull --rep /tmp/gfull.ncu-rep --key C4:hex8:csr_gather_full:stored --note "ncu --set full of csr_gather_kernel<8,false,false> in: $B --global-format full" > /dev/null 2>$OUT/s2.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval_mma -s 3 -c 1 -o /tmp/jpack $B > $OUT/n3.log 2>&1
python scripts/ncu_summary.py --tag r2g_jpack --rep /tmp/jpack.ncu-rep --key C4:hex8:jacobian_packed:stored --note "ncu --set full of eval_mma_kernel<Hex8> packed in: $B" > /dev/null 2>$OUT/s3.err
cp profiles/r2g_* $OUT/
bash scripts/gpu_abn.sh r2g_unroll "--config C4" cur build/libstokesfo_unroll2.so
bash scripts/gpu_abn.sh r2g_unroll_cmp "--config C4 --geometry compact" cur build/libstokesfo_unroll2.so
