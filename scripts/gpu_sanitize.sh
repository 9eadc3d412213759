#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_san.log 2>&1
for T in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $T --target-processes all --print-limit 20 python scripts/sanitize.py > $OUT/sanitize_$T.log 2>&1
  echo "$T exit $? : $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $OUT/sanitize_$T.log | tail -2 | tr '\n' ' ')" >> $OUT/sanitize_summary.txt
done
cat $OUT/sanitize_summary.txt
