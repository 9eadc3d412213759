#!/bin/bash
# Quick GPU pass: selected parity tests + same-box interleaved A/B of the in-tree build vs other builds.
# Usage (under gpurun): bash scripts/gpu_abq.sh TAG "pytest -k expr" "bench args;bench args;..." LIB...
TAG=$1; KEXPR=$2; ARGSETS=$3; shift 3
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
if [ -n "$KEXPR" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "$KEXPR" > $OUT/pytest_$TAG.log 2>&1
  echo "pytest: $(tail -1 $OUT/pytest_$TAG.log)"
fi
IFS=';' read -ra SETS <<< "$ARGSETS"
for A in "${SETS[@]}"; do
  bash scripts/gpu_abn.sh $TAG "$A --sustain 0" cur "$@" > /dev/null
done
cat $OUT/samebox_$TAG.txt
