#!/bin/bash
# Round-2 pass za: compute-sanitizer on the new paths -- the tcgen05 cluster-pair gridder and the banded grid
# (every family), small configs.
set -u
TAG=${1:-r02za}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; exit 1; }
S=$OUT/sanitizer_$TAG.txt; : > $S
for spec in "ska_small umma" "predict_small umma" "ska_small default" "lofar_small default" "small_dde simt" "small_dde8 tc"; do
  set -- $spec
  for tool in memcheck racecheck synccheck; do
    timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_run.py $1 $2 > $OUT/san_$1_$2_${tool}_$TAG.log 2>&1
    rc=$?
    echo "$1 $2 $tool rc=$rc $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize_run' $OUT/san_$1_$2_${tool}_$TAG.log | tr '\n' ' ')" | tee -a $S
  done
done
