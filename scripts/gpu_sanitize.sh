#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on small configs for every kernel family.
set -u
TAG=${1:-r02}
OUT=gpurun_out; mkdir -p $OUT
S=$OUT/sanitizer_$TAG.txt; : > $S
for cfg in ${CONFIGS:-tiny small_dde lofar_small ska_small small_dde8 short_items}; do
  for fam in default tc simt; do
    for tool in memcheck racecheck synccheck; do
      timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_run.py $cfg $fam > $OUT/san_${cfg}_${fam}_${tool}.log 2>&1
      rc=$?
      echo "$cfg $fam $tool rc=$rc $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize_run' $OUT/san_${cfg}_${fam}_${tool}.log | tr '\n' ' ')" | tee -a $S
    done
  done
done
