#!/bin/bash
# ncu --set full (source-level) of the default gridder and degridder on a config: bash scripts/prof_kernels_src.sh TAG [CFG]
TAG=$1; CFG=${2:-lofar}
OUT=gpurun_out; mkdir -p $OUT
for K in gridder degridder; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
     -o $OUT/prof_${K}_$TAG -f python bench.py --config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_${K}_$TAG.log 2>&1
  echo "ncu $K rc=$?"
done
