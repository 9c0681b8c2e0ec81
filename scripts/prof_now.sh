#!/bin/bash
# ncu full capture of the current default gridder / degridder on the LOFAR bench (tag $1)
TAG=${1:-now}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; exit 1; }
for K in gridder degridder; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
      -o $OUT/prof_${K}_$TAG -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_${K}_$TAG.log 2>&1
  echo "ncu $K rc=$?"
done
