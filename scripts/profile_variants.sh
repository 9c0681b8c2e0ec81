#!/bin/bash
# ncu --set full of named kernel variants on the LOFAR config (one capture each).
# usage: bash scripts/profile_variants.sh TAG "gridder:NAME" "degridder:NAME" ...
TAG=$1; shift
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || exit 1
i=0
for spec in "$@"; do
  K=${spec%%:*}; V=${spec#*:}
  if [ "$K" = "gridder" ]; then ENV="IDG_GRIDDER_VARIANT=$V"; else ENV="IDG_DEGRIDDER_VARIANT=$V"; fi
  env $ENV timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
      -o $OUT/prof_${TAG}_$i -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_${TAG}_$i.log 2>&1
  echo "ncu $K $V -> prof_${TAG}_$i rc=$?"
  i=$((i+1))
done
