#!/bin/bash
# Round-2 pass zg: ncu --set full of the fixed-point-split SKA degridder (T = 256 sample, one launch).
set -u
TAG=${1:-r02zg}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 256 --which degridder --reps 1 --warmup 0 --variants \
  'degridder_rot16s2<32,W8,minB2,U1,C32>' > /dev/null 2>&1; echo "plain rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:degridder -c 1 -o $OUT/ska_degrid_fx_$TAG -f \
  python scripts/variant_sweep.py --config ska --timesteps 256 --which degridder --reps 1 --warmup 0 --variants \
  'degridder_rot16s2<32,W8,minB2,U1,C32>' > $OUT/ncu_$TAG.log 2>&1; echo "ncu rc=$?"
