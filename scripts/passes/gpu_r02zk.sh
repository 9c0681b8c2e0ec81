#!/bin/bash
# Round-2 pass zk: launch shapes of the integer-form degridder (SKA / predict / LOFAR / lofar_short).
set -u
TAG=${1:-r02zk}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 1024 --which degridder --variants \
  'degridder_rot16i<32,W4,minB2,U2,C32>' 'degridder_rot16i<32,W4,minB2,U1,C32>' 'degridder_rot16i<32,W4,minB2,U4,C32>' \
  'degridder_rot16i<32,W6,minB2,U2,C32>' 'degridder_rot16i<32,W8,minB1,U2,C32>' 2>&1 | tee $OUT/sweep_i8shapes_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config predict --timesteps 256 --which degridder --variants \
  'degridder_rot16i<32,W4,minB2,U2,C16>' 'degridder_rot16i<32,W4,minB2,U1,C16>' 2>&1 | tee -a $OUT/sweep_i8shapes_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config lofar --timesteps 8192 --which degridder --variants \
  'degridder_rot16i<24,W4,minB3,U4,C16>' 'degridder_rot16i<24,W4,minB3,U2,C16>' 'degridder_rot16i<24,W6,minB2,U4,C16>' \
  'degridder_rot16i<24,W4,minB4,U4,C16>' 2>&1 | tee -a $OUT/sweep_i8shapes_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config lofar_short --timesteps 8192 --which degridder --variants \
  'degridder_rot8<24,W4,minB3,U2,C16>' 'degridder_rot16i<24,W4,minB3,U4,C16>' 'degridder_rot8i<24,W8,minB2,U2,C16>' 2>&1 | tee -a $OUT/sweep_i8shapes_$TAG.txt
