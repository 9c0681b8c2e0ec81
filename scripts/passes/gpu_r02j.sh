#!/bin/bash
# Round-2 pass j: Horner-form group rotation in the gridder.
set -u
TAG=${1:-r02j}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2<32,W16,MT4,minB2,KPT4,GP2,nsm>' 'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP2,nsm>' \
  'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP4,nsm>' 'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP1,nsm>' 2>&1 | tee $OUT/sweep_ska_grd_$TAG.txt
python scripts/variant_sweep.py --config ska --timesteps 8192 --which gridder --reps 3 --variants \
  'gridder_rot2<32,W16,MT4,minB2,KPT4,GP2,nsm>' 'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP2,nsm>' 2>&1 | tee -a $OUT/sweep_ska_grd_$TAG.txt
