#!/bin/bash
set -u
TAG=${1:-r02l}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP4,nsm>' 'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP4,lmnsm>' \
  'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP2,r>' 2>&1 | tee $OUT/sweep_ska_grd_$TAG.txt
python scripts/variant_sweep.py --config predict --timesteps 256 --which gridder --variants \
  'gridder_rot2<32,W16,MT4,minB2,KPT2,GP2,lmnsm>' 'gridder_rot2h<32,W16,MT4,minB2,KPT2,GP2,lmnsm>' 2>&1 | tee $OUT/sweep_predict_grd_$TAG.txt
