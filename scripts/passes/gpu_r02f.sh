#!/bin/bash
# Round-2 pass f: packed-rotation gridder variants (LOFAR, SKA T=1024, predict T=256, lofar_short).
set -u
TAG=${1:-r02f}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
python scripts/variant_sweep.py --config lofar --timesteps 8192 --which gridder --variants \
  'gridder_rot2<24,W12,MT3,minB2,KPT2>' 'gridder_rot2p<24,W12,MT3,minB2,KPT2,GP2,r>' 2>&1 | tee $OUT/sweep_lofar_grd_$TAG.txt
python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2<32,W16,MT4,minB2,KPT4,GP2,nsm>' 'gridder_rot2p<32,W16,MT4,minB2,KPT4,GP2,nsm>' \
  'gridder_rot2p<32,W16,MT4,minB2,KPT4,GP4,nsm>' 'gridder_rot2p<32,W32,MT2,minB1,KPT4,GP2,nsm>' \
  'gridder_rot2p<32,W32,MT2,minB1,KPT4,GP4,r>' 2>&1 | tee $OUT/sweep_ska_grd_$TAG.txt
python scripts/variant_sweep.py --config predict --timesteps 256 --which gridder --variants \
  'gridder_rot2<32,W16,MT4,minB2,KPT2,GP2,lmnsm>' 'gridder_rot2p<32,W16,MT4,minB2,KPT2,GP2,lmnsm>' 2>&1 | tee $OUT/sweep_predict_grd_$TAG.txt
python scripts/variant_sweep.py --config lofar_short --timesteps 8192 --which gridder --variants \
  'gridder_rot2<24,W12,MT3,minB2,KPT2>' 'gridder_rot2p<24,W12,MT3,minB2,KPT2,GP2,r>' 2>&1 | tee $OUT/sweep_lshort_grd_$TAG.txt
