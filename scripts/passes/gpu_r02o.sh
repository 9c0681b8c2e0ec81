#!/bin/bash
set -u
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_r02o.log 2>&1 || { echo BUILD FAILED; exit 1; }
python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP4,lmnsm>' 'gridder_rot2h<32,W16,MT4,minB1,KPT4,GP4,lmnsm>' \
  'gridder_rot2h<32,W32,MT2,minB1,KPT4,GP4,lmnsm>' 'gridder_rot2h<32,W16,MT4,minB1,KPT4,GP4,r>' 2>&1 | tee $OUT/sweep_ska_grd_r02o.txt
