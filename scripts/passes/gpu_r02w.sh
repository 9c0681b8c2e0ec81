#!/bin/bash
# Round-2 pass w: cluster-pair tcgen05 gridder, batch length / wait back-off sweep (SKA-T1024).
set -u
TAG=${1:-r02w}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 900 python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP4,lmnsm>' 'gridder_umma_rot<32,KPT4,pair>' \
  'gridder_umma_rot<32,KPT4,pair,T5,S0>' 'gridder_umma_rot<32,KPT4,pair,T4,S32>' 'gridder_umma_rot<32,KPT4,pair,T5,S32>' \
  'gridder_umma_rot<32,KPT4,pair,T5,S100>' 'gridder_umma_rot<32,KPT4,pair,T5,S20>' 2>&1 | tee $OUT/sweep_umma_$TAG.txt
