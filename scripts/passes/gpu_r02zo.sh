#!/bin/bash
# Round-2 pass zo: fixed-point-split gridders at 8 warps x 8 tiles (16 warps/SM, 128 registers): speed + parity.
set -u
TAG=${1:-r02zo}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP4,lmnsm>' 'gridder_rot2hx<32,W8,MT8,minB2,KPT4,GP4,lmnsm>' \
  'gridder_rot2h<32,W8,MT8,minB2,KPT4,GP4,lmnsm>' 'gridder_rot2hx<32,W8,MT8,minB2,KPT4,GP2,lmnsm>' \
  'gridder_rot2hx<32,W8,MT8,minB2,KPT4,GP4,nsm>' 2>&1 | tee $OUT/sweep_gx8_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config predict --timesteps 256 --which gridder --variants \
  'gridder_rot2<32,W16,MT4,minB2,KPT2,GP2,lmnsm>' 'gridder_rot2x<32,W8,MT8,minB2,KPT2,GP2,lmnsm>' \
  'gridder_rot2<32,W8,MT8,minB2,KPT2,GP2,lmnsm>' 2>&1 | tee -a $OUT/sweep_gx8_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config lofar --timesteps 8192 --which gridder --variants \
  'gridder_rot2<24,W12,MT3,minB2,KPT2>' 'gridder_rot2x<24,W6,MT6,minB2,KPT2>' 2>&1 | tee -a $OUT/sweep_gx8_$TAG.txt
for V in 'gridder_rot2hx<32,W8,MT8,minB2,KPT4,GP4,lmnsm>' 'gridder_rot2x<32,W8,MT8,minB2,KPT2,GP2,lmnsm>' 'gridder_rot2x<24,W12,MT3,minB2,KPT2>'; do
  IDG_GRIDDER_VARIANT="$V" timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -s -k "grid_matches and default or full_l and grid and default" > $OUT/pytest_gx_$TAG.log 2>&1; echo "pytest $V rc=$?"
  grep -oE "grid\[default\][^:]*: rel rms [0-9.e-]+" $OUT/pytest_gx_$TAG.log | grep -v degrid | awk '{print $NF, $0}' | sort -g | tail -2
done
