#!/bin/bash
# Round-2 pass zn: the fixed-point split in the rotation gridders at 16 warps / 128 registers (no spills).
set -u
TAG=${1:-r02zn}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP4,lmnsm>' 'gridder_rot2hx<32,W16,MT4,minB1,KPT4,GP4,lmnsm>' \
  'gridder_rot2hx<32,W16,MT4,minB2,KPT4,GP4,lmnsm>' 'gridder_rot2hx<32,W8,MT8,minB2,KPT4,GP4,lmnsm>' \
  'gridder_rot2h<32,W16,MT4,minB1,KPT4,GP4,lmnsm>' 2>&1 | tee $OUT/sweep_gx_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config lofar --timesteps 8192 --which gridder --variants \
  'gridder_rot2<24,W12,MT3,minB2,KPT2>' 'gridder_rot2x<24,W12,MT3,minB2,KPT2>' 'gridder_rot2x<24,W12,MT3,minB1,KPT2>' \
  2>&1 | tee -a $OUT/sweep_gx_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config predict --timesteps 256 --which gridder --variants \
  'gridder_rot2<32,W16,MT4,minB2,KPT2,GP2,lmnsm>' 'gridder_rot2x<32,W16,MT4,minB1,KPT2,GP2,lmnsm>' 2>&1 | tee -a $OUT/sweep_gx_$TAG.txt
IDG_GRIDDER_VARIANT='gridder_rot2*x<*' timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -s -k "grid_matches and default or full_l and default" > $OUT/pytest_gx_$TAG.log 2>&1; echo "pytest gx rc=$?"
tail -2 $OUT/pytest_gx_$TAG.log
grep -oE "grid\[[a-z0-9]+\][^:]*: rel rms [0-9.e-]+" $OUT/pytest_gx_$TAG.log | awk '{print $NF, $0}' | sort -g | tail -4
