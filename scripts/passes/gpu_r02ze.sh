#!/bin/bash
# Round-2 pass ze: the fixed-point split in the rotation gridders -- grid parity (all families), then the
# gridders against their f16-split forms on SKA / predict / LOFAR.
set -u
TAG=${1:-r02ze}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -s -k "grid_matches or full_l or channel_table or accum" > $OUT/pytest_grid_$TAG.log 2>&1; echo "pytest grid rc=$?"
tail -3 $OUT/pytest_grid_$TAG.log; grep -E "rel rms" $OUT/pytest_grid_$TAG.log | sort -k5 -g | tail -4
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2hf<32,W16,MT4,minB2,KPT4,GP4,lmnsm>' 'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP4,lmnsm>' 2>&1 | tee $OUT/sweep_gfx_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config lofar --timesteps 8192 --which gridder --variants \
  'gridder_rot2f<24,W12,MT3,minB2,KPT2>' 'gridder_rot2<24,W12,MT3,minB2,KPT2>' 2>&1 | tee -a $OUT/sweep_gfx_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config predict --timesteps 256 --which gridder --variants \
  'gridder_rot2<32,W16,MT4,minB2,KPT2,GP2,lmnsm>' 2>&1 | tee -a $OUT/sweep_gfx_$TAG.txt
