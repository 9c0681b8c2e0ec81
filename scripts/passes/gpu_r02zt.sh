#!/bin/bash
# Round-2 pass zt: rotation gridders with E4 by sincos + lane-pair shuffle (3 sincos per lane, tile and
# timestep instead of 4) -- speed against the defaults, parity of each through the default-kind cases.
set -u
TAG=${1:-r02zt}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 600 python scripts/variant_sweep.py --config lofar --timesteps 8192 --which gridder --variants \
  'gridder_rot2<24,W12,MT3,minB2,KPT2>' 'gridder_rot2e<24,W12,MT3,minB2,KPT2>' 2>&1 | tee $OUT/sweep_e4s_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2h<32,W8,MT8,minB2,KPT4,GP4,r>' 'gridder_rot2he<32,W8,MT8,minB2,KPT4,GP4,r>' 2>&1 | tee -a $OUT/sweep_e4s_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config predict --timesteps 256 --which gridder --variants \
  'gridder_rot2<32,W8,MT8,minB2,KPT2,GP2,r>' 'gridder_rot2e<32,W8,MT8,minB2,KPT2,GP2,r>' 2>&1 | tee -a $OUT/sweep_e4s_$TAG.txt
for V in 'gridder_rot2e<24,W12,MT3,minB2,KPT2>' 'gridder_rot2he<32,W8,MT8,minB2,KPT4,GP4,r>' 'gridder_rot2e<32,W8,MT8,minB2,KPT2,GP2,r>'; do
  IDG_GRIDDER_VARIANT="$V" timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -s -k "grid_matches and default or full_l and grid and default" > $OUT/pytest_e4s_$TAG.log 2>&1; echo "pytest $V rc=$?"
  grep -oE "[^e]grid\[default\][^:]*: rel rms [0-9.e-]+" $OUT/pytest_e4s_$TAG.log | awk '{print $NF, $0}' | sort -g | tail -2
done
