#!/bin/bash
# Round-2 pass t+: tcgen05 rotation gridder iterations (parity, SKA/predict sweep, ncu).
set -u
TAG=${1:-r02t}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -q -s -k "umma" -x > $OUT/pytest_umma_$TAG.log 2>&1; echo "pytest umma rc=$?"
grep -E "grid\[umma\]|passed|failed|Error|error" $OUT/pytest_umma_$TAG.log | tail -12
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2h<32,W16,MT4,minB2,KPT4,GP4,lmnsm>' 'gridder_umma_rot<32,KPT4>' 2>&1 | tee $OUT/sweep_umma_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config predict --timesteps 256 --which gridder --variants \
  'gridder_rot2<32,W16,MT4,minB2,KPT2,GP2,lmnsm>' 'gridder_umma_rot<32,KPT2>' 2>&1 | tee -a $OUT/sweep_umma_$TAG.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:umma -s 1 -c 1 -o $OUT/prof_ska_umma_$TAG -f \
  python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --reps 1 --warmup 1 \
  --variants 'gridder_umma_rot<32,KPT4>' > $OUT/ncu_umma_$TAG.log 2>&1; echo "ncu rc=$?"
