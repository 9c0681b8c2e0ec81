#!/bin/bash
# Round-2 pass zb: N~ = 32 degridder launch shapes with 80 registers (12 warps x 2 CTAs = 24 warps / SM).
set -u
TAG=${1:-r02zb}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 900 python scripts/variant_sweep.py --config ska --timesteps 1024 --which degridder --variants \
  'degridder_rot16s2<32,W8,minB2,U1,C32>' 'degridder_rot16s2<32,W12,minB2,U1,C32>' 'degridder_rot16s2<32,W16,minB1,U1,C32>' 2>&1 | tee $OUT/sweep_deg_$TAG.txt
timeout 900 python scripts/variant_sweep.py --config predict --timesteps 256 --which degridder --variants \
  'degridder_rot16s2<32,W8,minB2,U1,C16>' 'degridder_rot16s2<32,W12,minB2,U1,C16>' 2>&1 | tee -a $OUT/sweep_deg_$TAG.txt
IDG_DEGRIDDER_VARIANT='degridder_rot16s2<32,W12,minB2,U1,C32>' timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "ska and default" > $OUT/pytest_deg12_$TAG.log 2>&1; echo "parity W12 C32 rc=$?"; tail -1 $OUT/pytest_deg12_$TAG.log
