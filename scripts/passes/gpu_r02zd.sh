#!/bin/bash
# Round-2 pass zd: the fixed-point (byte-permutation) A-operand split in the rotation degridders --
# degridder parity, then the new defaults against the f16-split kernels on SKA / predict / LOFAR.
set -u
TAG=${1:-r02zd}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "degrid" > $OUT/pytest_degrid_$TAG.log 2>&1; echo "pytest degrid rc=$?"
tail -3 $OUT/pytest_degrid_$TAG.log
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 1024 --which degridder --variants \
  'degridder_rot16s2f<32,W8,minB2,U1,C32>' 'degridder_rot16s2<32,W8,minB2,U1,C32>' 2>&1 | tee $OUT/sweep_fx_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config predict --timesteps 256 --which degridder --variants \
  'degridder_rot16s2<32,W8,minB2,U1,C16>' 2>&1 | tee -a $OUT/sweep_fx_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config lofar --timesteps 8192 --which degridder --variants \
  'degridder_rot16f<24,W4,minB3,U4,C16>' 'degridder_rot16<24,W4,minB3,U4,C16>' 2>&1 | tee -a $OUT/sweep_fx_$TAG.txt
