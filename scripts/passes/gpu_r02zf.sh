#!/bin/bash
# Round-2 pass zf: launch shapes of the fixed-point-split degridders (fewer registers than the f16 split).
set -u
TAG=${1:-r02zf}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 600 python scripts/variant_sweep.py --config lofar --timesteps 8192 --which degridder --variants \
  'degridder_rot16<24,W4,minB3,U4,C16>' 'degridder_rot16<24,W4,minB4,U4,C16>' 'degridder_rot16<24,W8,minB2,U4,C16>' \
  'degridder_rot16<24,W4,minB4,U2,C16>' 2>&1 | tee $OUT/sweep_shapes_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 1024 --which degridder --variants \
  'degridder_rot16s2<32,W8,minB2,U1,C32>' 'degridder_rot16s2<32,W8,minB2,U2,C32>' 'degridder_rot16s2<32,W4,minB4,U1,C32>' \
  2>&1 | tee -a $OUT/sweep_shapes_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config predict --timesteps 256 --which degridder --variants \
  'degridder_rot16s2<32,W8,minB2,U1,C16>' 'degridder_rot16s2<32,W8,minB2,U2,C16>' 2>&1 | tee -a $OUT/sweep_shapes_$TAG.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -s -k "degrid" > $OUT/pytest_degrid_$TAG.log 2>&1; echo "pytest degrid rc=$?"
tail -2 $OUT/pytest_degrid_$TAG.log
grep -oE "degrid\[[a-z0-9]+\][^:]*: rel rms [0-9.e-]+" $OUT/pytest_degrid_$TAG.log | awk '{print $NF, $0}' | sort -g | tail -4
