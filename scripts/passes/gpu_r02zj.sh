#!/bin/bash
# Round-2 pass zj: the integer (m16n8k32 u8 x s8) degridder form -- parity of the default-kind degrid cases
# through it, then its launch shapes against the fixed-point f16 defaults on SKA / predict / LOFAR.
set -u
TAG=${1:-r02zj}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 1024 --which degridder --variants \
  'degridder_rot16s2<32,W8,minB2,U2,C32>' 'degridder_rot16i<32,W4,minB2,U2,C32>' 'degridder_rot16s2i<32,W4,minB2,U1,C32>' \
  'degridder_rot8i<32,W8,minB2,U2,C32>' 2>&1 | tee $OUT/sweep_i8_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config predict --timesteps 256 --which degridder --variants \
  'degridder_rot16s2<32,W8,minB2,U1,C16>' 'degridder_rot16i<32,W4,minB2,U2,C16>' 2>&1 | tee -a $OUT/sweep_i8_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config lofar --timesteps 8192 --which degridder --variants \
  'degridder_rot16<24,W4,minB3,U4,C16>' 'degridder_rot16i<24,W4,minB3,U4,C16>' 'degridder_rot16i<24,W4,minB2,U4,C16>' \
  'degridder_rot8i<24,W8,minB2,U2,C16>' 2>&1 | tee -a $OUT/sweep_i8_$TAG.txt
IDG_DEGRIDDER_VARIANT='degridder_rot16i<*' timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -s -k "degrid and default" > $OUT/pytest_i8_$TAG.log 2>&1; echo "pytest i8 rc=$?"
tail -2 $OUT/pytest_i8_$TAG.log
grep -oE "degrid\[[a-z0-9]+\][^:]*: rel rms [0-9.e-]+" $OUT/pytest_i8_$TAG.log | awk '{print $NF, $0}' | sort -g | tail -5
