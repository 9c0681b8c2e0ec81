#!/bin/bash
# Round-2 pass zu: the integer form of the direct degridder (any channel table): shapes and parity.
set -u
TAG=${1:-r02zu}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 600 python scripts/variant_sweep.py --config lofar --timesteps 2048 --which degridder --variants \
  'degridder_tc<24,W8,MT2,minB4>' 'degridder_tci<24,W8,MT2,minB3>' 'degridder_tci<24,W8,MT2,minB2>' 'degridder_tci<24,W8,MT4,minB2>' \
  2>&1 | tee $OUT/sweep_tci_$TAG.txt
timeout 600 python scripts/variant_sweep.py --config ska --timesteps 256 --which degridder --variants \
  'degridder_tc<32,W8,MT4,minB2>' 'degridder_tci<32,W8,MT4,minB1>' 'degridder_tci<32,W8,MT2,minB2>' 'degridder_tci<32,W4,MT4,minB2>' \
  2>&1 | tee -a $OUT/sweep_tci_$TAG.txt
IDG_DEGRIDDER_VARIANT='degridder_tci<*' timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -s -k "degrid and default or channel_table or amplitude and default" > $OUT/pytest_tci_$TAG.log 2>&1; echo "pytest tci rc=$?"
tail -2 $OUT/pytest_tci_$TAG.log
grep -oE "degrid\[default\][^:]*: rel rms [0-9.e-]+|channel[^:]*: [^,]*rel rms [0-9.e-]+" $OUT/pytest_tci_$TAG.log | awk '{print $NF, $0}' | sort -g | tail -5
