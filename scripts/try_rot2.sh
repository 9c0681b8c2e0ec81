#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_rot2.log 2>&1 || { echo BUILD FAILED; tail $OUT/build_rot2.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "default or rot" 2>&1 | tail -3
bash scripts/sweep_degridder2.sh "degridder_tc<24,W8,MT2,minB4>" "degridder_rot<24,W8,minB4,U1,C16>" "degridder_rot<24,W8,minB3,U1,C16>"
CFG=predict TS=256 bash scripts/sweep_degridder2.sh "degridder_tc<32,W8,MT4,minB2>" "degridder_rot<32,W16,minB1,U2,C16>"
