#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_rot2.log 2>&1 || { echo BUILD FAILED; tail $OUT/build_rot2.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "default or rot" 2>&1 | tail -2
CFG=predict TS=256 bash scripts/sweep_gridder.sh "gridder_rot2<32,W16,MT4,minB2,KPT2>" "gridder_rot2<32,W16,MT4,minB1,KPT2>" "gridder_rot2<32,W32,MT2,minB1,KPT2>"
