#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_rot2.log 2>&1 || { echo BUILD FAILED; tail $OUT/build_rot2.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "rot2 or poly" 2>&1 | tail -3
bash scripts/sweep_degridder2.sh "degridder_tc<24,W8,MT2,minB4>" "degridder_tcp<24,W8,MT2,minB4,P1>" "degridder_tcp<24,W8,MT2,minB4,P2>" "degridder_tcp<24,W8,MT4,minB2,P1>" "degridder_tcp<24,W8,MT3,minB3,P1>"
CFG=ska TS=1024 bash scripts/sweep_gridder.sh "gridder_rot2<32,W16,MT4,minB2,KPT4,GP2>"
