#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_rot2.log 2>&1 || { echo BUILD FAILED; tail $OUT/build_rot2.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "rot16t" 2>&1 | tail -2
bash scripts/sweep_degridder2.sh "degridder_rot16<24,W4,minB3,U1,C16>" "degridder_rot16t<24,W4,minB3,U1,C16>" "degridder_rot16t<24,W8,minB2,U1,C16>"
CFG=ska TS=1024 bash scripts/sweep_degridder2.sh "degridder_rot16<32,W8,minB2,U1,C32>" "degridder_rot16t<32,W8,minB2,U1,C32>"
