#!/bin/bash
# ad-hoc variant sweep (edit the lists): bash scripts/try_variants.sh
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_try.log 2>&1 || { echo BUILD FAILED; tail $OUT/build_try.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "default" 2>&1 | tail -2
bash scripts/sweep_degridder2.sh "degridder_rot16<24,W4,minB3,U4,C16>" "degridder_rot16<24,W4,minB3,U6,C16>" "degridder_rot16<24,W4,minB3,U8,C16>"
CFG=ska TS=1024 bash scripts/sweep_degridder2.sh "degridder_rot16<32,W8,minB2,U8,C32>"
