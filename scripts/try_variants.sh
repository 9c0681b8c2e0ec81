#!/bin/bash
# ad-hoc variant sweep (edit the lists): bash scripts/try_variants.sh
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_try.log 2>&1 || { echo BUILD FAILED; tail $OUT/build_try.log; exit 1; }
CFG=ska TS=1024 bash scripts/sweep_gridder.sh "gridder_rot2<32,W16,MT4,minB2,KPT4,GP2,nsm>" "gridder_rot2<32,W16,MT4,minB2,KPT4,GP2,lmnsm>" "gridder_rot2<32,W16,MT4,minB2,KPT4,GP4,lmnsm>"
CFG=predict TS=256 bash scripts/sweep_gridder.sh "gridder_rot2<32,W16,MT4,minB2,KPT2,GP2,nsm>" "gridder_rot2<32,W16,MT4,minB2,KPT2,GP2,lmnsm>"
bash scripts/sweep_gridder.sh "gridder_rot2<24,W12,MT3,minB2,KPT2>" "gridder_rot2<24,W12,MT3,minB2,KPT2,GP2,lmnsm>"
