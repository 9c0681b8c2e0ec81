#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_rot2.log 2>&1 || { echo BUILD FAILED; tail $OUT/build_rot2.log; exit 1; }
bash scripts/sweep_degridder2.sh "degridder_rot<24,W8,minB4,U1,C16>" "degridder_rot<24,W8,minB4,U2,C16>" "degridder_rot<24,W8,minB4,U3,C16>" "degridder_rot<24,W16,minB2,U1,C16>" "degridder_rot<24,W4,minB6,U1,C16>"
bash scripts/sweep_gridder.sh "gridder_rot2<24,W12,MT3,minB2,KPT2,KB64>" "gridder_rot2<24,W12,MT3,minB2,KPT2,KB256>" "gridder_rot2<24,W6,MT6,minB3,KPT2,KB64>" "gridder_rot2<24,W6,MT6,minB2,KPT2>" "gridder_rot2<24,W18,MT2,minB1,KPT2>"
