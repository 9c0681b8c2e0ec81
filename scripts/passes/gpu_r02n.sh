#!/bin/bash
# What does ncu's tensor / shared pipe utilisation read when HMMA.16816 is saturated (pipe_probe.cu)?
set -u
OUT=gpurun_out; mkdir -p $OUT
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pipe_probe scripts/pipe_probe.cu && /tmp/pipe_probe | tee $OUT/pipe_probe_r02n.txt
timeout 600 ncu --metrics sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_tensor_subpipe_hmma.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active,smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio --csv /tmp/pipe_probe > $OUT/pipe_probe_ncu_r02n.csv 2>&1; echo "ncu rc=$?"
