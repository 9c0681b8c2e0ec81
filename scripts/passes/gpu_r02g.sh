#!/bin/bash
# Round-2 pass g: tcgen05 rotation-gridder loop probe vs the mma.sync rotation loop probe.
set -u
OUT=gpurun_out; mkdir -p $OUT
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/umma_rot scripts/umma_rot_probe.cu && timeout 300 /tmp/umma_rot 2>&1 | tee $OUT/umma_rot_probe_r02g.txt
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/rot_probe scripts/rot_probe.cu && timeout 300 /tmp/rot_probe 2>&1 | tee $OUT/rot_probe_r02g.txt
