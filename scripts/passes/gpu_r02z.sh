#!/bin/bash
# Round-2 pass z: the banded grid (multi-rank exchange fused into the kernels over CUDA-IPC peer memory):
# single-process bands for every family, two / three processes on one GPU, the two-rank bench both ways.
set -u
TAG=${1:-r02z}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_bands.py -q -s -x > $OUT/pytest_bands_$TAG.log 2>&1; echo "pytest bands rc=$?"
grep -E "grid_bands|banded|passed|failed|Error|error" $OUT/pytest_bands_$TAG.log | tail -24
timeout 1500 python -m pytest tests/test_gpu_multirank.py -q -x > $OUT/pytest_multirank_$TAG.log 2>&1; echo "pytest multirank rc=$?"
tail -3 $OUT/pytest_multirank_$TAG.log
