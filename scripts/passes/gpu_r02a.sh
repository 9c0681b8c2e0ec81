#!/bin/bash
# Round-2 first pass: box facts, GPU tests, smoke, ncu full captures of the SKA (N~=32) kernels.
set -u
TAG=${1:-r02a}
OUT=gpurun_out; mkdir -p $OUT
{ nvidia-smi; free -g; nproc; df -h /dev/shm /tmp; } > $OUT/box_$TAG.txt 2>&1
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q -s -p no:randomly > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest gpu rc=$?"
grep -E "rel rms|passed|failed|Error" $OUT/pytest_gpu_$TAG.log | tail -60
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"
tail -2 $OUT/smoke_$TAG.log
for K in gridder degridder; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
      -o $OUT/prof_ska_${K}_$TAG -f python bench.py --config ska --timesteps 1024 --steps 1 --warmup 3 --no-e2e \
      --no-cpu-baseline > $OUT/ncu_ska_${K}_$TAG.log 2>&1
  echo "ncu ska $K rc=$?"
done
