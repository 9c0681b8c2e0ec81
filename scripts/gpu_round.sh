#!/bin/bash
# One GPU pass: build, GPU tests, smoke, bench, ncu launch list + full capture of the top kernels.
# Usage (from the repo root, on a gpurun box): bash scripts/gpu_round.sh [tag]
set -u
TAG=${1:-r01}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/gpu_$TAG.txt 2>&1
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q -s > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest gpu rc=$?"
tail -5 $OUT/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"
tail -2 $OUT/smoke_$TAG.log
timeout 900 python bench.py --steps 10 --warmup 3 --rho-sweep > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench rc=$?"
tail -c 3000 $OUT/bench_$TAG.json; tail -5 $OUT/bench_$TAG.err
if [ "${NCU:-1}" = "1" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$TAG.csv \
      python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu launches rc=$?"
  for K in gridder degridder; do
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_kernel -s 1 -c 1 \
        -o $OUT/prof_${K}_$TAG -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_${K}_$TAG.log 2>&1
    echo "ncu $K rc=$?"
  done
fi
