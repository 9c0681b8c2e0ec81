#!/bin/bash
# Round-2 pass e: GPU tests, short-item workload, LOFAR ncu (pipes), SKA launch list, imaging cycle.
set -u
TAG=${1:-r02e}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q -s > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest gpu rc=$?"
grep -E "host adder|passed|failed|Error" $OUT/pytest_gpu_$TAG.log | tail -12
timeout 900 python bench.py --config lofar_short --steps 10 --warmup 3 --no-rho-sweep --no-cpu-baseline --no-e2e > $OUT/bench_lofar_short_$TAG.json 2> $OUT/bench_lofar_short_$TAG.err; echo "bench lofar_short rc=$?"
python -c "import json;d=json.loads(open('$OUT/bench_lofar_short_$TAG.json').read().splitlines()[-1]);print('lofar_short',d['value'],d['grid_mvis_s'],d['degrid_mvis_s'],d['config']['items_timesteps'],d['imaging_cycle']['share'] if d['imaging_cycle'] else None)"
timeout 900 python bench.py --config lofar --steps 10 --warmup 3 --no-rho-sweep --no-cpu-baseline --no-e2e > $OUT/bench_lofar_$TAG.json 2> $OUT/bench_lofar_$TAG.err; echo "bench lofar rc=$?"
python -c "import json;d=json.loads(open('$OUT/bench_lofar_$TAG.json').read().splitlines()[-1]);print('lofar',d['value'],d['grid_mvis_s'],d['degrid_mvis_s'],d['imaging_cycle'])"
for K in gridder degridder; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
      -o $OUT/prof_lofar_${K}_$TAG -f python bench.py --config lofar --steps 1 --warmup 3 --no-e2e --no-cpu-baseline \
      --no-rho-sweep --no-kernel-energy --no-imaging-cycle > $OUT/ncu_lofar_${K}_$TAG.log 2>&1
  echo "ncu lofar $K rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
      -o $OUT/prof_lofar_short_${K}_$TAG -f python bench.py --config lofar_short --steps 1 --warmup 3 --no-e2e \
      --no-cpu-baseline --no-rho-sweep --no-kernel-energy --no-imaging-cycle > $OUT/ncu_lofar_short_${K}_$TAG.log 2>&1
  echo "ncu lofar_short $K rc=$?"
done
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_ska_$TAG.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-rho-sweep --no-kernel-energy --no-imaging-cycle \
    > $OUT/bench_ska_under_ncu_$TAG.json 2>&1; echo "ncu ska launches rc=$?"
