#!/bin/bash
# Round-2 pass h: the default bench line (SKA), LOFAR-DDE, ncu of the SKA default kernels.
set -u
TAG=${1:-r02h}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap --format=csv -lms 500 > $OUT/clocks_$TAG.csv &
SMI=$!
timeout 1500 python bench.py --steps 20 --warmup 5 > $OUT/bench_ska_$TAG.json 2> $OUT/bench_ska_$TAG.err; echo "bench ska rc=$?"
kill $SMI
python -c "import json;d=json.loads(open('$OUT/bench_ska_$TAG.json').read().splitlines()[-1]);print('ska',d['value'],d['grid_mvis_s'],d['degrid_mvis_s'],d['e2e'],d['imaging_cycle'],d['clocks'])"
timeout 900 python bench.py --config lofar_dde --steps 10 --warmup 3 --no-rho-sweep --no-cpu-baseline > $OUT/bench_lofar_dde_$TAG.json 2> $OUT/bench_lofar_dde_$TAG.err; echo "bench lofar_dde rc=$?"
python -c "import json;d=json.loads(open('$OUT/bench_lofar_dde_$TAG.json').read().splitlines()[-1]);print('lofar_dde',d['value'],d['grid_mvis_s'],d['degrid_mvis_s'],d['e2e']['value'])"
for K in gridder degridder; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
      -o $OUT/prof_ska_${K}_$TAG -f python bench.py --config ska --timesteps 1024 --steps 1 --warmup 3 --no-e2e \
      --no-cpu-baseline --no-rho-sweep --no-kernel-energy --no-imaging-cycle > $OUT/ncu_ska_${K}_$TAG.log 2>&1
  echo "ncu ska $K rc=$?"
done
