#!/bin/bash
# ncu captures of the hot kernels (run on a gpurun box): full sets + launch list.
TAG=${1:-r03}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || exit 1
for K in gridder degridder; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
      -o $OUT/prof_${K}_$TAG -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_${K}_$TAG.log 2>&1
  echo "ncu $K rc=$?"
done
timeout 300 ncu --set full --clock-control none -k regex:rho_kernel -c 1 -o $OUT/prof_rho_$TAG -f \
    python -c "import paper_conf_ipps_veenboerpr17_b200 as i; print(i.rho_benchmark(17, 1024))" > $OUT/ncu_rho_$TAG.log 2>&1
echo "ncu rho rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$TAG.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu launches rc=$?"
