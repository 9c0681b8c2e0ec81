#!/bin/bash
# bench records for the SKA-shaped and predict-shaped configs (tag $1)
TAG=${1:-x}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; exit 1; }
for C in ska predict; do
  start=$(date +%s)
  timeout 1200 python bench.py --config $C --steps 3 --warmup 3 > $OUT/bench_${C}_$TAG.json 2> $OUT/bench_${C}_$TAG.err
  echo "$C rc=$? in $(( $(date +%s) - start ))s"
  python -c "import json; d=json.load(open('$OUT/bench_${C}_$TAG.json')); k=d['kernels']; print(d['value'], d['grid_mvis_s'], d['degrid_mvis_s'], k['gridder']['variant'], k['gridder']['avg_ms'], k['degridder']['variant'], k['degridder']['avg_ms'], d['clocks'])"
done
