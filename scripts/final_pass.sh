#!/bin/bash
# Consolidated GPU pass: full GPU suite, smoke, bench (ours + reference arm), launch list, ncu of defaults.
TAG=${1:-final}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; exit 1; }
start=$(date +%s)
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest gpu rc=$? in $(( $(date +%s) - start ))s"
tail -2 $OUT/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke_$TAG.log
start=$(date +%s)
timeout 900 python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench rc=$? in $(( $(date +%s) - start ))s"
start=$(date +%s)
timeout 900 python bench.py --impl reference > $OUT/bench_ref_$TAG.json 2> $OUT/bench_ref_$TAG.err; echo "reference rc=$? in $(( $(date +%s) - start ))s"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$TAG.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu launches rc=$?"
for K in gridder degridder; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
      -o $OUT/prof_${K}_$TAG -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_${K}_$TAG.log 2>&1
  echo "ncu $K rc=$?"
done
