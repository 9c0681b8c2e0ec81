#!/bin/bash
# Round-end records (tag $1): LOFAR bench + reference arm, launch list, ncu of the default kernels, SKA /
# predict bench lines, ncu of the SKA-shaped kernels at T = 1024 (summarised on the box; the large
# reports are deleted so gpurun_out/ stays under the copy-back limit).  GPU suite + smoke: final_pass.sh.
TAG=${1:-final}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; exit 1; }
if [ "${SUITE:-0}" = "1" ]; then
  timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest gpu rc=$?"; tail -1 $OUT/pytest_gpu_$TAG.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke_$TAG.log
fi
timeout 900 python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference > $OUT/bench_ref_$TAG.json 2> $OUT/bench_ref_$TAG.err; echo "reference rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$TAG.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu launches rc=$?"
for K in gridder degridder; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
      -o $OUT/prof_${K}_$TAG -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_${K}_$TAG.log 2>&1
  echo "ncu $K rc=$?"
done
bash scripts/bench_configs.sh $TAG
for K in gridder degridder; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^${K}_ -s 1 -c 1 \
      -o $OUT/prof_ska_${K}_$TAG -f python bench.py --config ska --timesteps 1024 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > $OUT/ncu_ska_${K}_$TAG.log 2>&1
  echo "ncu ska $K rc=$?"
done
python scripts/ncu_summary.py --tag ${TAG}_ska --config "ska (T=1024)" $OUT/prof_ska_gridder_$TAG.ncu-rep $OUT/prof_ska_degridder_$TAG.ncu-rep > /dev/null 2>&1
cp profiles/${TAG}_ska_ncu_summary.md $OUT/ 2>/dev/null
rm -f $OUT/prof_ska_*_$TAG.ncu-rep
du -sh $OUT
