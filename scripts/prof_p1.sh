set -u
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_p1.log 2>&1 || { echo BUILD FAILED; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_p1.json 2> $OUT/bench_p1.err; echo "bench rc=$?"
tail -c 1500 $OUT/bench_p1.json
timeout 900 ncu --set full --clock-control none --import-source on -k regex:^gridder_tc -s 1 -c 1 \
   -o $OUT/prof_gridder_p1 -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_g_p1.log 2>&1; echo "ncu g rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:^degridder_tc -s 1 -c 1 \
   -o $OUT/prof_degridder_p1 -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_d_p1.log 2>&1; echo "ncu d rc=$?"
ls -la $OUT
