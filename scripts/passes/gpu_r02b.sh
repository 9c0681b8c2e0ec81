#!/bin/bash
# Round-2 bench validation: the default (SKA, full T) bench line, then predict and LOFAR lines.
set -u
TAG=${1:-r02b}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
timeout 1200 python bench.py --steps 10 --warmup 3 > $OUT/bench_ska_$TAG.json 2> $OUT/bench_ska_$TAG.err; echo "bench ska rc=$?"
tail -c 2500 $OUT/bench_ska_$TAG.json; tail -5 $OUT/bench_ska_$TAG.err
timeout 900 python bench.py --config predict --steps 10 --warmup 3 --no-rho-sweep > $OUT/bench_predict_$TAG.json 2> $OUT/bench_predict_$TAG.err; echo "bench predict rc=$?"
tail -c 1500 $OUT/bench_predict_$TAG.json; tail -5 $OUT/bench_predict_$TAG.err
timeout 900 python bench.py --config lofar --steps 10 --warmup 3 --no-rho-sweep > $OUT/bench_lofar_$TAG.json 2> $OUT/bench_lofar_$TAG.err; echo "bench lofar rc=$?"
tail -c 1500 $OUT/bench_lofar_$TAG.json; tail -5 $OUT/bench_lofar_$TAG.err
