#!/bin/bash
# Round-2 pass k: GPU tests + smoke + SKA default bench + lofar_short (new defaults: Horner N~=32 gridder,
# short-item degridder).
set -u
TAG=${1:-r02k}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q -s > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest gpu rc=$?"
grep -E "short items|passed|failed|Error" $OUT/pytest_gpu_$TAG.log | tail -8
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"
timeout 1500 python bench.py --steps 20 --warmup 5 > $OUT/bench_ska_$TAG.json 2> $OUT/bench_ska_$TAG.err; echo "bench ska rc=$?"
python -c "import json;d=json.loads(open('$OUT/bench_ska_$TAG.json').read().splitlines()[-1]);print('ska',d['value'],d['grid_mvis_s'],d['degrid_mvis_s'],d['e2e']['value'],d['roofline']['frac'],d['clocks'])"
timeout 900 python bench.py --config lofar_short --steps 10 --warmup 3 --no-rho-sweep --no-cpu-baseline --no-e2e > $OUT/bench_lofar_short_$TAG.json 2> $OUT/bench_lofar_short_$TAG.err; echo "bench lofar_short rc=$?"
python -c "import json;d=json.loads(open('$OUT/bench_lofar_short_$TAG.json').read().splitlines()[-1]);print('lofar_short',d['value'],d['grid_mvis_s'],d['degrid_mvis_s'],d['kernels']['degridder']['variant'])"
