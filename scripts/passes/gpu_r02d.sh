#!/bin/bash
# Round-2 pass d: GPU tests (incl. host adder / splitter), smoke, SKA bench with the new N~=32 degridder default.
set -u
TAG=${1:-r02d}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q -s > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest gpu rc=$?"
grep -E "host adder|passed|failed|Error|error" $OUT/pytest_gpu_$TAG.log | tail -20
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"
timeout 1200 python bench.py --steps 10 --warmup 3 > $OUT/bench_ska_$TAG.json 2> $OUT/bench_ska_$TAG.err; echo "bench ska rc=$?"
python -c "import json;d=json.loads(open('$OUT/bench_ska_$TAG.json').read().splitlines()[-1]);print('ska',d['value'],d['grid_mvis_s'],d['degrid_mvis_s'],d['e2e']['value'],d['rho_sweep_TOps_s'])"
tail -3 $OUT/bench_ska_$TAG.err
