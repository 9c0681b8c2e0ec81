#!/bin/bash
# Round-2 pass zc: bench after moving the rho denominators before the host-streamed legs (SKA default, predict,
# lofar_short) -- the roofline denominators must not depend on what ran before them.
set -u
TAG=${1:-r02zc}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 1500 python bench.py > $OUT/bench_ska_$TAG.json 2> $OUT/bench_ska_$TAG.err; echo "bench ska rc=$?"
for C in predict lofar_short; do
  timeout 1200 python bench.py --config $C --steps 10 --warmup 3 --no-rho-sweep > $OUT/bench_${C}_$TAG.json 2> $OUT/bench_${C}_$TAG.err; echo "bench $C rc=$?"
done
for C in ska predict lofar_short; do
  python -c "import json;d=json.loads(open('$OUT/bench_${C}_$TAG.json').read().splitlines()[-1]);r=d['roofline'];print('$C',round(d['value'],1),(d['e2e'] or {}).get('value'),'rho17',round(r['peak_measured_rho17'],2),'frac',round(r['frac'],3),d['clocks'])"
done
