#!/bin/bash
# Round-2 pass i: group-pass gridder variants (SKA), 8-row degridder for short items, host adder bench (LOFAR).
set -u
TAG=${1:-r02i}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
python scripts/variant_sweep.py --config ska --timesteps 1024 --which gridder --variants \
  'gridder_rot2<32,W16,MT4,minB2,KPT4,GP2,nsm>' 'gridder_rot2<32,W16,MT4,minB2,KPT4,GP1,nsm>' \
  'gridder_rot2<32,W16,MT4,minB2,KPT4,GP4,nsm>' 'gridder_rot2<32,W32,MT2,minB1,KPT4,GP2,nsm>' 2>&1 | tee $OUT/sweep_ska_grd_$TAG.txt
python scripts/variant_sweep.py --config lofar_short --timesteps 8192 --which degridder --variants \
  'degridder_rot16<24,W4,minB3,U4,C16>' 'degridder_rot8<24,W8,minB2,U1,C16>' 'degridder_rot8<24,W4,minB3,U2,C16>' 2>&1 | tee $OUT/sweep_lshort_deg_$TAG.txt
python scripts/variant_sweep.py --config lofar --timesteps 8192 --which degridder --variants \
  'degridder_rot16<24,W4,minB3,U4,C16>' 'degridder_rot8<24,W8,minB2,U1,C16>' 'degridder_rot8<24,W4,minB3,U2,C16>' 2>&1 | tee $OUT/sweep_lofar_deg_$TAG.txt
timeout 900 python bench.py --config lofar --steps 10 --warmup 3 --no-rho-sweep --no-cpu-baseline --no-kernel-energy --no-imaging-cycle --host-adder > $OUT/bench_lofar_hostadder_$TAG.json 2> $OUT/bench_lofar_hostadder_$TAG.err; echo "bench lofar host adder rc=$?"
python -c "import json;d=json.loads(open('$OUT/bench_lofar_hostadder_$TAG.json').read().splitlines()[-1]);print('lofar',d['value'],d['host_adder'],d['e2e']['value'])"
tail -3 $OUT/bench_lofar_hostadder_$TAG.err
