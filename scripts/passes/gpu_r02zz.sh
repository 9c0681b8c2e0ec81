#!/bin/bash
# Round-2 pass zz: final records on HEAD (16-row integer degridders at unroll 8) -- smoke, bench lines for every config + reference arm, the SKA
# launch list of the default command, and the GPU suite.
set -u
TAG=${1:-r02zz}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -20 $OUT/build_$TAG.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_$TAG.log 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke_$TAG.log
timeout 1500 python bench.py > $OUT/bench_ska_$TAG.json 2> $OUT/bench_ska_$TAG.err; echo "bench ska rc=$?"
timeout 900 python bench.py --impl reference > $OUT/bench_ref_$TAG.json 2> $OUT/bench_ref_$TAG.err; echo "reference rc=$?"
for C in lofar lofar_dde predict lofar_short; do
  EXTRA=""; [ $C = lofar ] && EXTRA="--host-adder"
  timeout 1200 python bench.py --config $C --steps 10 --warmup 3 --no-rho-sweep $EXTRA > $OUT/bench_${C}_$TAG.json 2> $OUT/bench_${C}_$TAG.err; echo "bench $C rc=$?"
done
for C in ska lofar lofar_dde predict lofar_short; do
  python -c "import json;d=json.loads(open('$OUT/bench_${C}_$TAG.json').read().splitlines()[-1]);print('$C',round(d['value'],1),d['grid_mvis_s'],d['degrid_mvis_s'],(d['e2e'] or {}).get('value'),(d.get('host_adder') or {}).get('value'),d['clocks'])"
done
python -c "import json;d=json.loads(open('$OUT/bench_ref_$TAG.json').read().splitlines()[-1]);print('reference',d.get('value'),d.get('unit'))"
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_ska_$TAG.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-rho-sweep --no-kernel-energy --no-imaging-cycle \
    > $OUT/bench_ska_under_ncu_$TAG.json 2>&1; echo "ncu ska launches rc=$?"
start=$(date +%s)
timeout 1500 python -m pytest tests -m gpu -q > $OUT/pytest_gpu_$TAG.log 2>&1; echo "pytest gpu rc=$? in $(( $(date +%s) - start ))s"
tail -2 $OUT/pytest_gpu_$TAG.log
for C in ska lofar; do
  EXTRA=""; [ $C = ska ] && EXTRA="--timesteps 1024"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:^degridder_ -s 1 -c 1 \
      -o $OUT/prof_${C}_degridder_$TAG -f python bench.py --config $C $EXTRA --steps 1 --warmup 3 --no-e2e \
      --no-cpu-baseline --no-rho-sweep --no-kernel-energy --no-imaging-cycle > $OUT/ncu_${C}_degridder_$TAG.log 2>&1
  echo "ncu $C degridder rc=$?"
done
