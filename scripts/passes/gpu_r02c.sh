#!/bin/bash
# Round-2 probes: FMA encodings under the rho=17 mix, degridder schedule variants, predict/LOFAR e2e.
set -u
TAG=${1:-r02c}
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_$TAG.log 2>&1 || { echo BUILD FAILED; tail -30 $OUT/build_$TAG.log; exit 1; }
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/rho_forms scripts/rho_forms_probe.cu && /tmp/rho_forms | tee $OUT/rho_forms_$TAG.txt
timeout 300 ncu --metrics smsp__inst_executed.avg.per_cycle_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active,smsp__average_warps_issue_stalled_dispatch_stall_per_issue_active.ratio,smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio,smsp__average_warps_issue_stalled_wait_per_issue_active.ratio,smsp__issue_active.avg.pct_of_peak_sustained_active --csv -c 20 /tmp/rho_forms > $OUT/rho_forms_ncu_$TAG.csv 2>&1; echo "ncu rho forms rc=$?"
python scripts/variant_sweep.py --config ska --timesteps 1024 --which degridder --variants \
  'degridder_rot16<32,W8,minB2,U2,C32>' 'degridder_rot16s1<32,W8,minB2,U2,C32>' 'degridder_rot16s2<32,W8,minB2,U2,C32>' \
  'degridder_rot16s1<32,W8,minB2,U1,C32>' 'degridder_rot16s2<32,W8,minB2,U1,C32>' 2>&1 | tee $OUT/sweep_ska_deg_$TAG.txt
python scripts/variant_sweep.py --config lofar --timesteps 8192 --which degridder --variants \
  'degridder_rot16<24,W4,minB3,U4,C16>' 'degridder_rot16s1<24,W4,minB3,U4,C16>' 'degridder_rot16s2<24,W4,minB3,U2,C16>' 2>&1 | tee $OUT/sweep_lofar_deg_$TAG.txt
python scripts/variant_sweep.py --config predict --timesteps 256 --which degridder --variants \
  'degridder_rot16<32,W8,minB2,U2,C16>' 'degridder_rot16s1<32,W8,minB2,U2,C16>' 'degridder_rot16s2<32,W8,minB2,U1,C16>' 2>&1 | tee $OUT/sweep_predict_deg_$TAG.txt
timeout 900 python bench.py --config predict --steps 10 --warmup 3 --no-rho-sweep > $OUT/bench_predict_$TAG.json 2> $OUT/bench_predict_$TAG.err; echo "bench predict rc=$?"
tail -c 1200 $OUT/bench_predict_$TAG.json; tail -3 $OUT/bench_predict_$TAG.err
timeout 900 python bench.py --config lofar --steps 10 --warmup 3 --no-rho-sweep --no-cpu-baseline --no-kernel-energy > $OUT/bench_lofar_$TAG.json 2> $OUT/bench_lofar_$TAG.err; echo "bench lofar rc=$?"
python -c "import json;d=json.loads(open('$OUT/bench_lofar_$TAG.json').read().splitlines()[-1]);print('lofar',d['value'],d['e2e'])"
