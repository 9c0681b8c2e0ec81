#!/bin/bash
# N = 2 dry run of the default (SKA-shaped) bench path: two ranks on one GPU over gloo (IDG_BENCH_SHARED_GPU=1).
set -u
OUT=gpurun_out; mkdir -p $OUT
python __graft_entry__.py > $OUT/build_r02p.log 2>&1 || { echo BUILD FAILED; exit 1; }
IDG_BENCH_SHARED_GPU=1 timeout 1500 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29561 bench.py --gpus 2 --timesteps 1024 --steps 3 --warmup 3 --no-rho-sweep --no-kernel-energy \
  > $OUT/bench_ska_2rank_r02p.json 2> $OUT/bench_ska_2rank_r02p.err; echo "2-rank ska rc=$?"
python -c "import json;d=json.loads([l for l in open('$OUT/bench_ska_2rank_r02p.json') if l.startswith('{')][-1]);print(d['n_gpus'],d['value'],d['e2e'],d['config']['parallelism'])"
tail -3 $OUT/bench_ska_2rank_r02p.err
