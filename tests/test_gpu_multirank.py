"""Multi-rank bench path on a one-GPU box: two ranks launched by torchrun, both on cuda:0
over gloo (IDG_BENCH_SHARED_GPU=1; NCCL refuses two ranks on one GPU).  Exercises what the 1/2/4/8-GPU
runs execute: baseline shards, the covered-band grid reduce / model-grid broadcast, the max-over-ranks
timing, one JSON line from rank 0, and the host-streamed e2e path checked through the adjoint identity
<vis, degrid(grid(vis))> = ||grid(vis)||^2 summed over the shards."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.gpu
@pytest.mark.parametrize("exchange,port", [("nccl", 29547), ("peer", 29548)])
def test_two_rank_bench_on_one_gpu(exchange, port, tmp_path):
    env = dict(os.environ, IDG_BENCH_SHARED_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--config", "lofar", "--steps", "2", "--warmup", "3", "--timesteps", "512",
           "--e2e-steps", "2", "--no-cpu-baseline", "--rho-iterations", "256", "--no-rho-sweep", "--no-kernel-energy",
           "--exchange", exchange]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, p.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["gpu_launches"] > 0
    assert ("banded" in d["config"]["parallelism"]) == (exchange == "peer")
    assert d["e2e"]["value"] > 0
    assert d["e2e"]["check"]["adjoint_identity_rel_err"] < 1e-4
