"""The N>1 bench path on one GPU: torchrun with 2 ranks sharing cuda:0 (gloo collectives,
SF_SAME_GPU=1) -- shards, boundary exchange and max-over-ranks timing run end to end, and
the exchanged row-sharded Y equals the 1-rank result (checked inside tools/multirank_check.py)."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_two_ranks_same_gpu_exchange_matches_single(cuda_device):
    env = dict(os.environ, SF_SAME_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=29533", os.path.join(ROOT, "tools", "multirank_check.py")]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    assert "MULTIRANK OK" in r.stdout, r.stdout[-3000:]


def test_bench_two_ranks_same_gpu(cuda_device):
    env = dict(os.environ, SF_SAME_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=29534", os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "3", "--warmup", "3", "--config", "vast", "--no-cpu", "--e2e-steps", "1"]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    import json
    line = [l for l in r.stdout.splitlines() if l.startswith("{")][-1]
    d = json.loads(line)
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["config"]["parallelism"] == "nnz-shard2"
