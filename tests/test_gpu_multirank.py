"""The N>1 path on one GPU: torchrun with 2/3/5 ranks sharing cuda:0 (SF_SAME_GPU=1: the
library's exchange runs over the host-staged gloo allgatherv transport) -- shards, the
C-side boundary exchange (heavy rows spanning several shards at 3 and 5 ranks),
sf_allgather_rows, sharded CP-ALS and max-over-ranks timing run end to end and equal the
1-rank results (checked inside tools/multirank_check.py).  With >= 2 GPUs the same check
runs over NCCL (sf_comm_attach), one rank per GPU."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("world", [2, 3, 5])
def test_ranks_same_gpu_exchange_matches_single(cuda_device, world):
    env = dict(os.environ, SF_SAME_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr=127.0.0.1", f"--master-port={29533 + world}", os.path.join(ROOT, "tools", "multirank_check.py")]
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
    # both host-input paths at N = 2: resident shards, and the one-shot path on each rank's
    # nonzero range with the partial Ys combined across ranks
    assert set(d["e2e"]["paths"]) == {"resident", "one_shot"}, d["e2e"]
    assert all(v["ms_per_step"] > 0 for v in d["e2e"]["paths"].values())


def test_nccl_ranks_exchange_matches_single(cuda_device):
    """The NCCL data plane (sf_comm_attach: grouped ncclBroadcast allgatherv), one rank per GPU."""
    import torch
    n = torch.cuda.device_count()
    if n < 2:
        pytest.skip("needs >= 2 GPUs for NCCL (two ranks may not share a device)")
    env = dict(os.environ)
    env.pop("SF_SAME_GPU", None)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={min(n, 4)}",
           "--master-addr=127.0.0.1", "--master-port=29547", os.path.join(ROOT, "tools", "multirank_check.py")]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    assert "MULTIRANK OK" in r.stdout, r.stdout[-3000:]


def test_nccl_one_rank_data_plane(cuda_device):
    """The NCCL transport on the one GPU gpurun gives: a 1-rank communicator (dlopen'ed
    libnccl.so.2, ncclGetUniqueId, ncclCommInitRank, grouped ncclBroadcast = allgatherv, grouped
    ncclSend / ncclRecv to self = alltoallv) delivers every word (sf_comm_check), and the
    attached handle's MTTKRP and sf_allgather_rows equal the unattached result bitwise."""
    import numpy as np
    import torch

    import synth
    import paper_conf_cluster_linwds24_b200 as sf
    dims, R = (300, 200, 250), 32
    inds, vals = synth.gen_coo(dims, 30011, 5, zipf=(1.0, 0.7, 0.9), val_kind="int")
    facs = [torch.from_numpy(f).cuda() for f in synth.gen_factors(dims, R, 6, "int")]
    ti = [torch.from_numpy(a.view(np.int32)).cuda() for a in inds]
    tv = torch.from_numpy(vals).cuda()
    for n in range(3):
        ref = torch.empty((dims[n], R), device="cuda")
        with sf.Tensor(dims, ti, tv) as T0:
            T0.plan(n, R)
            T0.mttkrp(n, facs, ref)
        with sf.Tensor(dims, ti, tv) as T:
            T.comm_attach(1, 0, sf.comm_unique_id())
            T.comm_check()
            T.plan(n, R)
            y = torch.empty((T.plan_info(n, R)["out_rows"], R), device="cuda")
            T.mttkrp(n, facs, y)
            full = torch.empty((dims[n], R), device="cuda")
            T.allgather_rows(n, y, full)
            torch.cuda.synchronize()
            assert torch.equal(y, ref) and torch.equal(full, ref)
