"""World-size-2/3 gloo tests of the multi-GPU host logic (§8(e)) on CPU: shard cuts,
owner rule and the boundary exchange.  The per-rank partial Y comes from the ORACLE
run on that rank's shard (no GPU here); the row ops are CPU stand-ins injected by the
test (the product path uses sf_rows_op kernels)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from oracle import plan as oplan
from paper_conf_cluster_linwds24_b200.dist import BoundaryExchange, StepExchange, owner_maps


def _cpu_rows_op(Y, rows, buf, op, stream=None):
    for k, r in enumerate(rows.tolist()):
        if r < 0:
            continue
        if op == 0:
            buf[k] = Y[r]
        elif op == 1:
            Y[r] += buf[k]
        else:
            Y[r] = 0


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, dims, nnz, R, seed, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    inds, vals = synth.gen_coo(dims, nnz, seed, zipf=(1.5, 0.5, 0.5), val_kind="int")
    facs = synth.gen_factors(dims, R, seed + 1, "int")
    res = {}
    for n in range(len(dims)):
        perm0 = oplan.matricized_order(dims, inds, n)
        lo, hi = oplan.shard_range(nnz, world, rank)
        sel = perm0[lo:hi]
        Y, _ = oracle.mttkrp(dims, [a[sel] for a in inds], vals[sel], facs, R, n, with_scale=False)
        Yt = torch.from_numpy(Y.astype(np.float32))
        rb = int(inds[n][sel].min()) if hi > lo else 0
        re_ = int(inds[n][sel].max()) + 1 if hi > lo else rb
        ex = BoundaryExchange(world, rank, R, torch.device("cpu"), rows_op=_cpu_rows_op)
        ex.combine(Yt, rb, re_)
        ex.combine  # cached maps reused on a second call
        res[n] = (Yt.numpy(), rb, re_)
    # the same exchange for all modes at once (one all_gather per step) must agree exactly
    items = []
    for n in range(len(dims)):
        perm0 = oplan.matricized_order(dims, inds, n)
        lo, hi = oplan.shard_range(nnz, world, rank)
        sel = perm0[lo:hi]
        Y, _ = oracle.mttkrp(dims, [a[sel] for a in inds], vals[sel], facs, R, n, with_scale=False)
        items.append((torch.from_numpy(Y.astype(np.float32)), res[n][1], res[n][2]))
    sx = StepExchange(world, rank, R, torch.device("cpu"), rows_op=_cpu_rows_op)
    for _ in range(2):  # second call: cached layout; inputs re-made so the sums stay exact
        outs = sx.combine([(Y.clone(), rb, re_) for Y, rb, re_ in items])
    for n in range(len(dims)):
        assert np.array_equal(outs[n].numpy(), res[n][0]), n
    q.put((rank, res))
    dist.destroy_process_group()


@pytest.mark.parametrize("world,nnz", [(2, 3000), (3, 2000), (4, 5)])
def test_boundary_exchange_gloo(world, nnz):
    dims, R, seed = (40, 30, 20), 8, 123
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, dims, nnz, R, seed, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    inds, vals = synth.gen_coo(dims, nnz, seed, zipf=(1.5, 0.5, 0.5), val_kind="int")
    facs = synth.gen_factors(dims, R, seed + 1, "int")
    for n in range(3):
        Yfull, _ = oracle.mttkrp(dims, inds, vals, facs, R, n, with_scale=False)
        ranges = [(out[k][n][1], out[k][n][2]) for k in range(world)]
        zero_rows, _ = owner_maps(ranges)
        total = np.zeros_like(Yfull)
        owned = np.zeros(dims[n], int)
        for k in range(world):
            Yk, rb, re_ = out[k][n]
            mask = np.zeros(dims[n], bool)
            mask[rb:re_] = True
            for r in zero_rows[k]:
                mask[r] = False
            assert not Yk[~mask].any()  # zeros outside owned rows
            assert np.array_equal(Yk[mask], Yfull[mask].astype(np.float32))
            owned += mask
            total += Yk
        assert owned.max() <= 1  # every row owned at most once
        assert np.array_equal(total, Yfull)


def test_owner_maps_heavy_row_spanning_ranks():
    # rank 1 and 2 lie entirely inside row 5 which rank 0 also touches
    ranges = [(0, 6), (5, 6), (5, 6), (5, 9)]
    zero_rows, add_src = owner_maps(ranges)
    assert zero_rows == [[], [5], [5], [5]]
    assert sorted(add_src[0]) == [(5, 1, 0), (5, 2, 0), (5, 3, 0)]
    # empty shards are skipped
    zero_rows, add_src = owner_maps([(0, 3), (3, 3), (2, 4)])
    assert zero_rows == [[], [], [2]] and add_src[0] == [(2, 2, 0)]
