"""World-size-2/3/4 gloo tests of the multi-GPU host logic (§8(e)) on CPU.

* The exchange rule of libscalfrag (sf_exchange_map, host-only C code: which rank sends its
  first row, who owns it) against the rule written out by hand (owner = the
  lowest rank touching the row), including heavy rows spanning several shards and empty
  shards.
* The host-staged allgatherv transport (dist.TorchAllgatherv.allgatherv_host) over real
  gloo process groups with ragged and empty blocks.
* End to end on CPU: each rank's partial Y is the ORACLE on its shard (no GPU here); the
  first-row partials travel through the transport and the owner adds them in rank order
  with the C rule -- the row-sharded result must equal the full oracle Y exactly
  (integer data).  The CUDA side of the same exchange (csrc/sf_comm.cu) is checked on the
  GPU by tests/test_gpu_multirank.py.
"""
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
import paper_conf_cluster_linwds24_b200 as sf


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rule_by_hand(ranges):
    """the owner of a row is the lowest rank touching it; a rank sends its
    first row iff that owner is another rank."""
    P = len(ranges)
    send, owner = [], []
    for k, (b, e) in enumerate(ranges):
        if e <= b:
            send.append(0)
            owner.append(-1)
            continue
        o = min(j for j in range(P) if ranges[j][0] <= b < ranges[j][1] and ranges[j][1] > ranges[j][0])
        send.append(int(o != k))
        owner.append(o)
    return send, owner


@pytest.mark.parametrize("ranges,send,owner", [
    # rank 1 and 2 lie entirely inside row 5 which rank 0 also touches; rank 3 starts there
    ([(0, 6), (5, 6), (5, 6), (5, 9)], [0, 1, 1, 1], [0, 0, 0, 0]),
    # an empty shard in the middle; rank 2 starts on rank 0's last row
    ([(0, 3), (3, 3), (2, 4)], [0, 0, 1], [0, -1, 0]),
    # no shared rows at all
    ([(0, 4), (4, 8), (8, 9)], [0, 0, 0], [0, 1, 2]),
    # everything empty but the last rank
    ([(0, 0), (0, 0), (0, 7)], [0, 0, 0], [-1, -1, 2]),
])
def test_exchange_map_golden(ranges, send, owner):
    """Hand-written expectations for the C exchange rule (csrc/sf_comm.cu exchange_map)."""
    assert sf.exchange_map(ranges) == (send, owner)
    assert _rule_by_hand(ranges) == (send, owner)


def test_exchange_map_random_vs_rule():
    rng = np.random.default_rng(0)
    for _ in range(300):
        P = int(rng.integers(1, 9))
        cuts = np.sort(rng.integers(0, 30, P + 1))
        # monotone touched ranges [row(first), row(last) + 1) with shared boundary rows
        ranges = []
        for k in range(P):
            b, e = int(cuts[k]), int(cuts[k + 1])
            if rng.random() < 0.2:
                ranges.append((b, b))
            else:
                ranges.append((b, max(e, b) + 1 if rng.random() < 0.5 else max(e, b + 1)))
        # keep ranges monotone (row(first) of k+1 >= row(last) of k)
        fixed, last = [], 0
        for b, e in ranges:
            if e > b:
                b = max(b, last)
                e = max(e, b + 1)
                last = e - 1
            fixed.append((b, e))
        assert sf.exchange_map(fixed) == _rule_by_hand(fixed), fixed


def _transport_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_cluster_linwds24_b200.dist import TorchAllgatherv
    tr = TorchAllgatherv(device=torch.device("cpu"))
    nbytes = [(k * 7 + 3) % 11 for k in range(world)]  # ragged, some empty
    send = torch.tensor([(rank * 31 + i) % 251 for i in range(nbytes[rank])], dtype=torch.uint8)
    blocks = tr.allgatherv_host(send, nbytes)
    ok = all(blocks[k].tolist() == [(k * 31 + i) % 251 for i in range(nbytes[k])] for k in range(world))
    q.put((rank, ok))
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3, 4])
def test_torch_allgatherv_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_transport_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(out.values())


def _exchange_worker(rank, world, port, dims, nnz, R, seed, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_cluster_linwds24_b200.dist import TorchAllgatherv
    tr = TorchAllgatherv(device=torch.device("cpu"))
    inds, vals = synth.gen_coo(dims, nnz, seed, zipf=(1.5, 0.5, 0.5), val_kind="int")
    facs = synth.gen_factors(dims, R, seed + 1, "int")
    res = {}
    for n in range(len(dims)):
        perm0 = oplan.matricized_order(dims, inds, n)
        lo, hi = oplan.shard_range(nnz, world, rank)
        sel = perm0[lo:hi]
        Y, _ = oracle.mttkrp(dims, [a[sel] for a in inds], vals[sel], facs, R, n, with_scale=False)
        rb = int(inds[n][sel].min()) if hi > lo else 0
        re_ = int(inds[n][sel].max()) + 1 if hi > lo else rb
        blk = Y[rb:re_].astype(np.float32).copy()  # the local row block sf_mttkrp writes
        ranges = [None] * world
        dist.all_gather_object(ranges, (rb, re_))
        send_first, owner = sf.exchange_map(ranges)
        # the steps of csrc/sf_comm.cu exchange_rows, with the real transport
        send = torch.from_numpy(blk[0].copy()).view(torch.uint8) if send_first[rank] else \
            torch.zeros(R * 4, dtype=torch.uint8)
        got = tr.allgatherv_host(send, [R * 4] * world)
        if send_first[rank]:
            blk[0] = 0
        for k in range(world):  # senders in rank order
            if send_first[k] and owner[k] == rank:
                blk[-1] += got[k].view(torch.float32).numpy()
        res[n] = (blk, rb, re_)
    q.put((rank, res))
    dist.destroy_process_group()


@pytest.mark.parametrize("world,nnz", [(2, 3000), (3, 2000), (4, 5)])
def test_boundary_exchange_gloo(world, nnz):
    dims, R, seed = (40, 30, 20), 8, 123
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_exchange_worker, args=(r, world, port, dims, nnz, R, seed, q))
             for r in range(world)]
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
        send_first, _ = _rule_by_hand(ranges)
        total = np.zeros_like(Yfull)
        owned = np.zeros(dims[n], int)
        for k in range(world):
            blk, rb, re_ = out[k][n]
            mask = np.ones(re_ - rb, bool)
            if send_first[k] and re_ > rb:
                mask[0] = False
            assert not blk[~mask].any()  # zeros outside owned rows
            assert np.array_equal(blk[mask], Yfull[rb:re_][mask].astype(np.float32))
            owned[rb:re_] += mask
            total[rb:re_] += blk
        assert owned.max() <= 1  # every row owned at most once
        assert np.array_equal(total, Yfull)
