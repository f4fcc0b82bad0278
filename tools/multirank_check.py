"""Run under torchrun (any world size; SF_SAME_GPU=1 puts every rank on cuda:0 with the gloo
transport, else NCCL): each rank plans its shard of every mode, runs sf_mttkrp (which ends with
the boundary exchange inside libscalfrag), and
  * the row-sharded local blocks must equal the single-rank result bit-exactly on the rows
    each rank owns and be 0 elsewhere (integer data), every row owned at most once;
  * sf_allgather_rows must rebuild the full single-rank Y on every rank;
  * sf_cpals on the shards must give the same fits and factors as on one rank;
  * the one-shot path on each rank's nonzero range, summed over ranks, must equal one rank's Y."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
import paper_conf_cluster_linwds24_b200 as sf  # noqa: E402
from paper_conf_cluster_linwds24_b200 import dist as sfdist  # noqa: E402


def main():
    same = os.environ.get("SF_SAME_GPU") == "1"
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    dev = torch.device("cuda", 0 if same else int(os.environ.get("LOCAL_RANK", 0)))
    torch.cuda.set_device(dev)
    dist.init_process_group("gloo" if same else "nccl", device_id=None if same else dev)
    dims, R = (3000, 2000, 1500), 32
    # heavy first mode so one row spans several shards at world >= 3
    inds, vals = synth.gen_coo_device(dims, 2_000_000, 77, zipf=(1.3, 0.5, 0.5), val_kind="int")
    facs = synth.gen_factors_device(dims, R, 78, "int")
    ok = True
    msgs = []
    for n in range(3):
        with sf.Tensor(dims, inds, vals) as T1:
            T1.plan(n, R)
            full = torch.empty((dims[n], R), device=dev)
            T1.mttkrp(n, facs, full)
        with sf.Tensor(dims, inds, vals) as T:
            sfdist.attach(T, world, rank)
            if n == 0:
                T.comm_check()  # the transport's allgatherv / alltoallv deliver every word
            T.plan(n, R)
            info = T.plan_info(n, R)
            y = torch.full((info["out_rows"], R), float("nan"), device=dev)
            T.mttkrp(n, facs, y)
            torch.cuda.synchronize()
            ranges = [None] * world
            dist.all_gather_object(ranges, (info["row_begin"], info["row_end"]))
            send_first, owner = sf.exchange_map(ranges)
            lo, hi = ranges[rank]
            mine = torch.zeros(hi - lo, dtype=torch.bool, device=dev)
            mine[:] = True
            if send_first[rank] and hi > lo:
                mine[0] = False
            yf = full[lo:hi]
            ok_n = bool(torch.equal(y[mine], yf[mine])) and bool((y[~mine] == 0).all())
            cover = torch.zeros(dims[n], dtype=torch.int32)
            cover[lo:hi] = mine.to(torch.int32).cpu()
            dist.all_reduce(cover)
            ok_n &= bool((cover <= 1).all())
            # replicated Y from the row-sharded blocks
            rep = torch.empty((dims[n], R), device=dev)
            T.allgather_rows(n, y, rep)
            torch.cuda.synchronize()
            ok_n &= bool(torch.equal(rep, full))
            if not ok_n:
                msgs.append(f"mode {n} rank {rank} ranges {ranges}")
            ok &= ok_n
    # distributed ingest (sf_tensor_create_dist): rank p holds only input
    # positions [p*nnz/P, (p+1)*nnz/P); its shard plans must equal the v1 shard plans bit for bit
    # (kernel order as global input positions, chunks) and give the same Y blocks
    nnz = int(vals.numel())
    lo, hi = rank * nnz // world, (rank + 1) * nnz // world
    for n in range(3):
        L = sf.Launch.make(kernel=sf.KERNEL_FRAG, chunk_nnz=128)
        with sf.Tensor(dims, inds, vals) as T1, \
                sf.Tensor.create_dist(dims, nnz, lo, [a[lo:hi] for a in inds], vals[lo:hi]) as T2:
            sfdist.attach(T1, world, rank)
            sfdist.attach(T2, world, rank)
            T1.set_launch(n, R, L)
            T2.set_launch(n, R, L)
            p1, c1 = T1.plan_export(n, R)
            p2, c2 = T2.plan_export(n, R)
            i1, i2 = T1.plan_info(n, R), T2.plan_info(n, R)
            y1 = torch.empty((i1["out_rows"], R), device=dev)
            y2 = torch.empty((i2["out_rows"], R), device=dev)
            T1.mttkrp(n, facs, y1)
            T2.mttkrp(n, facs, y2)
            torch.cuda.synchronize()
            same = (np.array_equal(p1, p2) and np.array_equal(c1, c2) and i1["row_begin"] == i2["row_begin"]
                    and i1["row_end"] == i2["row_end"] and bool(torch.equal(y1, y2)))
            if not same:
                ok = False
                msgs.append(f"dist v2 mode {n} rank {rank}: plan/Y differ from v1")
            # the selector's own launches (hot rows where they apply) on both: integer data, so
            # any summation order gives the same Y bit for bit
            T1.plan_release(n, R)
            T2.plan_release(n, R)
            T1.plan(n, R)
            T2.plan(n, R)
            y1.zero_()
            y2.zero_()
            T1.mttkrp(n, facs, y1)
            T2.mttkrp(n, facs, y2)
            torch.cuda.synchronize()
            if not torch.equal(y1, y2):
                ok = False
                msgs.append(f"dist v2 mode {n} rank {rank}: auto-planned Y differs from v1")
    # the one-shot path at N ranks (bench.py's e2e leg): each rank streams its nonzero range from
    # host memory into partial Ys of every mode; their sum over ranks (all-reduce) must equal the
    # single-rank Y bit for bit (integer data)
    h_i = [a[lo:hi].cpu().pin_memory() for a in inds]
    h_v = vals[lo:hi].cpu().pin_memory()
    parts = [torch.empty((d, R), device=dev) for d in dims]
    sf.mttkrp_streamed_modes(dims, h_i, h_v, facs, parts, 4, 2)
    torch.cuda.synchronize()
    for n in range(3):
        with sf.Tensor(dims, inds, vals) as T1:
            T1.plan(n, R)
            full = torch.empty((dims[n], R), device=dev)
            T1.mttkrp(n, facs, full)
        torch.cuda.synchronize()
        tot = parts[n].cpu() if os.environ.get("SF_SAME_GPU") == "1" else parts[n]
        dist.all_reduce(tot)
        if not torch.equal(tot.to(dev), full):
            ok = False
            msgs.append(f"one-shot mode {n} rank {rank}: sum of the partial Ys differs from one rank")
    # CP-ALS on the shards == CP-ALS on one rank (same initial factors) up to fp32 summation
    # order (the shards sum M and the Grams in a different order): the bar of
    # tests/test_gpu_cpals.py against the fp64 oracle (fits 2e-4 over 3 sweeps, factors 2e-3
    # after one sweep)
    # signed initial factors: all-positive ones make V = *_m A_m^T A_m nearly rank one, and its
    # pseudo-inverse would amplify summation-order differences far beyond the fp32 level
    fd = [torch.rand((d, 16), device=dev, generator=torch.Generator(device=dev).manual_seed(5 + m)) * 2 - 1
          for m, d in enumerate(dims)]
    vals_f = torch.rand(vals.shape, device=dev, generator=torch.Generator(device=dev).manual_seed(9))
    res = {}
    for iters in (1, 3):
        with sf.Tensor(dims, inds, vals_f) as T1:
            a1 = [f.clone() for f in fd]
            fits1 = T1.cp_als(a1, iters=iters)
        with sf.Tensor(dims, inds, vals_f) as T:
            sfdist.attach(T, world, rank)
            a2 = [f.clone() for f in fd]
            fits2 = T.cp_als(a2, iters=iters)
        torch.cuda.synchronize()
        res[iters] = (fits1, fits2, [float((a1[m] - a2[m]).abs().max() / a1[m].abs().max()) for m in range(3)])
    fits1, fits2, _ = res[3]
    for k in range(3):
        if abs(fits1[k] - fits2[k]) > 2e-4:
            ok = False
            msgs.append(f"cpals fit {k}: {fits1[k]} vs {fits2[k]}")
    for m, rel in enumerate(res[1][2]):  # one sweep: 2e-3 (test_gpu_cpals.py's one-sweep bar)
        if not rel < 2e-3:
            ok = False
            msgs.append(f"cpals factor {m} after one sweep: rel diff {rel}")
    flag = torch.tensor([1 if ok else 0])
    dist.all_reduce(flag, op=dist.ReduceOp.MIN)
    for mm in msgs:
        print(mm, flush=True)
    if rank == 0:
        print("MULTIRANK OK" if flag.item() == 1 else "MULTIRANK MISMATCH", flush=True)
    dist.destroy_process_group()
    sys.exit(0 if flag.item() == 1 else 1)


if __name__ == "__main__":
    main()
