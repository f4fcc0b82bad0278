"""Run under torchrun (any world size; SF_SAME_GPU=1 puts every rank on cuda:0 with gloo):
each rank plans its shard of every mode, runs sf_mttkrp, exchanges boundary rows, and the
gathered row-sharded Y must equal the single-rank result bit-exactly (integer data)."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
import paper_conf_cluster_linwds24_b200 as sf  # noqa: E402
from paper_conf_cluster_linwds24_b200.dist import BoundaryExchange, owner_maps  # noqa: E402


def main():
    same = os.environ.get("SF_SAME_GPU") == "1"
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    dev = torch.device("cuda", 0 if same else int(os.environ.get("LOCAL_RANK", 0)))
    torch.cuda.set_device(dev)
    dist.init_process_group("gloo" if same else "nccl")
    dims, R = (3000, 2000, 1500), 32
    inds, vals = synth.gen_coo_device(dims, 2_000_000, 77, zipf=(1.3, 0.5, 0.5), val_kind="int")
    facs = synth.gen_factors_device(dims, R, 78, "int")
    ok = True
    for n in range(3):
        with sf.Tensor(dims, inds, vals) as T1:
            T1.plan(n, R)
            full = torch.empty((dims[n], R), device=dev)
            T1.mttkrp(n, facs, full)
        with sf.Tensor(dims, inds, vals) as T:
            T.set_shard(world, rank)
            T.plan(n, R)
            info = T.plan_info(n, R)
            y = torch.empty((dims[n], R), device=dev)
            T.mttkrp(n, facs, y)
            ex = BoundaryExchange(world, rank, R, dev, host_staging=same)
            ex.combine(y, info["row_begin"], info["row_end"])
            torch.cuda.synchronize()
            ranges = [None] * world
            dist.all_gather_object(ranges, (info["row_begin"], info["row_end"]))
            zero_rows, _ = owner_maps(ranges)
            lo, hi = ranges[rank]
            mine = torch.zeros(dims[n], dtype=torch.bool, device=dev)
            mine[lo:hi] = True
            for r in zero_rows[rank]:
                mine[r] = False
            ok &= bool(torch.equal(y[mine], full[mine]))
            ok &= bool((y[~mine] == 0).all())
            cover = mine.to(torch.int32).cpu()
            dist.all_reduce(cover)
            ok &= bool((cover[torch.from_numpy(np.arange(dims[n]))] <= 1).all())
    flag = torch.tensor([1 if ok else 0])
    dist.all_reduce(flag, op=dist.ReduceOp.MIN)
    if rank == 0:
        print("MULTIRANK OK" if flag.item() == 1 else "MULTIRANK MISMATCH", flush=True)
    dist.destroy_process_group()
    sys.exit(0 if flag.item() == 1 else 1)


if __name__ == "__main__":
    main()
