#!/usr/bin/env python
"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck):
every kernel family of libscalfrag on a skewed tiny tensor and a heavy-row tensor --
frag3 in owner / memset+atomics / shared-memory-staged / L2-tiled / hot-row / deterministic
launches, 3-way and 4-way (packed records), the sorted-segment streamed paths (one mode /
all modes from one upload), shards,
CP-ALS.  Checks every result against the oracle so a silent corruption also fails.

  compute-sanitizer --tool memcheck  python tools/sanitize_check.py
  compute-sanitizer --tool racecheck python tools/sanitize_check.py
  compute-sanitizer --tool synccheck python tools/sanitize_check.py
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import synth  # noqa: E402


def main():
    import torch

    import paper_conf_cluster_linwds24_b200 as sf
    FRAG = sf.KERNEL_FRAG
    cases = [((100, 80, 60), 10_000, (1.0, 1.0, 1.0), 16), ((40, 3000, 2000), 200_000, (2.0, 0.5, 0.5), 32),
             ((20, 30, 40, 50), 20_000, (1.0, 0.5, 0.8, 0.3), 16)]
    worst = 0.0
    for dims, nnz, zipf, R in cases:
        inds, vals = synth.gen_coo(dims, nnz, 5, zipf=zipf, val_kind="signed")
        facs = synth.gen_factors(dims, R, 6, "signed")
        ti = [torch.from_numpy(a.view(np.int32)).cuda() for a in inds]
        tv = torch.from_numpy(vals).cuda()
        tf = [torch.from_numpy(f).cuda() for f in facs]
        N = len(dims)
        for n in range(N):
            others = [m for m in range(N) if m != n]
            launches = [None,
                        sf.Launch.make(kernel=FRAG, chunk_nnz=64),
                        sf.Launch.make(kernel=FRAG, chunk_nnz=64, flags=sf.LAUNCH_NO_OWNER_STORES),
                        sf.Launch.make(kernel=FRAG, chunk_nnz=32, staged={others[0]: 7}),
                        sf.Launch.make(kernel=FRAG, chunk_nnz=48, staged={others[-1]: max(1, dims[others[-1]] // 3)},
                                       flags=sf.LAUNCH_L2_TILES, hot_kb=1),
                        sf.Launch.make(kernel=FRAG, chunk_nnz=64, block_threads=1024, hot_kb=2),
                        sf.Launch.make(kernel=FRAG, chunk_nnz=64, flags=sf.LAUNCH_DETERMINISTIC),
                        sf.Launch.make(kernel=sf.KERNEL_COO)]
            Y, S = oracle.mttkrp(dims, inds, vals, facs, R, n)
            for L in launches:
                for shard in (None, (3, 1)):
                    with sf.Tensor(dims, ti, tv) as T:
                        if shard:
                            T.set_shard(*shard)
                        if L is None:
                            T.plan(n, R)
                        else:
                            T.set_launch(n, R, L)
                        info = T.plan_info(n, R)
                        y = torch.full((info["out_rows"], R), float("nan"), device="cuda")
                        T.mttkrp(n, tf, y)
                        torch.cuda.synchronize()
                        if shard is None:
                            rel, zv = oracle.max_rel_err(y.cpu().numpy(), Y, S)
                            assert rel <= 1e-4 and zv == 0, (dims, n, L and L.as_dict(), rel)
                            worst = max(worst, rel)
                        else:
                            assert torch.isfinite(y).all()
            y = torch.full((dims[n], R), float("nan"), device="cuda")
            sf.mttkrp_streamed(dims, inds, vals, tf, n, y, 3, 2)
            rel, zv = oracle.max_rel_err(y.cpu().numpy(), Y, S)
            assert rel <= 1e-4 and zv == 0, ("streamed", dims, n, rel)
        # every mode from one upload (sf_mttkrp_streamed_modes, 16/32-byte segment records)
        outs = [torch.full((d, R), float("nan"), device="cuda") for d in dims]
        sf.mttkrp_streamed_modes(dims, inds, vals, tf, outs, 5, 3)
        for n in range(N):
            Y, S = oracle.mttkrp(dims, inds, vals, facs, R, n)
            rel, zv = oracle.max_rel_err(outs[n].cpu().numpy(), Y, S)
            assert rel <= 1e-4 and zv == 0, ("streamed_modes", dims, n, rel)
        if N == 3 and R <= 64:
            with sf.Tensor(dims, ti, tv) as T:
                A = [f.clone() for f in tf]
                fits = T.cp_als(A, iters=2)
                assert all(np.isfinite(fits))
    # host inputs: segmented upload with presort, the upload-time AoS copy and row counts of a
    # >= 2^18-row mode (warp-aggregated atomics), the smem-histogram counts of small modes,
    # one-pass run statistics, hot-row plans
    dims, R = (300_000, 50, 400), 16
    inds, vals = synth.gen_coo(dims, 100_003, 7, zipf=(1.2, 0.7, 0.9), val_kind="signed")
    facs = synth.gen_factors(dims, R, 8, "signed")
    tf = [torch.from_numpy(f).cuda() for f in facs]
    hi = [torch.from_numpy(a.view(np.int32)).pin_memory() for a in inds]
    hv = torch.from_numpy(vals).pin_memory()
    with sf.Tensor(dims, hi, hv, segments=5, streams=3) as T:
        for n in range(3):
            for L in (None, sf.Launch.make(kernel=FRAG, chunk_nnz=64, block_threads=1024, hot_kb=64)):
                if L is None:
                    T.plan(n, R)
                else:
                    T.set_launch(n, R, L)
                y = torch.full((dims[n], R), float("nan"), device="cuda")
                T.mttkrp(n, tf, y)
                torch.cuda.synchronize()
                Y, S = oracle.mttkrp(dims, inds, vals, facs, R, n)
                rel, zv = oracle.max_rel_err(y.cpu().numpy(), Y, S)
                assert rel <= 1e-4 and zv == 0, ("host input", n, rel)
                worst = max(worst, rel)
    print(f"SANITIZE WORKLOAD OK (worst rel err {worst:.2e}, {sf.kernel_launches()} kernels)")


if __name__ == "__main__":
    main()
