"""the other PAPER.md Table III tensor shapes (synthetic, full size) --
sampled-row parity of every mode in the selector's launch, and bit-exact features."""
import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_cluster_linwds24_b200 as sf
from tests import gpu_util as G

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.mark.parametrize("name", ["vast", "uber", "nips", "enron", "flickr3d", "deli3d", "flickr4d"])
def test_table3_shapes_sampled_rows(cuda_device, name):
    cfg = synth.CONFIGS[name]
    R = cfg.rank
    rng = np.random.default_rng(cfg.seed)
    d_inds, d_vals = synth.config_tensor_device(cfg)
    inds = [a.cpu().numpy().view(np.uint32) for a in d_inds]
    vals = d_vals.cpu().numpy()
    facs_h = synth.config_factors(cfg)
    facs = [torch.from_numpy(f).cuda() for f in facs_h]
    with sf.Tensor(cfg.dims, d_inds, d_vals) as T:
        del d_inds, d_vals
        for n in range(cfg.nmodes):
            T.plan(n, R)
            info = T.plan_info(n, R)
            y = torch.full((cfg.dims[n], R), float("nan"), device="cuda")
            T.mttkrp(n, facs, y)
            torch.cuda.synchronize()
            cnt = np.bincount(inds[n], minlength=cfg.dims[n])
            assert info["features"]["num_slices"] == int(np.count_nonzero(cnt))
            assert info["features"]["max_nnz_per_slice"] == int(cnt.max())
            nz = np.flatnonzero(cnt)
            rows = np.unique(np.r_[np.argsort(cnt)[-3:], rng.choice(nz, min(32, len(nz)), replace=False)])
            Yr, Sr = oracle.mttkrp_rows(cfg.dims, inds, vals, facs_h, R, n, rows)
            got = y[torch.from_numpy(rows).cuda()].cpu().numpy()
            rel, zv = oracle.max_rel_err(got, Yr, Sr)
            assert rel <= G.TOL, (name, n, rel, info["launch"])
            empty = np.flatnonzero(cnt == 0)
            if len(empty):
                e = rng.choice(empty, min(8, len(empty)), replace=False)
                assert not y[torch.from_numpy(e).cuda()].any()
            assert torch.isfinite(y).all()
            T.plan_release(n, R)
