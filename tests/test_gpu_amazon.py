"""Largest config (BASELINE.json configs[4], amazon-reviews-shaped 4.8M x 1.8M x 1.8M,
nnz = 1,741,809,018, R = 16) at full size on ONE B200: each mode planned by the selector,
run, checked on sampled rows against the oracle, then released (one plan resident at a
time keeps the footprint < 180 GB).  The oracle streams the tensor in 100M-nonzero chunks
(device generator -> host -> oracle.mttkrp_rows, fp64 sums over chunks).  The same rows are
then checked for the one-shot streamed path from pinned host memory."""
import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_cluster_linwds24_b200 as sf
from tests import gpu_util as G

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

CHUNK = 100_000_000


def test_amazon_fullsize_sampled_rows(cuda_device):
    cfg = synth.CONFIGS["amazon"]
    R = cfg.rank
    rng = np.random.default_rng(cfg.seed)
    facs_h = synth.config_factors(cfg)
    facs = [torch.from_numpy(f).cuda() for f in facs_h]
    inds, vals = synth.config_tensor_device(cfg)
    T = sf.Tensor(cfg.dims, inds, vals)
    del inds, vals
    torch.cuda.empty_cache()
    # sampled rows per mode: a random set, plus the heaviest rows found in the first chunk
    first_i, _ = synth.config_tensor_device(cfg, lo=0, hi=CHUNK)
    rows = {}
    for n in range(cfg.nmodes):
        c = torch.bincount(first_i[n].long(), minlength=cfg.dims[n])
        heavy = torch.topk(c, 4).indices.cpu().numpy()
        rnd = rng.choice(cfg.dims[n], 28, replace=False)
        rows[n] = np.unique(np.r_[heavy, rnd]).astype(np.int64)
    del first_i
    torch.cuda.empty_cache()
    # oracle: one pass over the tensor, all modes, chunk by chunk
    Yr = {n: np.zeros((len(rows[n]), R)) for n in range(cfg.nmodes)}
    Sr = {n: np.zeros((len(rows[n]), R)) for n in range(cfg.nmodes)}
    for lo in range(0, cfg.nnz, CHUNK):
        hi = min(cfg.nnz, lo + CHUNK)
        di, dv = synth.config_tensor_device(cfg, lo=lo, hi=hi)
        hi_ = [a.cpu().numpy().view(np.uint32) for a in di]
        hv = dv.cpu().numpy()
        del di, dv
        for n in range(cfg.nmodes):
            y, s = oracle.mttkrp_rows(cfg.dims, hi_, hv, facs_h, R, n, rows[n])
            Yr[n] += y
            Sr[n] += s
    torch.cuda.empty_cache()
    for n in range(cfg.nmodes):
        T.plan(n, R)
        info = T.plan_info(n, R)
        y = torch.full((cfg.dims[n], R), float("nan"), device="cuda")
        T.mttkrp(n, facs, y)
        torch.cuda.synchronize()
        assert torch.isfinite(y).all()
        got = y[torch.from_numpy(rows[n]).cuda()].cpu().numpy()
        rel, zv = oracle.max_rel_err(got, Yr[n], Sr[n])
        assert rel <= G.TOL, (n, rel, info["launch"])
        assert zv == 0.0
        assert info["features"]["nnz"] == cfg.nnz
        del y
        T.plan_release(n, R)
    T.close()
    sf.trim_cache()
    # the one-shot path (sf_mttkrp_streamed_modes: every mode from one upload of the pinned host
    # COO, 16 segments) against the same oracle rows -- the heavy rows' fp32 chains stay short
    inds, vals = synth.config_tensor_device(cfg)
    h_inds = [a.cpu().pin_memory() for a in inds]
    h_vals = vals.cpu().pin_memory()
    del inds, vals
    torch.cuda.empty_cache()
    outs = [torch.full((d, R), float("nan"), device="cuda") for d in cfg.dims]
    sf.mttkrp_streamed_modes(cfg.dims, h_inds, h_vals, facs, outs, 16, 4)
    torch.cuda.synchronize()
    for n in range(cfg.nmodes):
        assert torch.isfinite(outs[n]).all()
        got = outs[n][torch.from_numpy(rows[n]).cuda()].cpu().numpy()
        rel, zv = oracle.max_rel_err(got, Yr[n], Sr[n])
        assert rel <= G.TOL, ("one-shot", n, rel)
        assert zv == 0.0
    sf.trim_cache()
