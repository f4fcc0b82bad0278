"""CP-ALS (Algorithm 1) on the GPU (sf_cpals) against the fp64 oracle (oracle/cpals.py)."""
import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_cluster_linwds24_b200 as sf
from oracle import cpals as ocp
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


def _lowrank_coo(rng, dims, R, density, noise=0.01):
    T = [rng.uniform(0.2, 1.0, (d, R)) for d in dims]
    mask = rng.uniform(size=dims) < density
    idx = np.nonzero(mask)
    X = np.einsum("ir,jr,kr->ijk", *T)[idx] + noise * rng.standard_normal(len(idx[0]))
    return [i.astype(np.uint32) for i in idx], X.astype(np.float32)


@pytest.mark.parametrize("R", [8, 16, 32, 64])
def test_cpals_matches_oracle(cuda_device, R):
    rng = np.random.default_rng(R)
    dims = (60, 50, 40)
    inds, vals = _lowrank_coo(rng, dims, 4, 0.3)
    init = [rng.uniform(0.1, 1.0, (d, R)).astype(np.float32) for d in dims]
    A_ref, fits_ref = ocp.cp_als(dims, inds, vals, [a.astype(np.float64) for a in init], R, iters=3)
    facs = [G.dev_f(a) for a in init]
    with sf.Tensor(dims, G.dev_inds(inds), G.dev_f(vals)) as T:
        fits = T.cp_als(facs, iters=3)
    assert len(fits) == 3
    assert np.allclose(fits, fits_ref, atol=2e-4), (fits, fits_ref)
    for m in range(3):
        got = facs[m].cpu().numpy().astype(np.float64)
        rel = np.linalg.norm(got - A_ref[m]) / np.linalg.norm(A_ref[m])
        assert rel < 5e-3, (m, rel)


def test_cpals_one_sweep_tight(cuda_device):
    """One sweep from the same init: every factor within fp32 rounding x conditioning."""
    rng = np.random.default_rng(5)
    dims, R = (30, 25, 20, 6), 8
    inds, vals = synth.gen_coo(dims, 3000, 9, zipf=(0.5,) * 4, val_kind="signed")
    init = [rng.uniform(0.1, 1.0, (d, R)).astype(np.float32) for d in dims]
    A_ref, fits_ref = ocp.cp_als(dims, inds, vals, [a.astype(np.float64) for a in init], R, iters=1)
    facs = [G.dev_f(a) for a in init]
    with sf.Tensor(dims, G.dev_inds(inds), G.dev_f(vals)) as T:
        fits = T.cp_als(facs, iters=1)
    assert abs(fits[0] - fits_ref[0]) < 1e-4
    for m in range(4):
        got = facs[m].cpu().numpy().astype(np.float64)
        assert np.linalg.norm(got - A_ref[m]) / np.linalg.norm(A_ref[m]) < 2e-3


def test_cpals_fullsize_nell2_properties(cuda_device):
    """Full nell-2 shape: fits finite, in [-1, 1] and non-decreasing (ALS is monotone), and the
    last update solves its normal equations A_N V = M on sampled rows (oracle MTTKRP)."""
    cfg = synth.CONFIGS["nell2"]
    inds, vals = synth.config_tensor_device(cfg)
    facs = synth.config_factors_device(cfg)
    with sf.Tensor(cfg.dims, inds, vals) as T:
        fits = T.cp_als(facs, iters=3)
    assert all(np.isfinite(fits)) and fits[-1] <= 1.0
    assert all(b >= a - 1e-4 for a, b in zip(fits, fits[1:])), fits
    hi, hv = synth.config_tensor(cfg)
    A = [f.cpu().numpy() for f in facs]
    n = cfg.nmodes - 1
    V = ocp.hadamard_except(ocp.grams([a.astype(np.float64) for a in A]), n)
    rows = np.random.default_rng(0).choice(cfg.dims[n], 32, replace=False)
    M, S = oracle.mttkrp_rows(cfg.dims, hi, hv, A, cfg.rank, n, rows)
    lhs = A[n][rows].astype(np.float64) @ V
    assert np.max(np.abs(lhs - M) / (np.abs(M).max() + 1e-30)) < 1e-3
