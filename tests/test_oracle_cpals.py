"""Pins for the CP-ALS oracle (oracle/cpals.py, Algorithm 1)."""
import numpy as np

import oracle
from oracle import cpals
from tests import _brute as B


def _dense_coo(X):
    idx = np.nonzero(X)
    return [i.astype(np.uint32) for i in idx], X[idx].astype(np.float32)


def test_mttkrp64_matches_c_oracle():
    rng = np.random.default_rng(0)
    dims, R = (9, 7, 8), 5
    inds = [rng.integers(0, d, 300).astype(np.uint32) for d in dims]
    vals = rng.uniform(-1, 1, 300).astype(np.float32)
    A = [rng.uniform(-1, 1, (d, R)).astype(np.float32) for d in dims]
    for n in range(3):
        Y, _ = oracle.mttkrp(dims, inds, vals, A, R, n)
        M = cpals._mttkrp64(dims, inds, vals, [a.astype(np.float64) for a in A], R, n)
        assert np.allclose(M, Y, rtol=1e-12, atol=1e-12)


def test_fit_formula_vs_dense_reconstruction():
    rng = np.random.default_rng(1)
    dims, R = (6, 5, 4), 3
    X = rng.uniform(-1, 1, dims) * (rng.uniform(size=dims) < 0.5)
    inds, vals = _dense_coo(X)
    A = [rng.uniform(-1, 1, (d, R)) for d in dims]
    Xhat = np.einsum("ir,jr,kr->ijk", *A)
    M = cpals._mttkrp64(dims, inds, vals, A, R, 2)
    f = cpals.fit_value(float(np.sum(vals.astype(np.float64) ** 2)), cpals.grams(A), M, A[2])
    Xf = B.dense(dims, inds, vals)
    assert abs(f - (1 - np.linalg.norm(Xf - Xhat) / np.linalg.norm(Xf))) < 1e-12


def test_als_update_solves_normal_equations():
    """After line 5, A_n satisfies A_n V = M (least-squares optimality in mode n)."""
    rng = np.random.default_rng(2)
    dims, R = (10, 9, 8), 4
    X = rng.uniform(0, 1, dims) * (rng.uniform(size=dims) < 0.3)
    inds, vals = _dense_coo(X)
    A0 = [rng.uniform(0, 1, (d, R)) for d in dims]
    A, _ = cpals.cp_als(dims, inds, vals, A0, R, iters=1)
    # last update was mode N-1 with the final other factors
    n = 2
    V = cpals.hadamard_except(cpals.grams(A), n)
    M = cpals._mttkrp64(dims, inds, vals, A, R, n)
    assert np.allclose(A[n] @ V, M, rtol=1e-9, atol=1e-9)
    # and it is the least-squares solution against the dense unfolding
    K = B.krp_chain(A, n)
    sol, *_ = np.linalg.lstsq(K, B.unfold(B.dense(dims, inds, vals), n).T, rcond=None)
    assert np.allclose(A[n], sol.T, rtol=1e-8, atol=1e-8)


def test_recovers_exact_low_rank_tensor():
    rng = np.random.default_rng(3)
    dims, R = (12, 10, 9), 3
    T = [rng.uniform(0.5, 1.5, (d, R)) for d in dims]
    X = np.einsum("ir,jr,kr->ijk", *T)
    inds, vals = _dense_coo(X)
    A0 = [t + 0.05 * rng.standard_normal(t.shape) for t in T]
    A, fits = cpals.cp_als(dims, inds, vals, A0, R, iters=30)
    assert fits[-1] > 0.999
    assert all(b >= a - 1e-9 for a, b in zip(fits, fits[1:]))  # ALS is monotone
