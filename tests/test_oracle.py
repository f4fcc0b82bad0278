"""Pins for the MTTKRP oracle (oracle/oracle.c) against things other than itself:
hand-computed golden values, the cited textbook unfolding, brute force over the
dense unfolding x explicit Khatri-Rao product (Eq. (4)), einsum,
the rank-1 closed form (Eq. (1)), slice sums, exact integer
arithmetic, SpMM (N=2) via scipy, and invariants."""
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
from tests import _brute as B

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _rand_coo(rng, dims, nnz, signed=True, dup=True):
    inds = [rng.integers(0, d, nnz, dtype=np.int64).astype(np.uint32) for d in dims]
    if dup and nnz >= 4:  # force duplicates
        for a in inds:
            a[-2:] = a[:2]
    vals = (rng.uniform(-1, 1, nnz) if signed else rng.uniform(0, 1, nnz)).astype(np.float32)
    return inds, vals


def _rand_factors(rng, dims, R, signed=True):
    lo = -1 if signed else 0
    return [rng.uniform(lo, 1, (d, R)).astype(np.float32) for d in dims]


def test_golden_worked_example():
    g = json.load(open(os.path.join(GOLD, "worked_example_3way.json")))
    coo = np.array(g["coo"], dtype=np.float64)
    inds = [coo[:, m].astype(np.uint32) for m in range(3)]
    vals = coo[:, 3].astype(np.float32)
    fac = [np.array(f, dtype=np.float32) for f in g["factors"]]
    for n in range(3):
        Y, S = oracle.mttkrp(g["dims"], inds, vals, fac, g["rank"], n)
        assert np.array_equal(Y, np.array(g["Y"][n], dtype=np.float64)), n
        assert np.array_equal(S, np.array(g["S"][n], dtype=np.float64)), n


def test_kolda_bader_unfolding_golden():
    """Pins the brute-force unfolding helper to the textbook's printed example."""
    g = json.load(open(os.path.join(GOLD, "kolda_bader_unfolding.json")))
    X = np.zeros(g["dims"])
    for k, sl in enumerate(g["frontal_slices"]):
        X[:, :, k] = np.array(sl)
    for n, key in enumerate(["X1", "X2", "X3"]):
        assert np.array_equal(B.unfold(X, n), np.array(g[key], dtype=np.float64))


@pytest.mark.parametrize("dims,nnz,R", [((100, 80, 60), 10_000, 16), ((10, 12, 14, 16), 3000, 5),
                                        ((7, 1, 9), 50, 3), ((5, 6, 4, 3, 2), 200, 4)])
def test_brute_force_unfolding_times_krp(dims, nnz, R):
    rng = np.random.default_rng(hash(dims) % 2**32)
    inds, vals = _rand_coo(rng, dims, nnz)
    fac = _rand_factors(rng, dims, R)
    X = B.dense(dims, inds, vals)
    f64 = [f.astype(np.float64) for f in fac]
    for n in range(len(dims)):
        Y, S = oracle.mttkrp(dims, inds, vals, fac, R, n)
        ref = B.mttkrp_unfold(X, f64, n)
        ref2 = B.mttkrp_einsum(X, f64, n)
        scale = B.mttkrp_einsum(np.abs(X), [np.abs(f) for f in f64], n)
        assert np.max(np.abs(Y - ref)) <= 1e-12 * max(1.0, np.max(scale))
        assert np.max(np.abs(Y - ref2)) <= 1e-12 * max(1.0, np.max(scale))
        # S >= |Y| everywhere and S == |.|-MTTKRP when there are no duplicate cancellations
        assert np.all(S + 1e-12 >= np.abs(Y))


def test_scale_is_abs_mttkrp_of_abs_inputs():
    rng = np.random.default_rng(7)
    dims, R = (9, 8, 7), 6
    inds, vals = _rand_coo(rng, dims, 300)
    fac = _rand_factors(rng, dims, R)
    for n in range(3):
        _, S = oracle.mttkrp(dims, inds, vals, fac, R, n)
        Sabs, _ = oracle.mttkrp(dims, inds, np.abs(vals), [np.abs(f) for f in fac], R, n)
        assert np.allclose(S, Sabs, rtol=1e-14, atol=0)


def test_rank1_closed_form_large_dims():
    """X = a_1 ∘ a_2 ∘ a_3 on supports S_m (Eq. (1) with F = 1):
    Y(i, r) = a_n(i) * prod_{m != n} sum_{j in S_m} a_m(j) B_m(j, r)."""
    rng = np.random.default_rng(11)
    dims = (2_902_330, 2_143_368, 25_495_389)  # nell-1 dims: big index ranges
    R = 7
    sup = [np.sort(rng.choice(d, size=k, replace=False)) for d, k in zip(dims, (20, 30, 25))]
    a = [rng.integers(1, 4, len(s)).astype(np.float64) for s in sup]  # small ints: v exact
    grids = np.meshgrid(*[np.arange(len(s)) for s in sup], indexing="ij")
    flat = [g.ravel() for g in grids]
    inds = [sup[m][flat[m]].astype(np.uint32) for m in range(3)]
    vals = (a[0][flat[0]] * a[1][flat[1]] * a[2][flat[2]]).astype(np.float32)
    # factor rows on the supports (compact run), scattered into big factors below
    Bs = [rng.uniform(-1, 1, (len(sup[m]), R)).astype(np.float32) for m in range(3)]
    for n in range(3):
        dims_c = tuple(len(s) for s in sup)
        inds_c = [flat[m].astype(np.uint32) for m in range(3)]
        Y, _ = oracle.mttkrp(dims_c, inds_c, vals, Bs, R, n)
        closed = np.outer(a[n], np.prod([a[m] @ Bs[m].astype(np.float64) for m in range(3) if m != n],
                                        axis=0))
        assert np.allclose(Y, closed, rtol=1e-12, atol=1e-12)
    # big-dims run for the sampled-rows entry point (no I_n x R buffer)
    big_fac = []
    for m in range(3):
        if m == 2:
            big_fac.append(None)  # never read for mode n = 2
            continue
        F = np.zeros((dims[m], R), np.float32)
        F[sup[m]] = Bs[m]
        big_fac.append(F)
    Yr, _ = oracle.mttkrp_rows(dims, inds, vals, big_fac, R, 2, sup[2])
    closed = np.outer(a[2], np.prod([a[m] @ Bs[m].astype(np.float64) for m in (0, 1)], axis=0))
    assert np.allclose(Yr, closed, rtol=1e-12, atol=1e-12)


def test_all_ones_factors_give_slice_sums():
    rng = np.random.default_rng(3)
    dims, R = (50, 40, 30), 4
    inds, vals = _rand_coo(rng, dims, 2000)
    ones = [np.ones((d, R), np.float32) for d in dims]
    for n in range(3):
        Y, _ = oracle.mttkrp(dims, inds, vals, ones, R, n)
        sums = np.bincount(inds[n].astype(np.int64), weights=vals.astype(np.float64), minlength=dims[n])
        assert np.allclose(Y, sums[:, None], rtol=1e-13, atol=1e-13)
        Yc, _ = oracle.mttkrp(dims, inds, np.ones_like(vals), ones, R, n)
        cnt = np.bincount(inds[n].astype(np.int64), minlength=dims[n])
        assert np.array_equal(Yc, np.repeat(cnt[:, None], R, 1).astype(np.float64))


def test_exact_integers():
    rng = np.random.default_rng(5)
    dims, R = (20, 30, 25, 6), 5
    nnz = 4000
    inds = [rng.integers(0, d, nnz).astype(np.uint32) for d in dims]
    vals = rng.integers(1, 5, nnz).astype(np.float32)
    fac = [rng.integers(-2, 3, (d, R)).astype(np.float32) for d in dims]
    for n in range(4):
        Y, _ = oracle.mttkrp(dims, inds, vals, fac, R, n)
        exact = np.zeros((dims[n], R), np.int64)
        p = vals.astype(np.int64)[:, None].repeat(R, 1)
        for m in range(4):
            if m != n:
                p = p * fac[m].astype(np.int64)[inds[m].astype(np.int64)]
        np.add.at(exact, inds[n].astype(np.int64), p)
        assert np.array_equal(Y, exact.astype(np.float64))


def test_spmm_special_case():
    rng = np.random.default_rng(9)
    dims, R = (300, 200), 8
    inds, vals = _rand_coo(rng, dims, 5000)
    fac = _rand_factors(rng, dims, R)
    X = sp.coo_matrix((vals.astype(np.float64), (inds[0], inds[1])), shape=dims).tocsr()
    Y0, _ = oracle.mttkrp(dims, inds, vals, fac, R, 0)
    Y1, _ = oracle.mttkrp(dims, inds, vals, fac, R, 1)
    assert np.allclose(Y0, X @ fac[1].astype(np.float64), rtol=1e-12, atol=1e-12)
    assert np.allclose(Y1, X.T @ fac[0].astype(np.float64), rtol=1e-12, atol=1e-12)


def test_invariants():
    rng = np.random.default_rng(13)
    dims, R = (40, 35, 30), 6
    nnz = 3000
    inds = [rng.integers(0, d, nnz).astype(np.uint32) for d in dims]
    vals = rng.integers(1, 5, nnz).astype(np.float32)
    fac = [rng.integers(-2, 3, (d, R)).astype(np.float32) for d in dims]
    for n in range(3):
        Y, _ = oracle.mttkrp(dims, inds, vals, fac, R, n)
        # permutation of nonzero order (exact on integer data)
        p = rng.permutation(nnz)
        Yp, _ = oracle.mttkrp(dims, [a[p] for a in inds], vals[p], fac, R, n)
        assert np.array_equal(Y, Yp)
        # split every value into two halves (duplicates)
        Yh, _ = oracle.mttkrp(dims, [np.r_[a, a] for a in inds], np.r_[vals / 2, vals / 2], fac, R, n)
        assert np.array_equal(Y, Yh)
        # linearity under concatenation
        h = nnz // 3
        Ya, _ = oracle.mttkrp(dims, [a[:h] for a in inds], vals[:h], fac, R, n)
        Yb, _ = oracle.mttkrp(dims, [a[h:] for a in inds], vals[h:], fac, R, n)
        assert np.array_equal(Y, Ya + Yb)
        # column independence: rank-1 runs stacked == the R-wide run
        for r in (0, R - 1):
            Yr, _ = oracle.mttkrp(dims, inds, vals, [f[:, r:r + 1].copy() for f in fac], 1, n)
            assert np.array_equal(Yr[:, 0], Y[:, r])
        # column checksum 1^T Y(:, r) = sum_e v_e prod A_m(i_m, r)
        prod = vals.astype(np.float64)[:, None] * np.ones((1, R))
        for m in range(3):
            if m != n:
                prod = prod * fac[m].astype(np.float64)[inds[m]]
        assert np.array_equal(Y.sum(0), prod.sum(0))
    # mode relabeling: mode n of X == mode pi(n) of the transposed tensor
    pi = [2, 0, 1]
    dims_t = tuple(dims[pi[k]] for k in range(3))
    inds_t = [inds[pi[k]] for k in range(3)]
    fac_t = [fac[pi[k]] for k in range(3)]
    for k in range(3):
        Yt, _ = oracle.mttkrp(dims_t, inds_t, vals, fac_t, R, k)
        Y, _ = oracle.mttkrp(dims, inds, vals, fac, R, pi[k])
        assert np.array_equal(Y, Yt)


def test_rows_entry_matches_full():
    rng = np.random.default_rng(17)
    dims, R = (64, 50, 40), 8
    inds, vals = _rand_coo(rng, dims, 2500)
    fac = _rand_factors(rng, dims, R)
    for n in range(3):
        Y, S = oracle.mttkrp(dims, inds, vals, fac, R, n)
        rows = rng.choice(dims[n], 9, replace=False)
        Yr, Sr = oracle.mttkrp_rows(dims, inds, vals, fac, R, n, rows)
        assert np.array_equal(Yr, Y[rows]) and np.array_equal(Sr, S[rows])


def test_edge_cases():
    dims, R = (5, 4, 3), 2
    fac = [np.ones((d, R), np.float32) for d in dims]
    e = [np.zeros(0, np.uint32)] * 3
    Y, S = oracle.mttkrp(dims, e, np.zeros(0, np.float32), fac, R, 1)
    assert Y.shape == (4, 2) and not Y.any() and not S.any()
    bad = [np.array([0], np.uint32), np.array([4], np.uint32), np.array([0], np.uint32)]
    with pytest.raises(ValueError):
        oracle.mttkrp(dims, bad, np.ones(1, np.float32), fac, R, 0)


def test_max_rel_err_metric():
    Y = np.array([[1.0, 0.0]])
    S = np.array([[2.0, 0.0]])
    rel, zv = oracle.max_rel_err(np.array([[1.0002, 0.0]]), Y, S)
    assert abs(rel - 1e-4) < 1e-12 and zv == 0.0
    rel, zv = oracle.max_rel_err(np.array([[1.0, 1e-30]]), Y, S)
    assert zv == 1e-30
