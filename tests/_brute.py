"""Brute-force helpers used only by the oracle pins (tests).  Independent of
oracle/ (no shared code): dense tensors, Kolda-Bader unfolding, explicit
Khatri-Rao products."""
import numpy as np


def dense(dims, inds, vals, dtype=np.float64):
    X = np.zeros(dims, dtype=dtype)
    np.add.at(X, tuple(np.asarray(a, dtype=np.int64) for a in inds), np.asarray(vals, dtype=dtype))
    return X


def unfold(X, n):
    """Kolda-Bader mode-n matricization: column j = sum_{k != n} i_k * J_k,
    J_k = prod_{m < k, m != n} I_m  (lower modes vary fastest)."""
    return np.reshape(np.moveaxis(X, n, 0), (X.shape[n], -1), order="F")


def khatri_rao(A, B):
    """Column-wise Kronecker product: (A ⊙ B)[:, r] = kron(A[:, r], B[:, r])."""
    I, R = A.shape
    J, R2 = B.shape
    assert R == R2
    return (A[:, None, :] * B[None, :, :]).reshape(I * J, R)


def krp_chain(factors, n):
    """A^(N) ⊙ ... ⊙ A^(n+1) ⊙ A^(n-1) ⊙ ... ⊙ A^(1)   (Eq. (4))."""
    mats = [factors[m] for m in reversed(range(len(factors))) if m != n]
    K = mats[0]
    for M in mats[1:]:
        K = khatri_rao(K, M)
    return K


def mttkrp_unfold(X, factors, n):
    return unfold(X, n) @ krp_chain(factors, n)


def mttkrp_einsum(X, factors, n):
    N = X.ndim
    letters = "abcdefgh"[:N]
    terms = [letters] + [letters[m] + "z" for m in range(N) if m != n]
    spec = ",".join(terms) + "->" + letters[n] + "z"
    return np.einsum(spec, X, *[factors[m] for m in range(N) if m != n], optimize=True)
