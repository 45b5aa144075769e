"""Independent test-side helpers: dense expansion, textbook dense GEPP brute
force, backward error.  These are the *pins* the oracle is checked against;
they do not call oracle/ or the CUDA path.
"""
from __future__ import annotations

import numpy as np

EPS = 2.0 ** -53  # dlamch('E'), SURVEY 8(c) Q15


def band_to_dense(ab: np.ndarray, m: int, n: int, kl: int, ku: int) -> np.ndarray:
    """Original matrix A (m x n) from band storage ab [n, ldab] (AB(kv+i-j, j) = A(i, j))."""
    kv = kl + ku
    A = np.zeros((m, n))
    for j in range(n):
        for i in range(max(0, j - ku), min(m, j + kl + 1)):
            A[i, j] = ab[j, kv + i - j]
    return A


def dense_gepp(A: np.ndarray):
    """Textbook right-looking LU with partial pivoting (LAPACK dgetf2 order,
    whole-row swaps, first max on ties).  Returns (LU, ipiv 1-based, info)."""
    A = A.copy()
    m, n = A.shape
    ipiv = np.zeros(min(m, n), dtype=np.int64)
    info = 0
    for j in range(min(m, n)):
        col = np.abs(A[j:, j])
        p = j + int(np.argmax(col))  # numpy argmax returns the first max
        ipiv[j] = p + 1
        if A[p, j] != 0.0:
            if p != j:
                A[[j, p], :] = A[[p, j], :]
            A[j + 1:, j] /= A[j, j]
            A[j + 1:, j + 1:] -= np.outer(A[j + 1:, j], A[j, j + 1:])
        elif info == 0:
            info = j + 1
    return A, ipiv, info


def band_factors_to_dense(lu_band: np.ndarray, ipiv: np.ndarray, m: int, n: int, kl: int, ku: int):
    """(L, U) dense from band factors: U from band rows 0..kv; L column j from
    band rows kv+1.. with the later interchanges (k > j) applied, as dgetf2
    would have stored it."""
    kv = kl + ku
    mn = min(m, n)
    U = np.zeros((mn, n))
    for j in range(n):
        for i in range(max(0, j - kv), min(mn, j + 1)):
            U[i, j] = lu_band[j, kv + i - j]
    L = np.eye(m, mn)
    for j in range(mn):
        v = np.zeros(m)
        for i in range(j + 1, min(m, j + kl + 1)):
            v[i] = lu_band[j, kv + i - j]
        for k in range(j + 1, mn):
            p = ipiv[k] - 1
            v[[k, p]] = v[[p, k]]
        L[j + 1:, j] = v[j + 1:]
    return L, U


def backward_error(A: np.ndarray, X: np.ndarray, Bm: np.ndarray) -> float:
    """max over RHS columns of ||A x - b||_1 / (||A||_1 ||x||_1 n eps)."""
    n = A.shape[0]
    anorm = np.abs(A).sum(axis=0).max()
    R = A @ X - Bm
    worst = 0.0
    for r in range(X.shape[1]):
        xn = np.abs(X[:, r]).sum()
        den = anorm * xn * n * EPS
        eta = np.abs(R[:, r]).sum() / den if den > 0 else (0.0 if np.abs(R[:, r]).sum() == 0 else np.inf)
        worst = max(worst, eta)
    return worst


def same_bits(a: np.ndarray, b: np.ndarray) -> np.ndarray:
    """Elementwise: equal as values (== so +0 == -0) or both NaN."""
    return (a == b) | (np.isnan(a) & np.isnan(b))
