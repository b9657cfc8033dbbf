"""Test-side helpers: dense gate arithmetic (numpy) shared by oracle and GPU tests.

Nothing here is part of the method; it only measures results (G1-G3)."""
import numpy as np


def sym_from_lower(A):
    A = np.asarray(A, dtype=np.float64)
    return np.tril(A) + np.tril(A, -1).T


def band_from_lower(A, b):
    """Full symmetric band matrix from the lower band (diag + b subdiagonals) of A."""
    A = np.asarray(A, dtype=np.float64)
    n = A.shape[0]
    i, j = np.indices((n, n))
    L = np.where((i >= j) & (i - j <= b), A, 0.0)
    return L + np.tril(L, -1).T


def tridiag(d, e):
    return np.diag(d) + np.diag(e, 1) + np.diag(e, -1)


def gates(A, Q, d, e):
    """G1 backward error, G2 orthogonality (both /n, Frobenius)."""
    n = A.shape[0]
    T = tridiag(d, e)
    g1 = np.linalg.norm(A - Q @ T @ Q.T) / (n * np.linalg.norm(A))
    g2 = np.linalg.norm(Q.T @ Q - np.eye(n)) / n
    return g1, g2
