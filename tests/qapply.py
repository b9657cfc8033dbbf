"""Test-side application of Q = Q1 Q2 to a block of probe vectors (torch, on the GPU) — measurement only.

Used for the north_star gates at bench sizes (n >= 8192) where Q cannot be formed: G1 and G2 are estimated
with Hutchinson probes, E||E x||^2 = ||E||_F^2 for x ~ N(0, I).  The reflector layouts are the
C-ABI's (include/trid.h): SBR vector of column c below A's band (unit entry at row c+b), scalar tau1[c];
BC step (s, m) vector at V2[(S(s)+m)*b : +b] acting on rows s+1+m*b ..., scalar tau2[S(s)+m].
Q1 = H_0 H_1 ... H_{n-b-2};  Q2 = product of the BC reflectors in sweep-major order; Q = Q1 Q2."""
import torch


def _sweep_offsets(n, b):
    s = torch.arange(0, max(n - 2, 0), dtype=torch.int64)
    steps = (n - 3 - s) // b + 1
    off = torch.zeros_like(steps)
    off[1:] = torch.cumsum(steps, 0)[:-1]
    return steps.tolist(), off.tolist()


def apply_q2(X, V2, tau2, n, b, transpose=False):
    """X (n x p, column-major logical = torch (n, p) row-major) <- Q2 X (or Q2^T X).  Reflectors of one
    sweep act on disjoint row blocks of length b (zero padded), so a sweep is one batched update."""
    p = X.shape[1]
    Xp = torch.cat([X, torch.zeros((b + 1, p), dtype=X.dtype, device=X.device)])
    steps, off = _sweep_offsets(n, b)
    order = range(len(steps)) if transpose else range(len(steps) - 1, -1, -1)
    for s in order:
        nst, o = steps[s], off[s]
        V = V2[o * b:(o + nst) * b].view(nst, b)
        t = tau2[o:o + nst]
        Xs = Xp[s + 1:s + 1 + nst * b].view(nst, b, p)
        w = torch.einsum("mb,mbp->mp", V, Xs)
        Xs -= (t[:, None, None] * V[:, :, None]) * w[:, None, :]
    return Xp[:n]


def apply_q1(X, S, tau1, n, b, transpose=False):
    """X <- Q1 X (or Q1^T X); S is the storage tensor of A after stage 1 (S[c, i] = A(i, c))."""
    X = X.clone()
    last = n - b - 2
    cs = range(0, last + 1) if transpose else range(last, -1, -1)
    tau = tau1.tolist()
    for c in cs:
        t = tau[c]
        if t == 0.0:
            continue
        r0 = c + b
        v = torch.cat([torch.ones(1, dtype=X.dtype, device=X.device), S[c, r0 + 1:n]])
        w = v @ X[r0:n]
        X[r0:n] -= t * torch.outer(v, w)
    return X


def apply_q(X, S, tau1, V2, tau2, n, b, transpose=False):
    if transpose:
        return apply_q2(apply_q1(X, S, tau1, n, b, True), V2, tau2, n, b, True)
    return apply_q1(apply_q2(X, V2, tau2, n, b, False), S, tau1, n, b, False)


def tridiag_mm(d, e, X):
    Y = d[:, None] * X
    Y[:-1] += e[:, None] * X[1:]
    Y[1:] += e[:, None] * X[:-1]
    return Y


def probe_gates(A, S, d, e, tau1, V2, tau2, b, p=8, seed=0):
    """Hutchinson estimates of G1 = ||A - Q T Q^T||_F / (n ||A||_F) and G2 = ||Q^T Q - I||_F / n.
    A: the original symmetric matrix (torch (n, n), both triangles)."""
    n = A.shape[0]
    g = torch.Generator(device=A.device).manual_seed(seed)
    X = torch.randn((n, p), dtype=torch.float64, device=A.device, generator=g)
    QtX = apply_q(X, S, tau1, V2, tau2, n, b, transpose=True)
    E1 = A @ X - apply_q(tridiag_mm(d, e, QtX), S, tau1, V2, tau2, n, b)
    QX = apply_q(X, S, tau1, V2, tau2, n, b)
    E2 = apply_q(QX, S, tau1, V2, tau2, n, b, transpose=True) - X
    scale = p ** 0.5
    g1 = float(torch.linalg.norm(E1)) / scale / (n * float(torch.linalg.norm(A)))
    g2 = float(torch.linalg.norm(E2)) / scale / n
    return g1, g2
