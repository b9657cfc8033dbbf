"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (-m gpu).

Q is formed on the GPU by the two back-transformation kernels only in test_exact_gates_timed_input_n32768 (the
timed input, exact G1/G2); the other full-size cases check:
  * G3 on prescribed-spectrum inputs (trid_gen.clustered_symmetric: the 1-2-1 Toeplitz spectrum in closed
    form, or 32 tight clusters), eigenvalues of T sampled one by one with the oracle's Sturm count
    (bisection to full precision), against the known eigenvalues: within 1e-12 ||A||_2;
  * G1/G2 with 16 Hutchinson probes through the returned reflectors (tests/qapply.py): <= 1e-14;
  * the stage split is checked too: the band after stage 1 has the input's spectrum (sampled)."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
import trid_gen
from tests.qapply import probe_gates

pytestmark = pytest.mark.gpu


def sampled_eigs(d, e, idx):
    """k-th smallest eigenvalues of tridiag(e, d, e) for k in idx, each by bisection on the oracle's Sturm
    count (Gershgorin start, stop at width <= 2 eps max(|lo|, |hi|))."""
    g = np.abs(np.concatenate([[0.0], e])) + np.abs(np.concatenate([e, [0.0]]))
    lo0, hi0 = float(np.min(d - g)), float(np.max(d + g))
    out = []
    for k in idx:
        lo, hi = lo0, hi0
        while hi - lo > 2 * np.finfo(float).eps * max(abs(lo), abs(hi), 1e-300):
            mid = 0.5 * (lo + hi)
            if mid <= lo or mid >= hi:
                break
            if oracle.sturm_count(d, e, mid) > k:
                hi = mid
            else:
                lo = mid
        out.append(0.5 * (lo + hi))
    return np.array(out)


@pytest.mark.parametrize("n,b,nb,k,kind,seed", [
    (8192, 64, 16, 1024, "toeplitz", 2001),       # configs[1]
    (32768, 64, 16, 1024, "toeplitz", 3001),      # configs[2], the bench headline launch configuration
    (16384, 128, 16, 1024, "clusters", 5001),     # configs[4] (b sweep, widest default-path band)
])
def test_fullsize_gates(n, b, nb, k, kind, seed, dev):
    A, lam = trid_gen.clustered_symmetric(n, seed, kind=kind, device="cuda:0")
    A0 = A.clone()
    d, e, tau1, V2, tau2 = trid.sytrd_2stage(A, b, nb=nb, k=k)
    torch.cuda.synchronize()
    norm2 = float(np.max(np.abs(lam)))
    dn, en = d.cpu().numpy(), e.cpu().numpy()
    rng = np.random.default_rng(seed)
    idx = np.unique(np.concatenate([[0, n - 1], rng.integers(0, n, 62)]))
    w = sampled_eigs(dn, en, idx)
    assert np.max(np.abs(w - lam[idx])) <= 1e-12 * norm2
    g1, g2 = probe_gates(A0, A, d, e, tau1, V2, tau2, b, p=16)
    assert g1 <= 1e-14 and g2 <= 1e-14, (g1, g2)


def test_timed_input_gates(dev):
    """The exact input bench.py times (configs[2]: n = 32768 random symmetric, seed 3001, b = 64, nb = 16,
    k = 1024) in the bench's launch configuration: G1/G2 with 16 Hutchinson probes through the returned
    reflectors, and G3 for 64 sampled eigenvalues of T (oracle Sturm count) and all n (trid_stebz) against MAGMA's
    dsyevd of A (torch.linalg.eigvalsh)."""
    n, b, nb, k = 32768, 64, 16, 1024
    A = trid_gen.random_symmetric(n, 3001, device="cuda:0")
    # cuSOLVER's syevd rejects n = 32768 (32-bit workspace query); MAGMA's hybrid dsyevd takes it (~90 s)
    prev = torch.backends.cuda.preferred_linalg_library()
    try:
        torch.backends.cuda.preferred_linalg_library("magma")
        lam = torch.linalg.eigvalsh(A).cpu().numpy()
    finally:
        torch.backends.cuda.preferred_linalg_library(prev)
    A0 = A.clone()
    d, e, tau1, V2, tau2 = trid.sytrd_2stage(A, b, nb=nb, k=k)
    torch.cuda.synchronize()
    norm2 = float(np.max(np.abs(lam)))
    rng = np.random.default_rng(3001)
    idx = np.unique(np.concatenate([[0, n - 1], rng.integers(0, n, 62)]))
    w = sampled_eigs(d.cpu().numpy(), e.cpu().numpy(), idx)
    assert np.max(np.abs(w - lam[idx])) <= 1e-12 * norm2
    # all n eigenvalues of T by the GPU bisection (trid_stebz) against syevd
    wall = trid.stebz(d, e).cpu().numpy()
    assert np.max(np.abs(wall - lam)) <= 1e-12 * norm2
    g1, g2 = probe_gates(A0, A, d, e, tau1, V2, tau2, b, p=16)
    assert g1 <= 1e-14 and g2 <= 1e-14, (g1, g2)


def test_fullsize_random_b_sweep_spectrum(dev):
    """configs[4]: n = 16384 random symmetric, b in {32, 64, 256}: eigenvalues of T (sampled) equal those of
    the input (cuSOLVER syevd through torch as the independent reference for a random matrix)."""
    n = 16384
    A = trid_gen.random_symmetric(n, 5001, device="cuda:0")
    lam = torch.linalg.eigvalsh(A).cpu().numpy()
    norm2 = float(np.max(np.abs(lam)))
    rng = np.random.default_rng(5)
    idx = np.unique(np.concatenate([[0, n - 1], rng.integers(0, n, 30)]))
    for b in (32, 64, 256):
        Ab = A.clone()
        d, e, *_ = trid.sytrd_2stage(Ab, b, nb=min(16, b), k=1024, want_vectors=False)
        w = sampled_eigs(d.cpu().numpy(), e.cpu().numpy(), idx)
        assert np.max(np.abs(w - lam[idx])) <= 1e-12 * norm2, b


def test_probe_gates_detect_a_wrong_reflector(dev):
    """The probe estimator is sensitive: flipping one BC scalar breaks G1 by orders of magnitude."""
    n, b = 2048, 64
    A = trid_gen.random_symmetric(n, 7, device="cuda:0")
    A0 = A.clone()
    d, e, tau1, V2, tau2 = trid.sytrd_2stage(A, b, nb=16, k=256)
    g1, g2 = probe_gates(A0, A, d, e, tau1, V2, tau2, b)
    assert g1 <= 1e-14 and g2 <= 1e-14
    tau2[len(tau2) // 2] *= -1.0
    g1b, g2b = probe_gates(A0, A, d, e, tau1, V2, tau2, b)
    assert g1b > 1e-10


@pytest.mark.parametrize("n,b,seed,kind", [(32768, 64, 3001, "random"), (32768, 128, 3001, "random"),
                                           (49152, 64, 4001, "clusters")])
def test_exact_gates_timed_input_n32768(n, b, seed, kind, dev):
    """The north_star gates G1/G2 EXACTLY (no probes) on the inputs bench.py times (BASELINE configs[2]: n = 32768
    random symmetric, seed 3001, b = 64 and 128; configs[3]: n = 49152 clustered spectrum, seed 4001; nb = 16,
    k = 1024): Q = Q1 Q2 formed on the GPU by the two back-transformation kernels, then
    ||A - Q T Q^T||_F / (n ||A||_F) and ||Q^T Q - I||_F / n with cuBLAS DGEMMs (torch.matmul, test-side).  T is
    applied as a tridiagonal (column shifts), never formed."""
    nb, k = 16, 1024
    if kind == "clusters":
        A, _ = trid_gen.clustered_symmetric(n, seed, kind="clusters", device="cuda:0")
    else:
        A = trid_gen.random_symmetric(n, seed, device="cuda:0")
    A0 = A.clone()
    d, e, tau1, V2, tau2 = trid.sytrd_2stage(A, b, nb=nb, k=k)
    Qs = torch.eye(n, dtype=torch.float64, device="cuda:0")   # storage of the column-major identity
    trid.bc_backtransform(V2, tau2, n, b, Qs)
    del V2, tau2
    trid.sbr_backtransform(A, tau1, b, Qs)
    del A
    Q = Qs.mT                                                  # logical Q (a view)
    QT = Q * d                                                 # Q T: column j = d_j q_j + e_{j-1} q_{j-1} + e_j q_{j+1}
    QT[:, 1:] += Q[:, :-1] * e
    QT[:, :-1] += Q[:, 1:] * e
    R = torch.matmul(QT, Q.T)
    del QT
    A0l = A0.mT                                                # logical A (symmetric: the same matrix)
    nA = float(torch.linalg.norm(A0l))
    R.sub_(A0l)
    g1 = float(torch.linalg.norm(R)) / (n * nA)
    del R, A0, A0l
    G = torch.matmul(Q.T, Q)
    G.diagonal().sub_(1.0)
    g2 = float(torch.linalg.norm(G)) / n
    assert g1 <= 1e-14 and g2 <= 1e-14, (g1, g2)
    print(f"n={n} b={b} seed {seed} {kind}: exact G1={g1:.3e} G2={g2:.3e}")
