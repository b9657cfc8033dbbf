"""Pins for the CPU oracle (-m "not gpu").  Every oracle routine is checked against something other
than itself: LAPACK routines it must reduce to (scipy), closed forms, brute-force products of the
individual reflectors, and invariants (spectrum, orthogonality, structure).  Paper citations are
PAPER.md lines (P:<line>)."""
import math

import numpy as np
import pytest
import scipy.linalg as sla
from scipy.linalg import lapack

import oracle
import trid_gen
from tests.helpers import band_from_lower, gates, sym_from_lower, tridiag

EPS = np.finfo(np.float64).eps


def rand_sym(n, seed):
    return trid_gen.random_symmetric_np(n, seed)


# ---------------------------------------------------------------------------- inputs
def test_generator_numpy_torch_bit_identical():
    import torch
    for n, seed in [(1, 3), (17, 1001), (64, 2001)]:
        a = trid_gen.random_symmetric_np(n, seed)
        t = trid_gen.random_symmetric(n, seed, chunk=5).numpy()
        assert np.array_equal(a.view(np.uint64), t.view(np.uint64))
        assert np.array_equal(a, a.T)
        assert a.min() >= -1.0 and a.max() < 1.0
    # distinct seeds give distinct matrices
    assert not np.array_equal(trid_gen.random_symmetric_np(8, 1), trid_gen.random_symmetric_np(8, 2))
    # uniform moments (mean 0, var 1/3) on a big sample
    a = trid_gen.random_symmetric_np(300, 5)
    assert abs(a.mean()) < 0.01 and abs(a.var() - 1 / 3) < 0.01
    del torch


def test_clustered_generator_spectrum():
    A, lam = trid_gen.clustered_symmetric(96, 4001, kind="toeplitz")
    A = A.numpy()
    w = np.linalg.eigvalsh(sym_from_lower(A))
    assert np.allclose(w, trid_gen.toeplitz121_eigs(96), atol=1e-13)
    A, lam = trid_gen.clustered_symmetric(128, 4001, kind="clusters")
    w = np.linalg.eigvalsh(sym_from_lower(A.numpy()))
    assert np.allclose(w, lam, atol=1e-13)
    assert len(np.unique(np.round(lam, 6))) == 32


# ---------------------------------------------------------------------------- house (R1)
@pytest.mark.parametrize("x", [
    [3.0, 4.0], [-3.0, 4.0, 12.0], [0.5, -0.25, 0.125, 2.0], [-0.0, 1.0], [0.0, 1e-3, -2.0],
    [2.0, 0.0, 0.0], [-2.0, 0.0], [7.0], list(np.linspace(-1, 1, 33)),
])
def test_house_matches_lapack_dlarfg(x):
    x = np.array(x, dtype=np.float64)
    v, tau, beta = oracle.house(x)
    n = len(x)
    if n > 1:
        alpha_l, xl, tau_l = lapack.dlarfg(n, x[0], x[1:].copy())
        assert beta == pytest.approx(alpha_l, rel=4 * EPS, abs=0)
        assert tau == pytest.approx(tau_l, rel=4 * EPS, abs=1e-300)
        assert np.allclose(v[1:], xl, rtol=4 * EPS, atol=0)
    H = np.eye(n) - tau * np.outer(v, v)
    y = H @ x
    assert abs(y[0] - beta) <= 4 * EPS * max(1.0, abs(beta))
    assert np.all(np.abs(y[1:]) <= 8 * EPS * np.linalg.norm(x))
    assert abs(abs(beta) - np.linalg.norm(x)) <= 4 * EPS * np.linalg.norm(x)
    assert tau == 0.0 or 1.0 <= tau <= 2.0
    assert np.allclose(H @ H.T, np.eye(n), atol=8 * EPS)


def test_house_no_reflection_when_tail_zero():
    v, tau, beta = oracle.house([-2.0, 0.0, 0.0])
    assert tau == 0.0 and beta == -2.0


# ---------------------------------------------------------------------------- O1 sytd2
@pytest.mark.parametrize("n", [2, 3, 8, 33, 100])
def test_sytd2_matches_lapack_dsytrd_signed(n):
    A = rand_sym(n, 1001 + n)
    d, e, tau, _ = oracle.sytd2(A)
    _, dl, el, taul, info = lapack.dsytrd(A, lower=1)
    assert info == 0
    scale = np.linalg.norm(A, 2)
    assert np.max(np.abs(d - dl)) <= 1e-13 * scale
    assert np.max(np.abs(e - el), initial=0) <= 1e-13 * scale
    assert np.max(np.abs(tau - taul), initial=0) <= 1e-12


def test_sytd2_tridiagonal_input_unchanged_bitwise():
    n = 40
    T = trid_gen.toeplitz121(n) * 1.5 + np.diag(np.arange(n) * 0.01)
    d, e, tau, _ = oracle.sytd2(T)
    assert np.array_equal(d, np.diag(T)) and np.array_equal(e, np.diag(T, -1))
    assert np.all(tau == 0.0)


# ---------------------------------------------------------------------------- Sturm / Jacobi (G3 tools)
@pytest.mark.parametrize("n", [1, 2, 5, 64, 257])
def test_sturm_closed_form_toeplitz(n):
    d = np.full(n, 2.0)
    e = np.full(n - 1, -1.0)
    w = oracle.sturm_eig(d, e)
    assert np.max(np.abs(w - trid_gen.toeplitz121_eigs(n))) <= 8 * EPS * 4


def test_sturm_matches_lapack_dstebz_and_counts():
    n = 200
    rng = np.random.default_rng(7)
    d, e = rng.standard_normal(n), rng.standard_normal(n - 1)
    w = oracle.sturm_eig(d, e)
    wl = sla.eigvalsh_tridiagonal(d, e)
    assert np.max(np.abs(w - wl)) <= 1e-13 * np.max(np.abs(wl))
    for x in [-1.0, 0.0, 0.3, 2.5]:
        assert oracle.sturm_count(d, e, x) == int(np.sum(wl < x))


def test_jacobi_closed_form_and_numpy():
    n = 24
    w, sweeps = oracle.jacobi_eig(trid_gen.toeplitz121(n))
    assert np.max(np.abs(w - trid_gen.toeplitz121_eigs(n))) <= 8 * n * EPS * 4   # ~ n eps ||A||_2
    A = rand_sym(50, 9)
    w, _ = oracle.jacobi_eig(A)
    assert np.max(np.abs(w - np.linalg.eigvalsh(A))) <= 1e-13 * np.linalg.norm(A, 2)


# ---------------------------------------------------------------------------- panel QR / WY / Eq. (1)
@pytest.mark.parametrize("m,w", [(40, 8), (224, 32), (9, 12), (5, 5), (33, 1)])
def test_panel_qr_matches_lapack_dgeqrf(m, w):
    P = np.asfortranarray(np.random.default_rng(m * w).standard_normal((m, w)))
    Po, tau = oracle.panel_qr(P)
    ql, taul, _, info = lapack.dgeqrf(P.copy())
    assert info == 0
    kk = min(m, w)
    assert np.allclose(Po, ql, rtol=0, atol=1e-13 * np.linalg.norm(P))
    assert np.allclose(tau, taul[:kk], atol=1e-13)
    # Q^T P = R with Q the brute-force product of the reflectors
    Q = np.eye(m)
    for t in range(kk):
        v = np.zeros(m); v[t] = 1.0; v[t + 1:] = Po[t + 1:, t]
        Q = Q @ (np.eye(m) - tau[t] * np.outer(v, v))
    R = np.triu(Po[:kk, :]) if m >= w else np.triu(Po)
    assert np.allclose((Q.T @ P)[:R.shape[0]], R, atol=1e-13 * np.linalg.norm(P))


@pytest.mark.parametrize("m,kk", [(50, 8), (100, 32), (7, 7)])
def test_wy_recurrence_equals_reflector_product(m, kk):
    P = np.asfortranarray(np.random.default_rng(m + kk).standard_normal((m, kk)))
    V, tau = oracle.panel_qr(P)
    W = oracle.wy(V, tau)
    Vu = np.tril(V, -1)[:, :kk] + np.eye(m, kk)
    H = np.eye(m)
    for t in range(kk):
        H = H @ (np.eye(m) - tau[t] * np.outer(Vu[:, t], Vu[:, t]))
    assert np.allclose(np.eye(m) - W @ Vu.T, H, atol=1e-14 * m)


@pytest.mark.parametrize("m,kk", [(64, 8), (120, 16)])
def test_zy_two_sided_identity(m, kk):
    """Eq. (1): A - Y Z^T - Z Y^T = Q^T A Q for Q = I - W Y^T (holds for any W)."""
    A = rand_sym(m, m)
    P = np.random.default_rng(kk).standard_normal((m, kk))
    V, tau = oracle.panel_qr(P)
    Y = np.tril(V, -1) + np.eye(m, kk)
    W = oracle.wy(V, tau)
    Z = oracle.zy(A, W, Y)
    Q = np.eye(m) - W @ Y.T
    lhs = A - Y @ Z.T - Z @ Y.T
    assert np.allclose(lhs, Q.T @ A @ Q, atol=1e-13 * np.linalg.norm(A))
    # and with an arbitrary (non-orthogonal) W the algebraic identity still holds
    W2 = np.random.default_rng(1).standard_normal((m, kk))
    Z2 = oracle.zy(A, W2, Y)
    Q2 = np.eye(m) - W2 @ Y.T
    assert np.allclose(A - Y @ Z2.T - Z2 @ Y.T, Q2.T @ A @ Q2, atol=1e-12 * np.linalg.norm(A) * kk)


def test_syr2k_lower_vs_numpy_and_upper_untouched():
    m, kk = 70, 13
    rng = np.random.default_rng(3)
    C = np.asfortranarray(rng.standard_normal((m, m)))
    Y, Z = rng.standard_normal((m, kk)), rng.standard_normal((m, kk))
    out = oracle.syr2k_lower(C, Y, Z)
    ref = C - Y @ Z.T - Z @ Y.T
    il = np.tril_indices(m)
    iu = np.triu_indices(m, 1)
    assert np.allclose(out[il], ref[il], atol=1e-13 * kk)
    assert np.array_equal(out[iu], C[iu])


# ---------------------------------------------------------------------------- O2a SBR, Alg. 1 DBBR
def _check_band_reduction(A, Aout, tau1, b):
    n = A.shape[0]
    B = band_from_lower(Aout, b)
    Q1 = oracle.form_q(n, b, Aout, tau1)
    g_orth = np.linalg.norm(Q1.T @ Q1 - np.eye(n)) / n
    g_back = np.linalg.norm(A - Q1 @ B @ Q1.T) / (n * np.linalg.norm(A))
    assert g_orth <= 1e-14 and g_back <= 1e-14, (g_orth, g_back)
    assert np.allclose(np.linalg.eigvalsh(B), np.linalg.eigvalsh(A), atol=1e-12 * np.linalg.norm(A, 2))


@pytest.mark.parametrize("n,b", [(64, 8), (100, 7), (256, 32), (33, 32), (34, 32), (20, 1)])
def test_sbr_naive_reduces_to_band(n, b):
    A = rand_sym(n, 1000 + n + b)
    Aout, tau1 = oracle.sbr_naive(A, b)
    _check_band_reduction(A, Aout, tau1, b)
    assert np.all(tau1[max(n - b - 1, 0):] == 0.0)


def test_sbr_b1_is_lapack_dsytrd():
    A = rand_sym(60, 11)
    Aout, tau1 = oracle.sbr_naive(A, 1)
    _, dl, el, taul, _ = lapack.dsytrd(A, lower=1)
    assert np.allclose(np.diag(Aout), dl, atol=1e-13 * 20) and np.allclose(np.diag(Aout, -1), el, atol=1e-13 * 20)
    assert np.allclose(tau1[:59], taul, atol=1e-12)


def test_sbr_band_input_unchanged_bitwise():
    n, b = 80, 6
    Bm = band_from_lower(rand_sym(n, 5), b)
    Aout, tau1 = oracle.sbr_naive(Bm, b)
    assert np.all(tau1 == 0.0)
    assert np.array_equal(np.tril(Aout), np.tril(Bm))


@pytest.mark.parametrize("n,b,k", [(256, 32, 32), (256, 32, 64), (256, 32, 128), (256, 32, 256),
                                   (100, 8, 24), (101, 8, 64), (64, 16, 64), (45, 4, 12)])
def test_dbbr_equals_naive_sbr(n, b, k):
    """Alg. 1 (DBBR, readings R4) = plain SBR (reflectors and band) for every k."""
    A = rand_sym(n, 1001)
    An, tn = oracle.sbr_naive(A, b)
    Ad, td = oracle.dbbr(A, b, k)
    scale = np.linalg.norm(A)
    assert np.max(np.abs(band_from_lower(Ad, b) - band_from_lower(An, b))) <= 1e-13 * scale
    assert np.max(np.abs(np.tril(Ad) - np.tril(An))) <= 1e-12 * scale
    assert np.max(np.abs(td - tn)) <= 1e-12
    _check_band_reduction(A, Ad, td, b)


# ---------------------------------------------------------------------------- O2b bulge chasing
def test_bc_step_counts():
    assert oracle.bc_total_steps(256, 32) == 1136
    for n, b in [(10, 3), (257, 32), (50, 49), (8192, 64)]:
        assert oracle.bc_total_steps(n, b) == sum((t // b) + 1 for t in range(n - 2))


@pytest.mark.parametrize("n,b", [(40, 4), (64, 8), (33, 5)])
def test_bc_window_equals_full_bitwise(n, b):
    B = band_from_lower(rand_sym(n, n), b)
    d1, e1, V1, t1 = oracle.bc_naive(B, b, full=False)
    d2, e2, V2, t2 = oracle.bc_naive(B, b, full=True)
    assert np.array_equal(d1, d2) and np.array_equal(e1, e2)
    assert np.array_equal(V1, V2) and np.array_equal(t1, t2)


@pytest.mark.parametrize("n", [3, 9, 40])
def test_bc_full_band_is_lapack_dsytrd(n):
    """With b = n-1 every sweep is one step on rows s+1..n-1: exactly dsytd2 (R7 step 0)."""
    A = rand_sym(n, 31 + n)
    d, e, V2, tau2 = oracle.bc_naive(A, n - 1)
    _, dl, el, taul, _ = lapack.dsytrd(A, lower=1)
    assert np.max(np.abs(d - dl)) <= 1e-13 * n and np.max(np.abs(e - el)) <= 1e-13 * n
    assert np.allclose(tau2, taul[: len(tau2)], atol=1e-12)


@pytest.mark.parametrize("n,b", [(64, 8), (100, 7), (256, 32), (50, 2), (17, 16)])
def test_bc_similarity_and_spectrum(n, b):
    B = band_from_lower(rand_sym(n, 2 * n + b), b)
    d, e, V2, tau2 = oracle.bc_naive(B, b)
    Q2 = oracle.form_q(n, b, None, None, V2, tau2)
    g1, g2 = gates(B, Q2, d, e)
    assert g1 <= 1e-14 and g2 <= 1e-14, (g1, g2)
    w = oracle.sturm_eig(d, e)
    assert np.max(np.abs(w - np.linalg.eigvalsh(B))) <= 1e-12 * np.linalg.norm(B, 2)
    assert np.all(np.abs(V2.reshape(-1, b)[:, 0] - 1.0) == 0.0)
    assert np.all((tau2 == 0) | ((tau2 >= 1) & (tau2 <= 2)))


@pytest.mark.parametrize("n,b", [(64, 8), (200, 8), (256, 32), (300, 17), (130, 64), (100, 2), (50, 100)])
def test_bc_r7_grouping_equals_alg2_and_is_a_similarity(n, b):
    """O2c (R7 grouping: the next reflector is generated and left-applied inside the step, lower triangle only)
    computes O2b's reflectors and T up to rounding (amplified by the forward sensitivity of T, R15: a
    diagnostic bound), and is itself an orthogonal similarity (pinned by the gates with its own reflectors, not
    by O2b) with O2b's spectrum."""
    B = band_from_lower(rand_sym(n, 3 + n), min(b, n - 1))
    d, e, V2, tau2 = oracle.bc_naive(B, b)
    d7, e7, V7, t7 = oracle.bc_r7(B, b)
    tol = 1e-9 * np.linalg.norm(B)
    assert np.max(np.abs(d - d7)) <= tol and np.max(np.abs(e - e7), initial=0) <= tol
    assert np.max(np.abs(V2 - V7), initial=0) <= 1e-7 and np.max(np.abs(tau2 - t7), initial=0) <= 1e-7
    w, w7 = oracle.sturm_eig(d, e), oracle.sturm_eig(d7, e7)
    assert np.max(np.abs(w - w7)) <= 1e-12 * np.linalg.norm(B, 2)
    Q2 = oracle.form_q(n, b, None, None, V7, t7)
    g1, g2 = gates(B, Q2, d7, e7)
    assert g1 <= 1e-14 and g2 <= 1e-14, (g1, g2)


@pytest.mark.parametrize("n,b", [(200, 8), (256, 32), (300, 17), (130, 64), (100, 2)])
def test_bc_lag_rule_r9(n, b):
    """Reading R9: the sweeps pipelined in the wavefront order (slot t runs step t - lag*s
    of every sweep, later sweeps first).
      * R7 grouping (the GPU kernels' footprint: a step owns its columns R_m): lag 2 and lag 3 reproduce the
        sweep-major result bit for bit; lag 1 is wrong (O(1) differences).
      * Alg. 2's grouping (the left application of H_m to B_ol inside step m): lag 3 is bitwise
        ("after the first three bulges"); lag 1 is wrong."""
    B = band_from_lower(rand_sym(n, 3 + n), b)
    ref7 = oracle.bc_r7(B, b, 0)
    for lag in (2, 3):
        got = oracle.bc_r7(B, b, lag)
        assert all(np.array_equal(x, y) for x, y in zip(ref7, got)), lag
    bad = oracle.bc_r7(B, b, 1)
    assert np.max(np.abs(bad[0] - ref7[0])) > 1e-3
    ref2 = oracle.bc_naive(B, b)
    got3 = oracle.bc_wavefront(B, b, 3)
    assert all(np.array_equal(x, y) for x, y in zip(ref2, got3))
    bad2 = oracle.bc_wavefront(B, b, 1)
    assert np.max(np.abs(bad2[0] - ref2[0])) > 1e-3


def test_bc_noop_cases_bitwise():
    n = 30
    T = trid_gen.toeplitz121(n) + np.diag(np.linspace(0, 1, n))
    for b in [1, 2, 5]:
        d, e, V2, tau2 = oracle.bc_naive(T, b)
        assert np.array_equal(d, np.diag(T)) and np.array_equal(e, np.diag(T, -1))
        assert tau2 is None or np.all(tau2 == 0.0)
    D = np.diag(np.arange(n, dtype=np.float64))
    d, e, _, _ = oracle.bc_naive(D, 4)
    assert np.array_equal(d, np.arange(n)) and np.all(e == 0.0)


# ---------------------------------------------------------------------------- back-transformations
@pytest.mark.parametrize("n,b,k", [(96, 8, 32), (130, 16, None), (64, 4, 16)])
def test_sbr_backtransform_pins(n, b, k):
    """C <- Q1 C: with C = I it is Q1 as formed by right multiplication in form_q (a different loop order); Q1^T
    undoes Q1; and Q1^T A Q1 is the band stage 1 produced (sec. 4.3)."""
    A = rand_sym(n, 900 + n)
    Aout, tau1 = oracle.dbbr(A, b, k) if k else oracle.sbr_naive(A, b)
    Q1 = oracle.sbr_backtransform(Aout, tau1, b, np.eye(n))
    assert np.max(np.abs(Q1 - oracle.form_q(n, b, Aout, tau1))) <= 1e-14 * n
    C = np.random.default_rng(n).uniform(-1, 1, (n, 7))
    back = oracle.sbr_backtransform(Aout, tau1, b, oracle.sbr_backtransform(Aout, tau1, b, C), trans=True)
    assert np.max(np.abs(back - C)) <= 1e-14 * n
    Bt = oracle.sbr_backtransform(Aout, tau1, b, oracle.sbr_backtransform(Aout, tau1, b, A, trans=True).T, trans=True)
    assert np.max(np.abs(Bt - band_from_lower(Aout, b))) <= 64 * n * EPS * np.linalg.norm(A)


@pytest.mark.parametrize("n,b", [(64, 8), (100, 7), (50, 2), (40, 64)])
def test_bc_backtransform_pins(n, b):
    """C <- Q2 C: with C = I it is form_q's Q2; Q2^T undoes Q2; Q2^T B Q2 = T (the chase's own output)."""
    B = band_from_lower(rand_sym(n, 2 * n + b), min(b, n - 1))
    d, e, V2, tau2 = oracle.bc_naive(B, b)
    if b >= n - 1 or V2 is None or len(V2) == 0:
        return
    Q2 = oracle.bc_backtransform(V2, tau2, b, np.eye(n))
    assert np.max(np.abs(Q2 - oracle.form_q(n, b, None, None, V2, tau2))) <= 1e-14 * n
    C = np.random.default_rng(n).uniform(-1, 1, (n, 5))
    back = oracle.bc_backtransform(V2, tau2, b, oracle.bc_backtransform(V2, tau2, b, C), trans=True)
    assert np.max(np.abs(back - C)) <= 1e-14 * n
    T = oracle.bc_backtransform(V2, tau2, b, oracle.bc_backtransform(V2, tau2, b, B, trans=True).T, trans=True)
    assert np.max(np.abs(T - tridiag(d, e))) <= 64 * n * EPS * np.linalg.norm(B)


# ---------------------------------------------------------------------------- the whole method (G1-G3)
@pytest.mark.parametrize("k", [None, 32, 64, 128, 256])
def test_two_stage_gates_n256(k):
    n, b = 256, 32
    A = rand_sym(n, 1001)
    d, e, Aout, tau1, V2, tau2 = oracle.tridiagonalize(A, b, k)
    Q = oracle.form_q(n, b, Aout, tau1, V2, tau2)
    g1, g2 = gates(A, Q, d, e)
    assert g1 <= 1e-14 and g2 <= 1e-14
    assert np.allclose(Q[:, 0], np.eye(n)[:, 0])   # every reflector acts on rows >= 1
    w = oracle.sturm_eig(d, e)
    wj, _ = oracle.jacobi_eig(A)
    assert np.max(np.abs(w - wj)) <= 1e-12 * np.max(np.abs(wj))


def test_two_stage_toeplitz_closed_form_under_similarity():
    n, b = 128, 16
    A, lam = trid_gen.clustered_symmetric(n, 77, kind="toeplitz")
    A = sym_from_lower(A.numpy())
    d, e, *_ = oracle.tridiagonalize(A, b, 64)
    w = oracle.sturm_eig(d, e)
    assert np.max(np.abs(w - trid_gen.toeplitz121_eigs(n))) <= 1e-12 * 4


def test_two_stage_vs_one_stage_diagnostic():
    """T is unique up to e-signs (implicit-Q theorem); at n = 64 d and |e| agree closely."""
    n, b = 64, 8
    A = rand_sym(n, 4)
    d2, e2, *_ = oracle.tridiagonalize(A, b, 16)
    d1, e1, _, _ = oracle.sytd2(A)
    assert np.max(np.abs(d1 - d2)) < 1e-9 and np.max(np.abs(np.abs(e1) - np.abs(e2))) < 1e-9
    assert math.isfinite(float(np.sum(d2)))
