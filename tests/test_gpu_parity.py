"""GPU parity (-m gpu): the CUDA path through the C-ABI vs the CPU oracle, element by element, on the
same seeded inputs, plus the north_star gates G1-G3.

Tolerances: for a quantity computed by a length-K fp64 dot product
the rounding error of either side is <= gamma_K * sum|terms| with gamma_K ~ K u (u = 2^-53); the
kernels and the oracle sum in different orders, so elementwise comparisons use 2 * c * K * u *
(sum of |terms|) with a small constant c.  Reductions (DBBR/BC) compose O(n) such operations on
orthogonal transforms, so their outputs are compared with 64 n u ||A||_F; the gates use the
north_star bounds (1e-14 for G1/G2, 1e-12 ||A||_2 for G3)."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
import trid_gen
from tests.helpers import band_from_lower, gates, sym_from_lower

pytestmark = pytest.mark.gpu
U = 2.0 ** -53


def to_dev(X):
    """logical column-major numpy matrix -> storage tensor (X^T, row-major) on cuda:0."""
    return torch.from_numpy(np.ascontiguousarray(np.asarray(X, dtype=np.float64).T)).to("cuda:0")


def from_dev(S):
    return S.cpu().numpy().T.copy()


# ------------------------------------------------------------------------------------------ syr2k
@pytest.mark.parametrize("m,kk", [(1, 1), (100, 33), (257, 64), (300, 17), (513, 128), (128, 256)])
def test_syr2k_lower_parity(m, kk, dev):
    rng = np.random.default_rng(m * 1000 + kk)
    C = rng.uniform(-1, 1, (m, m))
    Y = rng.uniform(-1, 1, (m, kk))
    Z = rng.uniform(-1, 1, (m, kk))
    ref = oracle.syr2k_lower(C, Y, Z)
    Cd = to_dev(C)
    trid.syr2k_lower(Cd, to_dev(Y), to_dev(Z))
    got = from_dev(Cd)
    il = np.tril_indices(m)
    iu = np.triu_indices(m, 1)
    bound = 2 * 4 * (2 * kk + 1) * U * (np.abs(Y) @ np.abs(Z).T + np.abs(Z) @ np.abs(Y).T + np.abs(C))
    assert np.all(np.abs(got - ref)[il] <= bound[il])
    assert np.array_equal(got[iu], C[iu])      # strict upper untouched, bitwise


@pytest.mark.parametrize("m,kk", [(1000, 100), (512, 64), (258, 37), (2048, 256), (130, 3), (4100, 1024)])
def test_syr2k_tma_staging_bitwise(m, kk, dev, monkeypatch):
    """The TMA producers of the NT engine path (2: one tensor copy per operand and stage from FP64 tensor maps,
    out-of-bounds rows / k zero-filled by the copy engine; 1: one bulk copy per k-row) stage the same tile values
    into the same padded layout as the cp.async producer (0), so the consumers' DMMA order and the result are
    identical bit for bit (ragged row tails m % 128 != 0 and ragged K tails kk % 16 != 0 included); all match the
    oracle."""
    rng = np.random.default_rng(m + 7 * kk)
    C = rng.uniform(-1, 1, (m, m))
    Y = rng.uniform(-1, 1, (m, kk))
    Z = rng.uniform(-1, 1, (m, kk))
    outs = []
    for env in ("2", "1", "0"):
        monkeypatch.setenv("TRID_WS_TMA", env)
        Cd = to_dev(C)
        trid.syr2k_lower(Cd, to_dev(Y), to_dev(Z))
        outs.append(from_dev(Cd))
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], outs[2])
    ref = oracle.syr2k_lower(C, Y, Z)
    il = np.tril_indices(m)
    bound = 2 * 4 * (2 * kk + 1) * U * (np.abs(Y) @ np.abs(Z).T + np.abs(Z) @ np.abs(Y).T + np.abs(C))
    assert np.all(np.abs(outs[0] - ref)[il] <= bound[il])


@pytest.mark.parametrize("n,b", [(1024, 64), (1030, 32), (2101, 64), (1501, 16)])
def test_dbbr_tma_staging_bitwise(n, b, dev, monkeypatch):
    """DBBR with either TMA producer (tensor maps, per-row bulk copies) equals DBBR with the cp.async producer bit
    for bit."""
    A = trid_gen.random_symmetric_np(n, 4242 + n)
    outs = []
    for env in ("2", "1", "0"):
        monkeypatch.setenv("TRID_WS_TMA", env)
        Ad = to_dev(A)
        tau = trid.sbr_dbbr(Ad, b, nb=min(16, b), k=4 * b)
        outs.append((from_dev(Ad), tau.cpu().numpy()))
    for o in outs[1:]:
        assert np.array_equal(outs[0][0], o[0]) and np.array_equal(outs[0][1], o[1])


# ------------------------------------------------------------------------------------------ panel QR
@pytest.mark.parametrize("m,w", [(224, 32), (1000, 64), (5000, 64), (64, 64), (40, 64), (33, 8), (7000, 128),
                                 (3000, 256), (2, 4)])
def test_panel_qr_parity(m, w, dev):
    rng = np.random.default_rng(m + 7 * w)
    P = rng.uniform(-1, 1, (m, w))
    Po, tau_o = oracle.panel_qr(P)
    kk = min(m, w)
    Pd = to_dev(P)
    tau, T, Y = trid.panel_qr(Pd)
    got = from_dev(Pd)
    scale = np.linalg.norm(P)
    tol = 64 * m * U * scale
    assert np.max(np.abs(got - Po)) <= tol
    assert np.max(np.abs(tau.cpu().numpy() - tau_o)) <= 64 * m * U
    # Y = V explicit, and Y T equals the paper's WY recurrence W
    Yl = from_dev(Y)[:, :kk]
    Vu = np.tril(Po, -1)[:, :kk] + np.eye(m, kk)
    assert np.max(np.abs(Yl - Vu)) <= tol
    W_o = oracle.wy(Po[:, :kk], tau_o)
    Tl = from_dev(T)[:kk, :kk]
    assert np.allclose(np.triu(Tl), Tl)
    assert np.max(np.abs(Vu @ Tl - W_o)) <= 64 * m * U * np.max(np.abs(W_o))


@pytest.mark.parametrize("m,w,kind", [(5000, 64, "parallel"), (5000, 64, "near"), (1000, 32, "parallel"),
                                      (32704, 64, "near"), (700, 16, "zero")])
def test_panel_qr_dependent_columns(m, w, kind, dev):
    """Columns (nearly) parallel to their left neighbour make the pair kernel's look-ahead norm a cancelling
    difference; it must fall back to one reflector per reduction there.  Checked by backward error: the Householder
    product Q (from V, tau) is orthogonal and Q R reproduces the panel, both to O(m u) (the reflectors themselves
    are ill-conditioned here, so no element parity)."""
    rng = np.random.default_rng(m + w)
    P = rng.uniform(-1, 1, (m, w))
    if kind == "parallel":
        P[:, 1] = 2.0 * P[:, 0]
        P[:, 9] = -P[:, 8]
        P[:, w - 1] = 0.5 * P[:, w - 2]
    elif kind == "near":
        P[:, 1] = P[:, 0] * (1 + 1e-9) + 1e-12 * rng.uniform(-1, 1, m)
        P[:, 6] = P[:, 5] + 1e-7 * rng.uniform(-1, 1, m)
    else:
        P[:, 3] = 0.0
        P[:, 4] = 0.0
    Pd = to_dev(P)
    tau, T, Y = trid.panel_qr(Pd)
    got = from_dev(Pd)
    kk = min(m, w)
    tau = tau.cpu().numpy()
    V = np.tril(got, -1)[:, :kk] + np.eye(m, kk)
    R = np.triu(got)[:kk, :]
    E = np.eye(m, kk)
    Q = E.copy()
    for j in range(kk - 1, -1, -1):      # Q = H_0 ... H_{kk-1} applied to the first kk unit vectors
        v = V[:, j]
        Q -= tau[j] * np.outer(v, v @ Q)
    assert np.linalg.norm(Q.T @ Q - np.eye(kk)) <= 64 * m * U
    assert np.linalg.norm(Q @ R - P) <= 64 * m * U * np.linalg.norm(P)
    Tl = from_dev(T)[:kk, :kk]
    Qt = E - V @ (Tl @ (V.T @ E))
    assert np.linalg.norm(Qt - Q) <= 64 * m * U


# ------------------------------------------------------------------------------------------ Z builder
@pytest.mark.parametrize("m,w", [(200, 32), (1000, 64), (3000, 64), (700, 16), (513, 128)])
def test_zy_parity(m, w, dev):
    A = trid_gen.random_symmetric_np(m, 77 + m)
    rng = np.random.default_rng(w)
    Pn = rng.uniform(-1, 1, (m, w))
    V, tau = oracle.panel_qr(Pn)
    Y = np.tril(V, -1) + np.eye(m, w)
    W = oracle.wy(V, tau)
    ref = oracle.zy(A, W, Y)
    # the upper triangle of the logical A is garbage: the kernel must never read it
    Ag = np.tril(A) + np.triu(np.full((m, m), np.nan), 1)
    got = from_dev(trid.zy(to_dev(Ag), to_dev(W), to_dev(Y)))
    assert np.all(np.isfinite(got))
    absX = np.abs(A) @ np.abs(W)
    absS = np.abs(W).T @ absX
    bound = 2 * 8 * (m + w) * U * (absX + np.abs(Y) @ absS)
    assert np.all(np.abs(got - ref) <= bound)


# ------------------------------------------------------------------------------------------ DBBR
@pytest.mark.parametrize("n,b,k", [(256, 32, 32), (256, 32, 64), (256, 32, 128), (256, 32, 256), (300, 32, 96),
                                   (513, 16, 64), (257, 64, 128), (100, 8, 24), (40, 4, 8), (1000, 64, 256),
                                   (700, 128, 256), (900, 256, 512), (600, 96, 192)])
def test_dbbr_parity(n, b, k, dev):
    A = trid_gen.random_symmetric_np(n, 1001)
    Ao, to = oracle.dbbr(A, b, k)
    Ad = to_dev(A)
    tau1 = trid.sbr_dbbr(Ad, b, nb=min(8, b), k=k)
    got = from_dev(Ad)
    tol = 64 * n * U * np.linalg.norm(A)
    assert np.max(np.abs(np.tril(got) - np.tril(Ao))) <= tol
    assert np.max(np.abs(tau1.cpu().numpy() - to)) <= 64 * n * U * 16
    assert np.array_equal(np.triu(got, 1), np.triu(A, 1))   # strict upper never written


def test_dbbr_band_input_unchanged(dev):
    n, b = 200, 16
    B = band_from_lower(trid_gen.random_symmetric_np(n, 5), b)
    Ad = to_dev(B)
    tau1 = trid.sbr_dbbr(Ad, b, nb=8, k=64)
    assert torch.all(tau1 == 0)
    assert np.array_equal(np.tril(from_dev(Ad)), np.tril(B))


# ------------------------------------------------------------------------------------------ BC
@pytest.mark.parametrize("n,b", [(256, 32), (300, 32), (257, 64), (200, 8), (129, 2), (64, 63), (50, 100),
                                 (513, 128), (300, 256), (1000, 64)])
def test_bulge_chase_parity(n, b, dev):
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 2 * n + b), min(b, n - 1))
    d_o, e_o, V_o, t_o = oracle.bc_naive(Bm, b)
    d, e, V2, tau2 = trid.bulge_chase(to_dev(Bm), b)
    tol = 64 * n * U * np.linalg.norm(Bm)
    assert np.max(np.abs(d.cpu().numpy() - d_o)) <= tol
    assert np.max(np.abs(e.cpu().numpy() - e_o), initial=0) <= tol
    tot = oracle.bc_total_steps(n, b)
    assert V2.numel() == tot * b and tau2.numel() == tot
    assert np.max(np.abs(tau2.cpu().numpy() - t_o), initial=0) <= 1e-9
    assert np.max(np.abs(V2.cpu().numpy() - V_o), initial=0) <= 1e-9


@pytest.mark.parametrize("variant", ["6", "7"])
def test_bulge_chase_b64_variants(variant, dev, monkeypatch):
    """The B=64 chase (6: bc_v6 (default), 7: bc_v6 in CTA clusters with DSMEM forwarding) against the oracle
    (both the Alg. 2 grouping O2b and the R7 grouping O2c), bitwise reproducible."""
    monkeypatch.setenv("TRID_BC_FORCE", variant)
    n, b = 700, 64
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 99), b)
    d_o, e_o, V_o, t_o = oracle.bc_naive(Bm, b)
    d7, e7, V7, t7 = oracle.bc_r7(Bm, b)
    d, e, V2, tau2 = trid.bulge_chase(to_dev(Bm), b)
    tol = 64 * n * U * np.linalg.norm(Bm)
    for dr, er, Vr in ((d_o, e_o, V_o), (d7, e7, V7)):
        assert np.max(np.abs(d.cpu().numpy() - dr)) <= tol
        assert np.max(np.abs(e.cpu().numpy() - er)) <= tol
        assert np.max(np.abs(V2.cpu().numpy() - Vr)) <= 1e-9
    r1 = [x.clone() for x in trid.bulge_chase(to_dev(Bm), b)]
    for x, y in zip(r1, (d, e, V2, tau2)):
        assert torch.equal(x, y)


@pytest.mark.parametrize("n,b", [(700, 32), (700, 64), (700, 128), (3000, 32), (3000, 64), (3000, 128), (2001, 48),
                                 (12000, 32), (12000, 64), (12000, 128), (1500, 256)])
def test_bulge_chase_serial_equals_parallel_bitwise(n, b, dev, monkeypatch):
    """R9 and include/trid.h's promise: the pipelined chase (148 persistent CTAs, lag-2 progress counters) is bit
    for bit the sweep-major chase.  TRID_BC_SERIAL=1 runs the same kernel on ONE CTA, starting a sweep only after
    its predecessor stored every step (the oracle's order, O2b/O2c with lag 0); the oracle pins the lag rule
    itself (tests/test_oracle.py::test_bc_lag_rule_r9)."""
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 17 + n + b), b)
    Ad = to_dev(Bm)
    par = [x.clone() for x in trid.bulge_chase(Ad, b)]
    monkeypatch.setenv("TRID_BC_SERIAL", "1")
    ser = trid.bulge_chase(Ad, b)
    for x, y in zip(par, ser):
        assert torch.equal(x, y)


@pytest.mark.parametrize("n,b,cl", [(3000, 64, "2"), (3000, 64, "4"), (2500, 32, "2"), (1001, 48, "2"), (300, 64, "8"), (12000, 64, "2")])
def test_bulge_chase_cluster_forwarding_bitwise(n, b, cl, dev, monkeypatch):
    """The cluster variant (sweep s+1 fed from sweep s's shared memory) moves data differently but computes the
    same expressions in the same order: its output equals the single-CTA chase's bit for bit (R9)."""
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 5 + n), b)
    monkeypatch.setenv("TRID_BC_FORCE", "6")
    ref = [x.clone() for x in trid.bulge_chase(to_dev(Bm), b)]
    monkeypatch.setenv("TRID_BC_FORCE", "7")
    monkeypatch.setenv("TRID_BC_CLUSTER", cl)
    got = trid.bulge_chase(to_dev(Bm), b)
    for x, y in zip(ref, got):
        assert torch.equal(x, y)


@pytest.mark.parametrize("env", [("TRID_BC_FS", "1"), ("TRID_BC_FS", "32"), ("TRID_BC_OPT", "0"), ("TRID_BC_OPT", "1"), ("TRID_BC_OPT", "2"), ("TRID_BC_OPT", "8"), ("TRID_BC_OPT", "31"),
                                 ("TRID_BC_OPT", "4"), ("TRID_BC_OPT", "7")])
def test_bulge_chase_handoff_options_bitwise(env, dev, monkeypatch):
    """Counter layout (TRID_BC_FS) and hand-off options (TRID_BC_OPT) change only how data and progress move
    between CTAs, never the arithmetic: the chase output is bitwise that of the default (R9)."""
    n, b = 3000, 64
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 123), b)
    ref = [x.clone() for x in trid.bulge_chase(to_dev(Bm), b)]
    monkeypatch.setenv(*env)
    got = trid.bulge_chase(to_dev(Bm), b)
    for x, y in zip(ref, got):
        assert torch.equal(x, y)


def test_bulge_chase_bitwise_deterministic(dev):
    n, b = 2000, 32
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 11), b)
    Ad = to_dev(Bm)
    r1 = [x.clone() for x in trid.bulge_chase(Ad, b)]
    r2 = [x.clone() for x in trid.bulge_chase(Ad, b)]
    for x, y in zip(r1, r2):
        assert torch.equal(x, y)


def test_bulge_chase_noop_cases(dev):
    n = 100
    T = trid_gen.toeplitz121(n) + np.diag(np.linspace(0, 1, n))
    for b in [1, 2, 7]:
        d, e, V2, tau2 = trid.bulge_chase(to_dev(T), b)
        assert np.array_equal(d.cpu().numpy(), np.diag(T)) and np.array_equal(e.cpu().numpy(), np.diag(T, -1))
        if tau2 is not None and tau2.numel():
            assert torch.all(tau2 == 0)
    d, e, V2, tau2 = trid.bulge_chase(to_dev(T), 4, want_vectors=False)
    assert V2 is None and np.array_equal(d.cpu().numpy(), np.diag(T))


# ------------------------------------------------------------------------------------------ both stages
@pytest.mark.parametrize("n,b,k", [(256, 32, 32), (256, 32, 256), (256, 32, 1024), (300, 32, 64), (513, 64, 128),
                                   (1000, 16, 128), (1024, 64, 1024), (700, 128, 256), (800, 256, 512)])
def test_two_stage_gates(n, b, k, dev):
    A = trid_gen.random_symmetric_np(n, 1001 + n)
    d_o, e_o, Ao, t1o, V_o, t2o = oracle.tridiagonalize(A, b, k)
    Ad = to_dev(A)
    d, e, tau1, V2, tau2 = trid.sytrd_2stage(Ad, b, nb=min(8, b), k=k)
    Aout = from_dev(Ad)
    d, e = d.cpu().numpy(), e.cpu().numpy()
    Q = oracle.form_q(n, b, Aout, tau1.cpu().numpy(), V2.cpu().numpy(), tau2.cpu().numpy())
    g1, g2 = gates(A, Q, d, e)
    assert g1 <= 1e-14 and g2 <= 1e-14, (g1, g2)
    w = oracle.sturm_eig(d, e)
    w_o = oracle.sturm_eig(d_o, e_o)
    norm2 = np.max(np.abs(w_o))
    assert np.max(np.abs(w - w_o)) <= 1e-12 * norm2
    # elementwise diagnostic vs the oracle's signed T (same reflector convention on both sides)
    tol = 64 * n * U * np.linalg.norm(A)
    assert np.max(np.abs(d - d_o)) <= tol and np.max(np.abs(e - e_o)) <= tol


def test_two_stage_trivial_sizes(dev):
    for n, b in [(1, 1), (2, 1), (2, 4), (3, 1), (3, 2), (5, 4), (6, 32)]:
        A = trid_gen.random_symmetric_np(n, 3)
        d, e, tau1, V2, tau2 = trid.sytrd_2stage(to_dev(A), b)
        d_o, e_o, *_ = oracle.tridiagonalize(A, b, None)
        assert np.allclose(d.cpu().numpy(), d_o, atol=1e-13) and np.allclose(e.cpu().numpy(), e_o, atol=1e-13)


def test_two_stage_toeplitz_spectrum(dev):
    n, b = 1024, 32
    A, lam = trid_gen.clustered_symmetric(n, 4001, kind="toeplitz", device="cuda:0")
    d, e, *_ = trid.sytrd_2stage(A, b, nb=8, k=256)
    w = oracle.sturm_eig(d.cpu().numpy(), e.cpu().numpy())
    assert np.max(np.abs(w - lam)) <= 1e-12 * 4
