"""GPU back-transformations (include/trid.h trid_sbr_backtransform / trid_bc_backtransform)
against the oracle's one-reflector-at-a-time definitions, on the reflectors the GPU itself produced (-m gpu), and
the north_star gates G1/G2 evaluated EXACTLY at the bench size n = 8192 with Q formed by the two kernels.

Tolerance: every output entry is an inner product chain through at most n reflectors of norm-preserving updates:
|dC| <= 64 n u max_j ||C(:, j)||_2."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
import trid_gen
from tests.helpers import band_from_lower

pytestmark = pytest.mark.gpu
U = 2.0 ** -53


def to_dev(X):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(X, dtype=np.float64).T)).to("cuda:0")


def from_dev(S):
    return S.cpu().numpy().T.copy()


@pytest.mark.parametrize("n,b,k,kbt", [(256, 32, 64, 64), (513, 16, 64, 32), (1000, 64, 256, 256), (1000, 64, 256, 0),
                                       (2048, 64, 1024, 0), (700, 128, 256, 256), (300, 8, 64, 24)])
@pytest.mark.parametrize("trans", [False, True])
def test_sbr_backtransform_parity(n, b, k, kbt, trans, dev):
    A = trid_gen.random_symmetric_np(n, 11 + n)
    Ad = to_dev(A)
    tau1 = trid.sbr_dbbr(Ad, b, nb=min(16, b), k=k)
    Aout, t1 = from_dev(Ad), tau1.cpu().numpy()
    C = np.random.default_rng(n + b).uniform(-1, 1, (n, 37))
    ref = oracle.sbr_backtransform(Aout, t1, b, C, trans=trans)
    Cd = to_dev(C)
    trid.sbr_backtransform(Ad, tau1, b, Cd, trans=trans, k=kbt)
    got = from_dev(Cd)
    tol = 64 * n * U * np.max(np.linalg.norm(C, axis=0))
    assert np.max(np.abs(got - ref)) <= tol


@pytest.mark.parametrize("n,b", [(300, 32), (257, 64), (700, 64), (513, 128), (300, 256), (100, 8), (50, 100), (40, 2),
                                 (1500, 48), (4000, 64)])
@pytest.mark.parametrize("trans", [False, True])
def test_bc_backtransform_parity(n, b, trans, dev):
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 5 * n + b), min(b, n - 1))
    d, e, V2, tau2 = trid.bulge_chase(to_dev(Bm), b)
    ncols = 45
    C = np.random.default_rng(n).uniform(-1, 1, (n, ncols))
    ref = oracle.bc_backtransform(V2.cpu().numpy(), tau2.cpu().numpy(), b, C, trans=trans)
    Cd = to_dev(C)
    trid.bc_backtransform(V2, tau2, n, b, Cd, trans=trans)
    got = from_dev(Cd)
    tol = 64 * n * U * np.max(np.linalg.norm(C, axis=0))
    assert np.max(np.abs(got - ref)) <= tol


def form_q_gpu(n, b, S, tau1, V2, tau2):
    Q = torch.eye(n, dtype=torch.float64, device="cuda:0")   # storage of the column-major identity
    trid.bc_backtransform(V2, tau2, n, b, Q)
    trid.sbr_backtransform(S, tau1, b, Q)
    return Q.mT   # logical Q


@pytest.mark.parametrize("n,b,k", [(1024, 64, 256), (2048, 32, 1024), (8192, 64, 1024)])
def test_exact_gates_with_gpu_q(n, b, k, dev):
    """G1/G2 exactly (no probes): Q = Q1 Q2 formed on the GPU by the two back-transformations; at n = 8192 this is
    configs[1] in the bench configuration.  Cross-checked against the test-side probe estimate (tests/qapply.py)."""
    from tests.qapply import probe_gates
    A = trid_gen.random_symmetric(n, 2001 if n == 8192 else 7 + n, device="cuda:0")
    A0 = A.clone()
    d, e, tau1, V2, tau2 = trid.sytrd_2stage(A, b, nb=16 if b >= 16 else b, k=k)
    Q = form_q_gpu(n, b, A, tau1, V2, tau2)
    T = torch.diag(d) + torch.diag(e, 1) + torch.diag(e, -1)
    nA = float(torch.linalg.norm(A0))
    g1 = float(torch.linalg.norm(A0 - Q @ T @ Q.T)) / (n * nA)
    g2 = float(torch.linalg.norm(Q.T @ Q - torch.eye(n, dtype=torch.float64, device="cuda:0"))) / n
    assert g1 <= 1e-14 and g2 <= 1e-14, (g1, g2)
    p1, p2 = probe_gates(A0, A, d, e, tau1, V2, tau2, b, p=8)
    assert p1 <= 1e-14 and p2 <= 1e-14
    # Q e_0 = e_0 (every reflector acts on rows >= 1)
    assert float(torch.max(torch.abs(Q[:, 0] - torch.eye(n, dtype=torch.float64, device="cuda:0")[:, 0]))) == 0.0
