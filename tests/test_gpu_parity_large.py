"""GPU parity in the full-size regimes (-m gpu): element by element against the CPU oracle at sizes where the
kernels run the launch configurations of the bench workloads (rows per CTA, cluster counts, general-panel
fallback, many concurrent sweeps), which the small cases of test_gpu_parity.py do not reach.

Tolerances as in test_gpu_parity.py: 64 m u ||P||_F for a Householder QR of an m-row panel (each entry is
the result of O(m)-long dot products through at most w reflectors), 64 n u ||A||_F for the reductions."""
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


@pytest.mark.parametrize("m,w", [
    (32704, 64),    # first panel of the n = 32768, b = 64 headline (register kernel, 33 clusters, 248 rows/CTA)
    (49088, 64),    # first panel at n = 49152 (config 4): taller than the register kernel, general kernel
    (32640, 128),   # first panel at n = 32768, b = 128 (general kernel, w = 128)
    (16256, 256),   # first panel at n = 16384, b = 256 (config 5)
])
def test_panel_qr_parity_fullsize(m, w, dev):
    rng = np.random.default_rng(m + w)
    P = rng.uniform(-1, 1, (m, w))
    Po, tau_o = oracle.panel_qr(P)
    Pd = to_dev(P)
    tau, T, Y = trid.panel_qr(Pd)
    got = from_dev(Pd)
    tol = 64 * m * U * np.linalg.norm(P)
    assert np.max(np.abs(got - Po)) <= tol
    assert np.max(np.abs(tau.cpu().numpy() - tau_o)) <= 64 * m * U
    W_o = oracle.wy(Po, tau_o)
    Vu = np.tril(Po, -1) + np.eye(m, w)
    Tl = from_dev(T)
    assert np.max(np.abs(Vu @ Tl - W_o)) <= 64 * m * U * np.max(np.abs(W_o))


@pytest.mark.parametrize("n,b", [(4096, 64), (4096, 32), (4096, 128)])
def test_bulge_chase_parity_n4096(n, b, dev):
    """4094 sweeps on 148 CTAs (every CTA runs ~28 sweeps, ~140 steps in flight) against O2b and O2c."""
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 4096 + b), b)
    d, e, V2, tau2 = trid.bulge_chase(to_dev(Bm), b)
    d, e, V2, tau2 = (x.cpu().numpy() for x in (d, e, V2, tau2))
    tol = 64 * n * U * np.linalg.norm(Bm)
    for ref in (oracle.bc_naive(Bm, b), oracle.bc_r7(Bm, b)):
        d_o, e_o, V_o, t_o = ref
        assert np.max(np.abs(d - d_o)) <= tol
        assert np.max(np.abs(e - e_o)) <= tol
        assert np.max(np.abs(tau2 - t_o)) <= 1e-8
        assert np.max(np.abs(V2 - V_o)) <= 1e-8


@pytest.mark.parametrize("n,b,k", [(2048, 64, 1024), (1024, 32, 256)])
def test_dbbr_parity_n2048(n, b, k, dev):
    """Stage 1 with the headline b and k: two outer blocks, 31 panels, syr2k of rank 1024."""
    A = trid_gen.random_symmetric_np(n, 2048 + b)
    Ao, to = oracle.dbbr(A, b, k)
    Ad = to_dev(A)
    tau1 = trid.sbr_dbbr(Ad, b, nb=16, k=k)
    got = from_dev(Ad)
    tol = 64 * n * U * np.linalg.norm(A)
    assert np.max(np.abs(np.tril(got) - np.tril(Ao))) <= tol
    assert np.max(np.abs(tau1.cpu().numpy() - to)) <= 64 * n * U * 16
    assert np.array_equal(np.triu(got, 1), np.triu(A, 1))
