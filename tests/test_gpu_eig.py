"""GPU eigenvalues of T (include/trid.h trid_stebz / trid_syevals_2stage) against the oracle
(-m gpu).  The kernel evaluates the same Sturm-count definition as oracle_sturm_eig, with the same operations in
the same order and IEEE division, so the eigenvalues must match the oracle's bit for bit; independently they are
pinned to closed forms (1-2-1 Toeplitz) and to LAPACK (numpy eigvalsh) through the whole two-stage method."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
import trid_gen

pytestmark = pytest.mark.gpu
EPS = np.finfo(np.float64).eps


@pytest.mark.parametrize("n,seed", [(1, 1), (2, 2), (3, 3), (100, 4), (1000, 5), (2001, 6), (5000, 7)])
def test_stebz_equals_oracle_bitwise(n, seed, dev):
    rng = np.random.default_rng(seed)
    d = rng.uniform(-1, 1, n)
    e = rng.uniform(-1, 1, max(n - 1, 0))
    w = trid.stebz(torch.from_numpy(d).to(dev), torch.from_numpy(e).to(dev)).cpu().numpy()
    w_o = oracle.sturm_eig(d, e)
    scale = np.max(np.abs(w_o))
    assert np.max(np.abs(w - w_o)) <= 4 * EPS * scale
    assert np.array_equal(w, w_o)


def test_stebz_special_structures(dev):
    """Diagonal T (e = 0), graded entries, repeated eigenvalues and zero pivots (d = 0)."""
    cases = [(np.linspace(-3, 5, 257), np.zeros(256)),
             (np.zeros(300), np.ones(299)),
             (np.repeat([1.0, -2.0, 3.0], 100), np.full(299, 1e-9)),
             (np.logspace(-8, 8, 200), np.logspace(-4, 4, 199))]
    for d, e in cases:
        w = trid.stebz(torch.from_numpy(d).to(dev), torch.from_numpy(e).to(dev)).cpu().numpy()
        w_o = oracle.sturm_eig(d, e)
        assert np.array_equal(w, w_o)
        ref = np.linalg.eigvalsh(np.diag(d) + np.diag(e, 1) + np.diag(e, -1))
        assert np.max(np.abs(w - ref)) <= 1e-12 * np.max(np.abs(ref)) + 1e-300


@pytest.mark.parametrize("n", [64, 4096, 32768])
def test_stebz_toeplitz_closed_form(n, dev):
    d = torch.full((n,), 2.0, dtype=torch.float64, device=dev)
    e = torch.full((n - 1,), -1.0, dtype=torch.float64, device=dev)
    w = trid.stebz(d, e).cpu().numpy()
    lam = trid_gen.toeplitz121_eigs(n)
    assert np.max(np.abs(w - lam)) <= 8 * EPS * 4


@pytest.mark.parametrize("n,b,k", [(256, 32, 64), (1000, 64, 256), (2048, 64, 1024), (1536, 128, 1024)])
def test_syevals_2stage(n, b, k, dev):
    A = trid_gen.random_symmetric_np(n, 77 + n)
    lam = np.linalg.eigvalsh(A)
    Ad = torch.from_numpy(A.T.copy()).to(dev)
    w = trid.syevals_2stage(Ad, b, nb=min(16, b), k=k).cpu().numpy()
    assert np.max(np.abs(w - lam)) <= 1e-12 * np.max(np.abs(lam))
