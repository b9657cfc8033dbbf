"""Multi-GPU stage 1 (-m gpu): the sharded DBBR of DESIGN.md sec. 8 run as g virtual ranks on one device
(libtrid's local communicator: one host thread + stream per rank, collectives as device copies / fixed-order
sums), compared with the CPU oracle element by element, then the north_star gates after the band gather
and the GPU bulge chase from band storage.  Every code path except the three NCCL calls is the one the
NCCL ranks run.  Tolerances as in test_gpu_parity.py."""
import threading

import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
import trid_gen
from tests.helpers import gates

pytestmark = pytest.mark.gpu
U = 2.0 ** -53


def run_mg(n, b, k, g, seed, nb=8):
    """Returns (full matrix after stage 1 (column-major numpy), tau1 per rank, band storage on root)."""
    comms = trid.comm_local(g)
    cols = [trid_gen.block_cyclic_columns(n, b, g, q) for q in range(g)]
    for q in range(g):
        assert trid.mg_local_cols(n, b, g, q) == len(cols[q])
    A_loc = [trid_gen.random_symmetric_rows(n, seed, c, device="cuda:0") for c in cols]
    taus, ABs, errs = [None] * g, [None] * g, []
    streams = [torch.cuda.Stream() for _ in range(g)]

    def rank(q):
        try:
            with torch.cuda.stream(streams[q]):
                taus[q] = trid.sbr_dbbr_mg(comms[q], A_loc[q], n, b, nb=min(nb, b), k=k)
                ABs[q] = trid.band_gather(comms[q], A_loc[q], n, b, root=0)
            streams[q].synchronize()
        except Exception as ex:  # pragma: no cover - reported below
            errs.append(ex)

    th = [threading.Thread(target=rank, args=(q,)) for q in range(g)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert not errs, errs
    torch.cuda.synchronize()
    full = np.zeros((n, n))
    for q in range(g):
        full[:, cols[q]] = A_loc[q].cpu().numpy().T      # storage row x = global column cols[x]
    for c in comms:
        c.destroy()
    return full, [t.cpu().numpy() for t in taus], ABs[0]


@pytest.mark.parametrize("shard", ["1", "0"])
@pytest.mark.parametrize("n,b,k,g", [(256, 32, 64, 1), (256, 32, 64, 2), (300, 32, 96, 3), (300, 32, 64, 4),
                                     (513, 16, 64, 3), (1000, 64, 256, 2), (640, 64, 128, 5)])
def test_mg_dbbr_parity(n, b, k, g, shard, dev, monkeypatch):
    """shard = 1 (default): the implicit-update corrections are split by rows over the ranks and ride in the X
    all-reduce; 0: every rank applies them after it.  Both against the oracle's Alg. 1 (R4e)."""
    monkeypatch.setenv("TRID_MG_SHARD_CORR", shard)
    A = trid_gen.random_symmetric_np(n, 1001)
    Ao, to = oracle.dbbr(A, b, k)
    full, taus, AB = run_mg(n, b, k, g, 1001)
    tol = 64 * n * U * np.linalg.norm(A)
    assert np.max(np.abs(np.tril(full) - np.tril(Ao))) <= tol
    for t in taus:                                      # tau1 complete and identical on every rank
        assert np.max(np.abs(t - to)) <= 64 * n * U * 16
        assert np.array_equal(t, taus[0])
    # band storage on root = the band of the assembled matrix, bitwise
    ABh = AB.cpu().numpy()                              # storage (n, b+1): ABh[j, o] = A(j+o, j)
    for o in range(b + 1):
        j = np.arange(n - o)
        assert np.array_equal(ABh[j, o], full[j + o, j])


@pytest.mark.parametrize("n,b,k,g", [(256, 32, 64, 2), (513, 64, 128, 4), (1024, 64, 256, 3)])
def test_mg_two_stage_gates(n, b, k, g, dev):
    A = trid_gen.random_symmetric_np(n, 1001 + n)
    full, taus, AB = run_mg(n, b, k, g, 1001 + n)
    d, e, V2, tau2 = trid.bulge_chase_band(AB, n, b)
    d, e = d.cpu().numpy(), e.cpu().numpy()
    Q = oracle.form_q(n, b, full, taus[0], V2.cpu().numpy(), tau2.cpu().numpy())
    g1, g2 = gates(A, Q, d, e)
    assert g1 <= 1e-14 and g2 <= 1e-14, (g1, g2)
    d_o, e_o, *_ = oracle.tridiagonalize(A, b, k)
    w, w_o = oracle.sturm_eig(d, e), oracle.sturm_eig(d_o, e_o)
    assert np.max(np.abs(w - w_o)) <= 1e-12 * np.max(np.abs(w_o))


def test_bulge_chase_band_equals_full_storage(dev):
    """trid_bulge_chase_band on LAPACK band storage == trid_bulge_chase on the full matrix, bitwise."""
    n, b = 700, 64
    A = trid_gen.random_symmetric(n, 5, device="cuda:0")
    trid.sbr_dbbr(A, b, nb=16, k=256)
    r_full = trid.bulge_chase(A, b)
    Al = A.T.contiguous()                      # logical column-major matrix as a row-major array
    AB = torch.zeros((n, b + 1), dtype=torch.float64, device="cuda:0")
    for o in range(b + 1):
        AB[: n - o, o] = torch.diagonal(Al, -o)
    r_band = trid.bulge_chase_band(AB, n, b)
    for x, y in zip(r_full, r_band):
        assert torch.equal(x, y)


def test_local_comm_and_argument_checks(dev):
    L = trid.lib()
    comms = trid.comm_local(2)
    try:
        assert comms[0].size == 2 and comms[1].rank == 1
        assert L.trid_sbr_dbbr_mg(comms[0].handle, 1000, None, 1000, 32, 64, 16, 256, None, None, 0, None) == -3
        assert L.trid_band_gather(comms[0].handle, 1000, 64, None, 1000, 64, 0, None, 65, None) == -4
    finally:
        for c in comms:
            c.destroy()
