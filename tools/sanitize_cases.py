"""Small hot-path invocations for compute-sanitizer (racecheck / synccheck / memcheck): the bulge chase (v6 at
b = 32/64, bc_kernel at b = 128, serial and pipelined), the register and general panel kernels, and one small
two-stage run, the TMA-staged syr2k and a DBBR with the folded Z-builder corrections.  Usage: compute-sanitizer --tool racecheck python tools/sanitize_cases.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402
import trid_gen  # noqa: E402


def to_dev(X):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(X, dtype=np.float64).T)).to("cuda:0")


def main():
    from tests.helpers import band_from_lower
    for n, b in [(300, 32), (300, 64), (200, 128), (130, 64)]:
        Bm = band_from_lower(trid_gen.random_symmetric_np(n, n + b), b)
        trid.bulge_chase(to_dev(Bm), b)
    for m, w in [(500, 64), (300, 32), (400, 128)]:
        P = np.random.default_rng(m).uniform(-1, 1, (m, w))
        trid.panel_qr(to_dev(P))
    # the syr2k on the bulk-copy (TMA) producer path, and a DBBR whose Z builder folds the corrections into the SYMM
    C = to_dev(trid_gen.random_symmetric_np(300, 5))
    rng = np.random.default_rng(3)
    trid.syr2k_lower(C, to_dev(rng.uniform(-1, 1, (300, 40))), to_dev(rng.uniform(-1, 1, (300, 40))))
    A = to_dev(trid_gen.random_symmetric_np(600, 7))
    trid.sbr_dbbr(A, 32, nb=8, k=128)
    A = to_dev(trid_gen.random_symmetric_np(256, 1001))
    trid.sytrd_2stage(A, 32, nb=8, k=64)
    torch.cuda.synchronize()
    print("sanitize cases done")


if __name__ == "__main__":
    main()
