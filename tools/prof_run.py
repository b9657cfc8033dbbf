"""One (or a few) two-stage tridiagonalizations for ncu / compute-sanitizer captures (test-side tool).

  ncu --set full -k regex:bc_fast -c 1 -o gpurun_out/prof_bc python tools/prof_run.py --n 8192
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402
import trid_gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=8192)
    ap.add_argument("--b", type=int, default=64)
    ap.add_argument("--k", type=int, default=1024)
    ap.add_argument("--nb", type=int, default=16)
    ap.add_argument("--reps", type=int, default=1)
    ap.add_argument("--stage", default="both", choices=["both", "sbr", "bc", "syr2k"])
    a = ap.parse_args()
    if a.stage == "syr2k":
        C = trid_gen.random_symmetric(a.n, 1, device="cuda")
        Y = torch.randn(a.k, a.n, dtype=torch.float64, device="cuda")
        Z = torch.randn(a.k, a.n, dtype=torch.float64, device="cuda")
        for _ in range(a.reps):
            trid.syr2k_lower(C, Y, Z)
        torch.cuda.synchronize()
        print("ok")
        return
    A0 = trid_gen.random_symmetric(a.n, 2001, device="cuda")
    A = torch.empty_like(A0)
    for _ in range(a.reps):
        A.copy_(A0)
        if a.stage == "bc":
            trid.sbr_dbbr(A, a.b, nb=min(a.nb, a.b), k=a.k)
            torch.cuda.synchronize()
            trid.bulge_chase(A, a.b)
        elif a.stage == "sbr":
            trid.sbr_dbbr(A, a.b, nb=min(a.nb, a.b), k=a.k)
        else:
            trid.sytrd_2stage(A, a.b, nb=min(a.nb, a.b), k=a.k)
    torch.cuda.synchronize()
    print("ok")


if __name__ == "__main__":
    main()
