"""One invocation per 8(f)/wide-chase kernel for ncu --set full captures (test-side tool):
  python tools/prof_next.py wide|bt|stebz|sbrbt|panel128 [n]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
import trid_gen
what = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 8192
dev = torch.device("cuda:0")
if what == "wide":
    A = trid_gen.random_symmetric(n, 5001, device=dev)
    trid.sbr_dbbr(A, 128, nb=16, k=1024)
    torch.cuda.synchronize()
    trid.bulge_chase(A, 128)
elif what in ("bt", "sbrbt", "stebz"):
    A = trid_gen.random_symmetric(n, 2001, device=dev)
    d, e, tau1, V2, tau2 = trid.sytrd_2stage(A, 64, nb=16, k=1024)
    torch.cuda.synchronize()
    if what == "bt":
        C = torch.randn((n, n), dtype=torch.float64, device=dev)
        trid.bc_backtransform(V2, tau2, n, 64, C)
    elif what == "sbrbt":
        C = torch.randn((n, n), dtype=torch.float64, device=dev)
        trid.sbr_backtransform(A, tau1, 64, C)
    else:
        trid.stebz(d, e)
elif what == "panel128":
    P = torch.rand((128, n), dtype=torch.float64, device=dev)
    trid.panel_qr(P)
torch.cuda.synchronize()
