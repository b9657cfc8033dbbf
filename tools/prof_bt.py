import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
import trid_gen
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
b = 64
A = trid_gen.random_symmetric(n, 1, device="cuda")
d, e, tau1, V2, tau2 = trid.sytrd_2stage(A, b, nb=16, k=1024)
C = torch.randn((n, n), dtype=torch.float64, device="cuda")
trid.bc_backtransform(V2, tau2, n, b, C)
torch.cuda.synchronize()
