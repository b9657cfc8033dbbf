import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, trid_gen
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
from tests.helpers import band_from_lower
def to_dev(X): return torch.from_numpy(np.ascontiguousarray(np.asarray(X, dtype=np.float64).T)).to("cuda:0")
for n, b in [(300, 256), (600, 256), (520, 200), (300, 129), (300, 128)]:
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 2 * n + b), min(b, n - 1))
    d_o, e_o, V_o, t_o = oracle.bc_naive(Bm, b)
    d, e, V2, tau2 = trid.bulge_chase(to_dev(Bm), b)
    d = d.cpu().numpy(); e = e.cpu().numpy()
    print(n, b, "dmax", np.max(np.abs(d - d_o)), "d==diag", np.allclose(d, np.diag(Bm)), "tau2 nz", int((tau2 != 0).sum()), len(t_o), "V2diff", float(np.max(np.abs(V2.cpu().numpy() - V_o))), flush=True)
for n, b in [(1024, 128), (2048, 128), (1024, 256)]:
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 1), b)
    Ad = to_dev(Bm)
    for serial in ("0", "1"):
        os.environ["TRID_BC_SERIAL"] = serial
        trid.bulge_chase(Ad, b); torch.cuda.synchronize()
        t = time.perf_counter(); trid.bulge_chase(Ad, b); torch.cuda.synchronize(); dt = time.perf_counter() - t
        print(n, b, "serial", serial, "ms", dt * 1e3, "steps", trid.bc_total_steps(n, b), "us/step", dt * 1e6 / trid.bc_total_steps(n, b), flush=True)
    os.environ["TRID_BC_SERIAL"] = "0"
