import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, trid_gen
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
from tests.helpers import band_from_lower
def to_dev(X): return torch.from_numpy(np.ascontiguousarray(np.asarray(X, dtype=np.float64).T)).to("cuda:0")
for n, b in [(300, 128), (300, 100), (200, 72)]:
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 2 * n + b), min(b, n - 1))
    d_o, e_o, V_o, t_o = oracle.bc_naive(Bm, b)
    for cs in ("1", "2", "4"):
        for ser in ("0", "1"):
            os.environ["TRID_BC_WCS"] = cs; os.environ["TRID_BC_SERIAL"] = ser
            d, e, V2, tau2 = trid.bulge_chase(to_dev(Bm), b)
            V2 = V2.cpu().numpy().reshape(-1, b); Vo = V_o.reshape(-1, b)
            bad = np.where(np.max(np.abs(V2 - Vo), axis=1) > 1e-8)[0]
            print(n, b, "cs", cs, "serial", ser, "dmax", float(np.max(np.abs(d.cpu().numpy() - d_o))), "first bad step", bad[:3].tolist(), "tau first bad", (tau2.cpu().numpy()[bad[0]], t_o[bad[0]]) if len(bad) else None, flush=True)
