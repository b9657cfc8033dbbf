import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, trid_gen
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
from tests.helpers import band_from_lower
def to_dev(X): return torch.from_numpy(np.ascontiguousarray(np.asarray(X, dtype=np.float64).T)).to("cuda:0")
cases = []
for n, b in [(200, 72), (300, 100), (300, 128), (600, 256)]:
    Bm = band_from_lower(trid_gen.random_symmetric_np(n, 2 * n + b), min(b, n - 1))
    cases.append((n, b, Bm, oracle.bc_naive(Bm, b)))
for cs in ("2", "4"):
    for opt in ("24", str(24 | 64), str(24 | 128), str(24 | 256), str(24 | 512), str(24 | 64 | 128 | 256 | 512)):
        os.environ["TRID_BC_WCS"] = cs; os.environ["TRID_BC_OPT"] = opt
        res = []
        for n, b, Bm, ref in cases:
            bad = 0
            for rep in range(3):
                try:
                    d, e, V2, tau2 = trid.bulge_chase(to_dev(Bm), b)
                except Exception:
                    bad = -1
                    break
                if float(np.max(np.abs(d.cpu().numpy() - ref[0]))) > 1e-8: bad += 1
            res.append(f"{n}/{b}:{bad}")
        print("cs", cs, "opt", opt, res, flush=True)
