"""Per-phase %globaltimer trace of two consecutive bulge-chasing sweeps (debug tool, TRID_BC_TRACE)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
b = int(sys.argv[2]) if len(sys.argv) > 2 else 64
sw = int(sys.argv[3]) if len(sys.argv) > 3 else 1000
os.environ["TRID_BC_TRACE"] = str(sw)
import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402
import trid_gen  # noqa: E402

A = trid_gen.random_symmetric(n, 2001, device="cuda")
trid.sbr_dbbr(A, b, nb=16, k=1024)
nbytes, _, _ = trid.bulge_chase_bufsize(n, b)
work = torch.zeros(nbytes, dtype=torch.uint8, device="cuda")
for _ in range(2):
    trid.bulge_chase(A, b, work=work)
torch.cuda.synchronize()
ldab = 2 * b
band = (8 * n * ldab + 255) // 256 * 256
flags = (4 * (2 * n + 128) * 32 + 255) // 256 * 256   # BC_FLAG_STRIDE = 32
tr = work[band + flags: band + flags + 8 * 2 * 1024 * 16].view(torch.int64).cpu().numpy().reshape(2, 1024, 16)
steps = (n - 3 - sw) // b + 1
out = {}
for k, name in [(0, "sweep0"), (1, "sweep1")]:
    t = tr[k, :steps, :9].astype(np.float64)
    t0 = t[0, 0]
    d = np.diff(t, axis=1)
    out[name] = {"phase_means_us": [round(float(x), 3) for x in np.nanmean(d[2:-2], axis=0) / 1e3],
                 "step_period_us": round(float(np.mean(np.diff(t[2:-2, 0]))) / 1e3, 3)}
# wake-up latency: sweep1 step m (t1) vs sweep0 release of step m+1 (t8)
wake = (tr[1, 2:steps - 3, 1] - tr[0, 3:steps - 2, 8]) / 1e3
out["wake_latency_us_mean"] = round(float(np.mean(wake)), 3)
cyc = (tr[0, 2:steps - 2, 11] - tr[0, 2:steps - 2, 10]).astype(np.float64)
ns = (tr[0, 2:steps - 2, 3] - tr[0, 2:steps - 2, 2]).astype(np.float64)
sub = tr[0, 2:steps - 2].astype(np.float64)
out["phase2_split_cycles"] = {"prefetch_issue": round(float(np.mean(sub[:, 12] - sub[:, 10])), 1),
                              "e_loads": round(float(np.mean(sub[:, 13] - sub[:, 12])), 1),
                              "matvec_warp0": round(float(np.mean(sub[:, 14] - sub[:, 13])), 1),
                              "barrier_wait": round(float(np.mean(sub[:, 11] - sub[:, 14])), 1)}
out["phase2_cycles_mean"] = round(float(np.mean(cyc)), 1)
out["sm_ghz_est"] = round(float(np.sum(cyc) / np.sum(ns)), 3)
out["phases"] = "0 start,1 after flag wait,2 after window load,3 after matvec,4 after D/O writeback,5 after z,6 before store,7 after store+V2,8 after release"
print(json.dumps(out, indent=1))
