"""Per-link latency breakdown of the warp-specialized bulge chase (debug tool, TRID_BC_TRACE=s).

Slots (bulge.cu BCW_TRACE): compute 0 data ready, 1 col0 final, 2 step done; STORE 3 col0 seen, 4 col0 bulk
store complete, 5 prog released, 6 prog_full released; LOAD 7 fill start, 8 body deps met, 9 last-col dep met.
For sweep s+1 step m the critical link is (s, m+1) publishes col0 -> (s+1, m) computes its col0."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
b = int(sys.argv[2]) if len(sys.argv) > 2 else 64
sw = int(sys.argv[3]) if len(sys.argv) > 3 else 1000
os.environ["TRID_BC_TRACE"] = str(sw)
import numpy as np  # noqa: E402
import torch  # noqa: E402

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
tr = tr.astype(np.float64)
steps = (n - 3 - (sw + 1)) // b + 1
m = np.arange(2, steps - 3)
p, c = tr[0], tr[1]          # sweep s (producer), s+1 (consumer)
out = {
    "poll_detect_us (prod 5 -> cons 9)": np.mean(c[m, 9] - p[m + 1, 5]) / 1e3,
    "last_col_load_us (cons 9 -> 0)": np.mean(c[m, 0] - c[m, 9]) / 1e3,
    "compute_to_col0_us (0 -> 1)": np.mean(c[m, 1] - c[m, 0]) / 1e3,
    "store_wakeup_us (1 -> 3)": np.mean(c[m, 3] - c[m, 1]) / 1e3,
    "col0_store_complete_us (3 -> 4)": np.mean(c[m, 4] - c[m, 3]) / 1e3,
    "release_us (4 -> 5)": np.mean(c[m, 5] - c[m, 4]) / 1e3,
    "col0_to_step_end_us (1 -> 2)": np.mean(c[m, 2] - c[m, 1]) / 1e3,
    "cols_store_us (2 -> 6)": np.mean(c[m, 6] - c[m, 2]) / 1e3,
    "body_dep_wait_us (7 -> 8)": np.mean(c[m, 8] - c[m, 7]) / 1e3,
    "step_period_us (cons 0 -> next 0)": np.mean(np.diff(c[2:steps - 3, 0])) / 1e3,
    "link_us (prod 5(m+1) -> cons 5(m))": np.mean(c[m, 5] - p[m + 1, 5]) / 1e3,
    "c: matvec partial (0 -> 10)": np.mean(c[m, 10] - c[m, 0]) / 1e3,
    "c: cbar1 (10 -> 11)": np.mean(c[m, 11] - c[m, 10]) / 1e3,
    "c: reduce+cbar2 (11 -> 12)": np.mean(c[m, 12] - c[m, 11]) / 1e3,
    "c: pv+update+writeback+cbar3 (12 -> 13)": np.mean(c[m, 13] - c[m, 12]) / 1e3,
    "c: house+z+cbar4 (13 -> 14)": np.mean(c[m, 14] - c[m, 13]) / 1e3,
    "c: finalize+fence+cbar5 (14 -> 15)": np.mean(c[m, 15] - c[m, 14]) / 1e3,
    "data_ready_gap (cons 0 - max(9 of cons, 2 of cons prev))": np.mean(c[m, 0] - np.maximum(c[m, 9], c[m - 1, 2])) / 1e3,
}
if os.environ.get("TRID_BC_FORCE", "6") == "6":   # bc_v6_kernel slot meanings
    for k in [k for k in out if k.startswith("c: ")]:
        del out[k]
    out.update({
        "v6: body loads+matvec+cbar1 (0 -> 10)": np.mean(c[m, 10] - c[m, 0]) / 1e3,
        "v6: last-col wait (10 -> 11)": np.mean(c[m, 11] - c[m, 10]) / 1e3,
        "v6: col0 path (11 -> 1)": np.mean(c[m, 1] - c[m, 11]) / 1e3,
        "v6: cbar2 (1 -> 12)": np.mean(c[m, 12] - c[m, 1]) / 1e3,
        "v6: update+D writeback+z partials+cbar3 (12 -> 13)": np.mean(c[m, 13] - c[m, 12]) / 1e3,
        "v6: z sum+left apply+O writeback (13 -> 14)": np.mean(c[m, 14] - c[m, 13]) / 1e3,
        "v6: V2+cbar4 (14 -> 2)": np.mean(c[m, 2] - c[m, 14]) / 1e3,
    })
print(json.dumps({k: round(float(v), 3) for k, v in out.items()}, indent=1))
