"""Per-step phase timeline of the wide-band chase (bc_wide_kernel, b > 64; debug tool, TRID_BC_TRACE=s).

Slots (q == 0, tid 0): 0 body deps met (prog_full), 1 body loaded, 2 last-column deps met (prog), 3 partials complete
(barrier 1), 4 next reflector everywhere (barrier 2), 5 fused pass done, 6 stores issued (barrier 3), 7 prog_full
released, 8 column 0 published (prog), 9 thread 0's warp done with the body matvec.  Prints medians relative to slot 0 of the same step, the step-to-step advance
and the link (predecessor's prog release -> our step's deps)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
n = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
b = int(sys.argv[2]) if len(sys.argv) > 2 else 128
sw = int(sys.argv[3]) if len(sys.argv) > 3 else 2000
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
flags = (4 * (2 * n + 128) * 32 + 255) // 256 * 256
tr = work[band + flags: band + flags + 8 * 2 * 1024 * 16].view(torch.int64).cpu().numpy().reshape(2, 1024, 16)
tr = tr.astype(np.float64)
steps = min((n - 3 - (sw + 1)) // b + 1, 1024)
p, c = tr[0], tr[1]
m = np.arange(2, steps - 3)
rel = {str(k): round(float(np.median(c[m, k] - c[m, 0])), 1) for k in range(10)}
adv = {"step_advance_ns (0: m -> m+1)": round(float(np.median(np.diff(c[m, 0]))), 1),
       "prog_full_link_ns (prod 7(m) -> cons 0(m))": round(float(np.median(c[m, 0] - p[m, 7])), 1),
       "col0_link_ns (prod 8(m+1) -> cons 2(m))": round(float(np.median(c[m, 2] - p[m + 1, 8])), 1),
       "sweep_offset_ns (prod 0(m) -> cons 0(m))": round(float(np.median(c[m, 0] - p[m, 0])), 1)}
print(json.dumps({"n": n, "b": b, "sweep": sw + 1, "median_rel_ns": rel, "advances": adv}))
