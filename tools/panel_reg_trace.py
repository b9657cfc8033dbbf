"""Per-column phase times of the register-resident panel QR (debug tool, TRID_PANEL_TRACE=m)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
m = int(sys.argv[1]) if len(sys.argv) > 1 else 32704
w = int(sys.argv[2]) if len(sys.argv) > 2 else 64
os.environ["TRID_PANEL_TRACE"] = str(m)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402

P = torch.randn((w, m), dtype=torch.float64, device="cuda")
for _ in range(3):
    Pc = P.clone()
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record()
    trid.panel_qr(Pc)
    ev1.record()
    torch.cuda.synchronize()
print("panel_ms", ev0.elapsed_time(ev1))
# the binding allocates the workspace inside panel_qr; re-run with an explicit workspace to read the trace
import ctypes  # noqa: E402
L = trid.lib()
out = ctypes.c_size_t()
L.trid_panel_qr_bufsize(m, w, ctypes.byref(out))
work = torch.zeros(out.value, dtype=torch.uint8, device="cuda")
tau = torch.zeros(w, dtype=torch.float64, device="cuda")
T = torch.zeros((w, w), dtype=torch.float64, device="cuda")
Y = torch.zeros((w, m), dtype=torch.float64, device="cuda")
Pc = P.clone()
L.trid_panel_qr(m, w, Pc.data_ptr(), m, tau.data_ptr(), T.data_ptr(), w, Y.data_ptr(), m, work.data_ptr(),
                work.numel(), ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
torch.cuda.synchronize()
off = 8 * (2 * 148 * 2 * w + 2 * 2 * w)
tr = work[off: off + 8 * 2 * 256 * 8].view(torch.int64).cpu().numpy().reshape(2, 256, 8).astype(np.float64)
d = np.diff(tr[:, 2:w - 2, :7], axis=2) / 1e3
names = ["gram", "cl.sync", "dsmem+gpart", "grid_barrier", "totals", "house+update+T"]
res = {"cta0": dict(zip(names, [round(float(x), 3) for x in d[0].mean(axis=0)])),
       "ctaLast": dict(zip(names, [round(float(x), 3) for x in d[1].mean(axis=0)])),
       "column_period_us": round(float(np.mean(np.diff(tr[0, 2:w - 2, 0]))) / 1e3, 3)}
print(json.dumps(res, indent=1))
