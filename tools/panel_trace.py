"""Per-column phase timing of one DBBR panel (debug tool, TRID_PANEL_TRACE)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
b = int(sys.argv[2]) if len(sys.argv) > 2 else 64
j = int(sys.argv[3]) if len(sys.argv) > 3 else 640
m = n - j - b
os.environ["TRID_PANEL_TRACE"] = str(m)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402

P = torch.randn(b, m, dtype=torch.float64, device="cuda")
out = torch.empty(1)
# call the building block directly and read the trace from its workspace
import ctypes  # noqa: E402
L = trid.lib()
sz = ctypes.c_size_t()
L.trid_panel_qr_bufsize(m, b, ctypes.byref(sz))
work = torch.zeros(sz.value, dtype=torch.uint8, device="cuda")
tau = torch.zeros(b, dtype=torch.float64, device="cuda")
T = torch.zeros(b, b, dtype=torch.float64, device="cuda")
Y = torch.zeros(b, m, dtype=torch.float64, device="cuda")
for _ in range(2):
    Pc = P.clone()
    st = L.trid_panel_qr(m, b, Pc.data_ptr(), m, tau.data_ptr(), T.data_ptr(), b, Y.data_ptr(), m, work.data_ptr(),
                         sz.value, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    assert st == 0
torch.cuda.synchronize()
off = 8 * (2 * 148 * 2 * b + 2 * 2 * b)
tr = work[off: off + 8 * 2 * 256 * 8].view(torch.int64).cpu().numpy().reshape(2, 256, 8)[:, :b, :].astype(np.float64)
res = {}
for k, name in [(0, "cta0"), (1, "ctaLast")]:
    d = np.diff(tr[k], axis=1)
    res[name] = [round(float(x), 3) for x in d[2:-2].mean(axis=0) / 1e3]
    res[name + "_col_period_us"] = round(float(np.mean(np.diff(tr[k, 2:-2, 0]))) / 1e3, 3)
res["phases"] = "0->1 partials, 1->2 barrier1, 2->3 slot reduce, 3->4 barrier2, 4->5 totals, 5->6 house+update, 6->7 T"
res["panel_us"] = round(float(tr[0, b - 1, 7] - tr[0, 0, 0]) / 1e3, 1)
print(json.dumps(res, indent=1))
