"""Measured FP64 ceilings on the GPU box (test-side tooling, not product code).

Runs cuBLAS DGEMM through torch.matmul(float64) as a burst and back-to-back for a few seconds,
sampling SM clocks, and prints one JSON line per measurement. The numbers feed the FP64
roofline denominator recorded in DESIGN.md / profiles/.
"""
import json
import subprocess
import time

import torch


def dgemm(n, seconds):
    a = torch.randn(n, n, dtype=torch.float64, device="cuda")
    b = torch.randn(n, n, dtype=torch.float64, device="cuda")
    for _ in range(3):
        a @ b
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    best = 1e30
    for _ in range(5):
        e0.record()
        a @ b
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    burst = 2 * n ** 3 / (best * 1e-3) / 1e12
    smi = subprocess.Popen(
        ["nvidia-smi", "--query-gpu=clocks.sm,power.draw,clocks_event_reasons.active", "--format=csv,noheader",
         "-lms", "200"], stdout=subprocess.PIPE, text=True)
    t0 = time.time()
    cnt = 0
    e0.record()
    while time.time() - t0 < seconds:
        a @ b
        cnt += 1
        if cnt % 4 == 0:
            torch.cuda.synchronize()
    e1.record()
    torch.cuda.synchronize()
    smi.terminate()
    out = smi.communicate()[0].strip().splitlines()
    sustained = 2 * n ** 3 * cnt / (e0.elapsed_time(e1) * 1e-3) / 1e12
    clocks = [int(l.split(",")[0].split()[0]) for l in out if l.strip() and l.split(",")[0].strip().split()[0].isdigit()]
    clocks.sort()
    print(json.dumps({"kind": "cublas_dgemm", "n": n, "burst_tflops": round(burst, 3),
                      "sustained_tflops": round(sustained, 3),
                      "sm_mhz_median": clocks[len(clocks) // 2] if clocks else None,
                      "smi_tail": out[-3:]}))


if __name__ == "__main__":
    dgemm(8192, 4.0)
