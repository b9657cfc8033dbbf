"""Standalone timing of the DMMA contractions (test-side tool): syr2k (a5) and the Z builder SYMM (a3)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402


def timeit(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
    k = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
    w = int(sys.argv[3]) if len(sys.argv) > 3 else 64
    C = torch.randn(n, n, dtype=torch.float64, device="cuda")
    Y = torch.randn(k, n, dtype=torch.float64, device="cuda")
    Z = torch.randn(k, n, dtype=torch.float64, device="cuda")
    ms = timeit(lambda: trid.syr2k_lower(C, Y, Z))
    fl = 2.0 * n * (n + 1) * k
    out = {"syr2k": {"n": n, "k": k, "ms": round(ms, 3), "tflops": round(fl / ms / 1e9, 2)}}
    W = torch.randn(w, n, dtype=torch.float64, device="cuda")
    ms = timeit(lambda: trid.zy(C, W, W))
    fl = 2.0 * n * n * w
    out["zy_symm"] = {"m": n, "w": w, "ms": round(ms, 3), "tflops_symm_part": round(fl / ms / 1e9, 2)}
    A = torch.randn(n, n, dtype=torch.float64, device="cuda")
    B = torch.randn(n, n, dtype=torch.float64, device="cuda")
    ms = timeit(lambda: A @ B, reps=2)
    out["cublas_dgemm"] = {"n": n, "ms": round(ms, 3), "tflops": round(2.0 * n ** 3 / ms / 1e9, 2)}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
