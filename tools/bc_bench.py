"""Bulge-chase-only timing (test-side tool): reduce one seeded matrix to band once, then time trid_bulge_chase
R times with CUDA events on the launching stream (median, min, max), for low-noise A/B of chase variants.

  python tools/bc_bench.py 32768 64 5        # n b reps   (env TRID_BC_FORCE / TRID_LIB_PATH select variants)
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402
import trid_gen  # noqa: E402


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
    b = int(sys.argv[2]) if len(sys.argv) > 2 else 64
    reps = int(sys.argv[3]) if len(sys.argv) > 3 else 5
    A = trid_gen.random_symmetric(n, 3001 if n >= 32768 else 2001, device="cuda")
    trid.sbr_dbbr(A, b, nb=16, k=1024)
    nbytes, _, _ = trid.bulge_chase_bufsize(n, b)
    work = torch.zeros(nbytes, dtype=torch.uint8, device="cuda")
    trid.bulge_chase(A, b, work=work)          # warm-up
    torch.cuda.synchronize()
    st = torch.cuda.current_stream()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        trid.bulge_chase(A, b, work=work)
        e1.record(st)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(json.dumps({"n": n, "b": b, "reps": reps, "variant": os.environ.get("TRID_BC_FORCE", "default"),
                      "lib": os.environ.get("TRID_LIB_PATH", "in-tree"), "median_ms": round(statistics.median(ts), 3),
                      "min_ms": round(min(ts), 3), "max_ms": round(max(ts), 3)}))


if __name__ == "__main__":
    main()
