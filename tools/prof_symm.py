"""Time (and, under ncu, capture) the DBBR SYMM X = A W at one panel size: the first ws_kernel launch of trid.zy
is the SYMM.  Usage: python tools/prof_symm.py [--m 32704] [--w 64] [--reps 5]"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402
import trid_gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--m", type=int, default=32704)
    ap.add_argument("--w", type=int, default=64)
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    m, w = args.m, args.w
    A = trid_gen.random_symmetric(m, 5, device=dev)
    g = torch.Generator(device=dev).manual_seed(9)
    W = torch.rand((w, m), dtype=torch.float64, device=dev, generator=g) - 0.5
    Y = torch.rand((w, m), dtype=torch.float64, device=dev, generator=g) - 0.5
    trid.profile_begin()
    for _ in range(args.reps):
        trid.zy(A, W, Y)
    torch.cuda.synchronize()
    prof = trid.profile_end()
    print(json.dumps({"m": m, "w": w, "reps": args.reps, "prof": prof,
                      "symm_flops": 2.0 * m * m * w}))


if __name__ == "__main__":
    main()
