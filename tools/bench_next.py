"""Measurement of the SURVEY 8(f) rows on one B200: f1 SBR back-transformation, f2 BC back-transformation, f3
eigenvalues of T (Sturm bisection) and the eigenvalues-only two-stage EVD.  One JSON line per row with the
device time (CUDA events on the launching stream, after warm-up), the algorithmic work and the roofline.

Usage: python tools/bench_next.py [--n 8192] [--b 64] [--k 1024] [--ncols N] [--reps 3]
  f1/f2 transform an n x ncols matrix (ncols = n: the full eigenvector back-transformation).

Algorithmic work:
  f1  4 * sum_g m_g * kg * ncols flops (the two apply contractions of every k-group, m_g = n - c0 - b rows): the
      work of applying Q1 as blocked reflectors; the W-merge and T flops are extra (reported as executed).
  f2  4 * sum over BC reflectors of L * ncols flops (dot + rank-1 update per reflector, L = its length).
  f3  latency-bound recurrence (one IEEE division per element per bisection step): reported as time and the
      Sturm-count element rate, no tensor/HBM roofline.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402
import trid_gen  # noqa: E402

PEAK_FP64 = 37.0


def timed(fn, reps, stream):
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    fn()
    torch.cuda.synchronize()
    for a, b in ev:
        a.record(stream)
        fn()
        b.record(stream)
    torch.cuda.synchronize()
    ts = sorted(a.elapsed_time(b) for a, b in ev)
    return ts[len(ts) // 2], ts


def f1_flops(n, b, k, ncols):
    nref = n - b - 1
    fl = 0.0
    c0 = 0
    while c0 < nref:
        kg = min(k, nref - c0)
        m = n - c0 - b
        fl += 4.0 * m * kg * ncols
        c0 += k
    return fl


def f2_flops(n, b, ncols):
    s = np.arange(0, n - 2, dtype=np.int64)
    nst = (n - 3 - s) // b + 1
    tot = 0.0
    for m in range(int(nst.max())):
        sel = s[nst > m]
        r0 = sel + 1 + m * b
        r1 = np.minimum(sel + (m + 1) * b, n - 1)
        tot += float(np.sum(r1 - r0 + 1))
    return 4.0 * tot * ncols


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=8192)
    ap.add_argument("--b", type=int, default=64)
    ap.add_argument("--k", type=int, default=1024)
    ap.add_argument("--kbt", type=int, default=0, help="back-transformation group width (0: 2048, P:419)")
    ap.add_argument("--ncols", type=int, default=0)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--seed", type=int, default=2001)
    ap.add_argument("--rows", default="f1,f2,f3,evals")
    args = ap.parse_args()
    n, b, k = args.n, args.b, args.k
    ncols = args.ncols or n
    dev = torch.device("cuda:0")
    st = torch.cuda.current_stream()
    A0 = trid_gen.random_symmetric(n, args.seed, device=dev)
    A = A0.clone()
    d, e, tau1, V2, tau2 = trid.sytrd_2stage(A, b, nb=min(16, b), k=k)
    torch.cuda.synchronize()
    rows = args.rows.split(",")
    common = {"n": n, "b": b, "k": k, "ncols": ncols, "seed": args.seed, "dtype": "f64", "data": "synthetic",
              "gpu": torch.cuda.get_device_name(0)}
    if "f1" in rows:
        C0 = torch.randn((ncols, n), dtype=torch.float64, device=dev)
        C = C0.clone()
        nb_, _ = None, None
        kb = args.kbt or max(b, (2048 // b) * b)
        work = torch.empty(trid_bufsize_sbr(n, b, args.kbt, ncols), dtype=torch.uint8, device=dev)

        def run():
            C.copy_(C0)
            trid.sbr_backtransform(A, tau1, b, C, k=args.kbt, work=work)
        copy_ms, _ = timed(lambda: C.copy_(C0), args.reps, st)
        ms, ts = timed(run, args.reps, st)
        ms -= copy_ms
        fl = f1_flops(n, b, kb, ncols)
        tf = fl / (ms * 1e-3) / 1e12
        print(json.dumps({"row": "f1 SBR back-transformation (Alg. 3, k-group W merge)", **common, "kbt": kb,
                          "ms": round(ms, 3), "algorithmic_flops": fl, "tflops": round(tf, 3),
                          "roofline": {"bound": "tensor", "achieved": round(tf, 3), "peak": PEAK_FP64,
                                       "unit": "TFLOP/s", "frac": round(tf / PEAK_FP64, 4)},
                          "copy_ms_subtracted": round(copy_ms, 3), "samples_ms": [round(t, 3) for t in ts]}))
        del C, C0, work
    if "f2" in rows:
        C0 = torch.randn((ncols, n), dtype=torch.float64, device=dev)
        C = C0.clone()

        def run():
            C.copy_(C0)
            trid.bc_backtransform(V2, tau2, n, b, C)
        copy_ms, _ = timed(lambda: C.copy_(C0), args.reps, st)
        ms, ts = timed(run, args.reps, st)
        ms -= copy_ms
        fl = f2_flops(n, b, ncols)
        tf = fl / (ms * 1e-3) / 1e12
        nbb = trid_bc_bt_nb(b)
        cbytes = 16.0 * n * ncols * ((n - 2 + nbb - 1) // nbb)
        print(json.dumps({"row": "f2 BC back-transformation (sweep blocks regrouped by step)", **common,
                          "sweep_block": nbb, "ms": round(ms, 3), "algorithmic_flops": fl, "tflops": round(tf, 3),
                          "roofline": {"bound": "fp64-pipe (DFMA)", "achieved": round(tf, 3), "peak": PEAK_FP64,
                                       "unit": "TFLOP/s", "frac": round(tf / PEAK_FP64, 4)},
                          "c_stream_bytes_min": cbytes, "c_stream_gbs": round(cbytes / (ms * 1e-3) / 1e9, 1),
                          "copy_ms_subtracted": round(copy_ms, 3), "samples_ms": [round(t, 3) for t in ts]}))
        del C, C0
    if "f3" in rows:
        w = torch.empty(n, dtype=torch.float64, device=dev)
        ms, ts = timed(lambda: trid.stebz(d, e, w=w), args.reps, st)
        lam = w.cpu().numpy()
        print(json.dumps({"row": "f3 eigenvalues of T (Sturm bisection)", **common, "ms": round(ms, 3),
                          "eigs_per_s": round(n / (ms * 1e-3), 1),
                          "sturm_elements_per_s_upper": round(n * n * 55 / (ms * 1e-3), 1),
                          "roofline": {"bound": "latency (dependent IEEE division chain per eigenvalue)",
                                       "achieved": None, "peak": None, "unit": None, "frac": None},
                          "lam_min": float(lam[0]), "lam_max": float(lam[-1]),
                          "samples_ms": [round(t, 3) for t in ts]}))
    if "evals" in rows:
        Aw = torch.empty_like(A0)
        w = torch.empty(n, dtype=torch.float64, device=dev)
        from ctypes import byref
        out = trid._SZ()
        trid._check(trid.lib().trid_syevals_2stage_bufsize(n, b, min(16, b), k, byref(out)), "bufsize")
        work = torch.empty(out.value, dtype=torch.uint8, device=dev)

        def run():
            Aw.copy_(A0)
            trid.syevals_2stage(Aw, b, nb=min(16, b), k=k, w=w, work=work)
        ms, ts = timed(run, args.reps, st)
        print(json.dumps({"row": "eigenvalues-only EVD (DBBR + BC without V2 + Sturm bisection)", **common,
                          "ms": round(ms, 3), "tflops_4n3_3": round(4.0 * n ** 3 / 3.0 / (ms * 1e-3) / 1e12, 3),
                          "samples_ms": [round(t, 3) for t in ts]}))


def trid_bufsize_sbr(n, b, k, ncols):
    from ctypes import byref
    out = trid._SZ()
    trid._check(trid.lib().trid_sbr_backtransform_bufsize(n, b, k, ncols, byref(out)), "bufsize")
    return out.value


def trid_bc_bt_nb(b):
    rw = 8 * (8 if b <= 32 else (12 if b <= 64 else (20 if b <= 128 else 36)))
    nb = rw - b + 1
    cap = 200 * 1024 // (16 * rw) - 2
    return max(1, min(nb, cap))


if __name__ == "__main__":
    main()
