"""SURVEY 8(f) row 4 (Table 1 / Fig. 8 analog) and cuSOLVER context:
  * the deferred syr2k C -= Y Z^T + Z Y^T (lower) of libtrid (trid_syr2k_lower, the DMMA engine with the triangular
    tile order of Fig. 7) against cuBLAS cublasDsyr2k (the library routine the paper measures in Table 1), over
    n in {8192, 32768, 49152} and k = 16 ... 4096, same operands, results compared;
  * cuSOLVER's one-stage cusolverDnDsytrd on the bench matrices (n = 8192, 32768) for context next to the two-stage
    method.
Test-side tool (library baselines through ctypes, nothing here is on the product path).  One JSON line per point.

Usage: python tools/syr2k_study.py [--ns 8192,32768,49152] [--ks 16,...,4096] [--sytrd 8192,32768] [--reps 3]
Flop convention: 2 n (n+1) k for the lower-triangular syr2k (the work of the n(n+1)/2 stored entries); cuSOLVER
sytrd: 4 n^3 / 3.
"""
import argparse
import ctypes
import glob
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402
import trid_gen  # noqa: E402


def _load(name):
    import nvidia
    for base in nvidia.__path__:
        for p in glob.glob(os.path.join(base, "*", "lib", name)):
            return ctypes.CDLL(p)
    return ctypes.CDLL(name)


def timed(fn, reps, prep=None):
    st = torch.cuda.current_stream()
    ts = []
    for r in range(reps + 1):
        if prep:
            prep()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        fn()
        e1.record(st)
        torch.cuda.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1))
    ts.sort()
    return ts[len(ts) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ns", default="8192,32768,49152")
    ap.add_argument("--ks", default="16,32,64,128,256,512,1024,2048,4096")
    ap.add_argument("--sytrd", default="8192,32768")
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    cublas = _load("libcublas.so.12")
    handle = ctypes.c_void_p()
    assert cublas.cublasCreate_v2(ctypes.byref(handle)) == 0
    cublas.cublasSetStream_v2(handle, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    cublas.cublasDsyr2k_v2.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                       ctypes.POINTER(ctypes.c_double), ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p,
                                       ctypes.c_int, ctypes.POINTER(ctypes.c_double), ctypes.c_void_p, ctypes.c_int]
    am1, ap1 = ctypes.c_double(-1.0), ctypes.c_double(1.0)
    for n in [int(x) for x in args.ns.split(",") if x]:
        C0 = trid_gen.random_symmetric(n, 7, device=dev)
        C = torch.empty_like(C0)
        for k in [int(x) for x in args.ks.split(",") if x]:
            g = torch.Generator(device=dev).manual_seed(k)
            Y = torch.rand((k, n), dtype=torch.float64, device=dev, generator=g) * 2 - 1   # column-major n x k
            Z = torch.rand((k, n), dtype=torch.float64, device=dev, generator=g) * 2 - 1
            fl = 2.0 * n * (n + 1) * k
            ours = timed(lambda: trid.syr2k_lower(C, Y, Z), args.reps, prep=lambda: C.copy_(C0))
            R1 = torch.tril(C.mT).clone() if n <= 32768 else None   # logical lower triangle

            def cub():
                # cuBLAS column-major: C (n x n, ld n) lower, op N: C = -1 * (Y Z^T + Z Y^T) + C
                st = cublas.cublasDsyr2k_v2(handle, 0, 0, n, k, ctypes.byref(am1), ctypes.c_void_p(Y.data_ptr()), n,
                                            ctypes.c_void_p(Z.data_ptr()), n, ctypes.byref(ap1),
                                            ctypes.c_void_p(C.data_ptr()), n)
                assert st == 0, st
            cb = timed(cub, args.reps, prep=lambda: C.copy_(C0))
            diff = None
            if R1 is not None:
                R2 = torch.tril(C.mT)
                diff = float(torch.max(torch.abs(R1 - R2)) / torch.max(torch.abs(R2)))
                del R2
            print(json.dumps({"row": "syr2k lower: libtrid vs cuBLAS Dsyr2k", "n": n, "k": k,
                              "ours_ms": round(ours, 3), "ours_tflops": round(fl / ours / 1e9, 3),
                              "cublas_ms": round(cb, 3), "cublas_tflops": round(fl / cb / 1e9, 3),
                              "speedup": round(cb / ours, 3), "max_rel_diff": diff}), flush=True)
            del Y, Z, R1
        del C0, C
        torch.cuda.empty_cache()
    # cuSOLVER one-stage sytrd (context)
    cus = _load("libcusolver.so.11")
    sh = ctypes.c_void_p()
    assert cus.cusolverDnCreate(ctypes.byref(sh)) == 0
    cus.cusolverDnSetStream(sh, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    for n in [int(x) for x in args.sytrd.split(",") if x]:
        A0 = trid_gen.random_symmetric(n, 3001 if n == 32768 else 2001, device=dev)
        A = torch.empty_like(A0)
        d = torch.empty(n, dtype=torch.float64, device=dev)
        e = torch.empty(n, dtype=torch.float64, device=dev)
        tau = torch.empty(n, dtype=torch.float64, device=dev)
        info = torch.zeros(1, dtype=torch.int32, device=dev)
        lwork = ctypes.c_int()
        assert cus.cusolverDnDsytrd_bufferSize(sh, 0, n, ctypes.c_void_p(A.data_ptr()), n, ctypes.c_void_p(d.data_ptr()),
                                               ctypes.c_void_p(e.data_ptr()), ctypes.c_void_p(tau.data_ptr()),
                                               ctypes.byref(lwork)) == 0
        work = torch.empty(max(lwork.value, 1), dtype=torch.float64, device=dev)

        def run():
            st = cus.cusolverDnDsytrd(sh, 0, n, ctypes.c_void_p(A.data_ptr()), n, ctypes.c_void_p(d.data_ptr()),
                                      ctypes.c_void_p(e.data_ptr()), ctypes.c_void_p(tau.data_ptr()),
                                      ctypes.c_void_p(work.data_ptr()), lwork.value, ctypes.c_void_p(info.data_ptr()))
            assert st == 0, st
        ms = timed(run, 1 if n >= 32768 else args.reps, prep=lambda: A.copy_(A0))
        print(json.dumps({"row": "cuSOLVER cusolverDnDsytrd (one-stage, context)", "n": n, "ms": round(ms, 1),
                          "tflops_4n3_3": round(4.0 * n ** 3 / 3.0 / ms / 1e9, 3), "info": int(info.item())}),
              flush=True)
        del A0, A, work
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
