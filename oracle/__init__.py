"""CPU oracle for the two-stage FP64 tridiagonalization — TEST INFRASTRUCTURE ONLY.

Thin ctypes wrapper over ``oracle/trid_oracle.c`` (plain C, fp64, no blocking; see that file and
``trid_oracle.h`` for the paper citations).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this package.  It shares no
code with ``paper_conf_ppopp_wangdzwzljz25_b200`` and never imports it.

All matrices are numpy float64 arrays in Fortran (column-major) order; symmetric matrices are read
through their lower triangle.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "trid_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None
# Compiler-flag builds of the same source (bench.py's cpu_baseline times the oracle "as it stands" under the
# flags SURVEY 8(d) names; the code is never changed for speed).  The tests use the default -O2 build.
FLAG_BUILDS = {"O2": ["-O2"], "O3native": ["-O3", "-march=native"]}
_variant_libs = {}

_D = ctypes.c_double
_I = ctypes.c_int64
_P = ctypes.c_void_p


def _build_one(path, flags, force):
    if force or not os.path.exists(path) or os.path.getmtime(path) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "trid_oracle.h"))):
        tmp = path + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", *flags, "-std=c11", "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, path)
    return path


def build(force: bool = False, variant: str | None = None) -> str:
    """Compile liboracle.so with gcc (plain -O2, no fast-math); variant (FLAG_BUILDS key) builds the same source
    with other flags into liboracle_<variant>.so."""
    if variant and variant != "O2":
        return _build_one(os.path.join(_HERE, f"liboracle_{variant}.so"), FLAG_BUILDS[variant], force)
    return _build_one(_LIB, FLAG_BUILDS["O2"], force)


def timing_lib(variant: str):
    """The oracle built with FLAG_BUILDS[variant] (for bench.py's cpu_baseline only)."""
    if variant == "O2":
        return lib()
    if variant not in _variant_libs:
        L = ctypes.CDLL(build(variant=variant))
        L.oracle_sytd2.argtypes = [_I, _P, _I, _P, _P, _P]
        L.oracle_sbr_naive.argtypes = [_I, _I, _P, _I, _P]
        L.oracle_bc_naive.argtypes = [_I, _I, _P, _I, _P, _P, _P, _P, ctypes.c_int]
        L.oracle_bc_total_steps.restype = _I
        L.oracle_bc_total_steps.argtypes = [_I, _I]
        _variant_libs[variant] = L
    return _variant_libs[variant]


def timed_run(kind: str, A, b: int, variant: str = "O2") -> float:
    """Seconds for one run of O1 (kind "O1": sytd2) or O2 (kind "O2": naive SBR + naive bulge chase, vectors
    stored) on A with the given flag build.  Timing only (bench.py cpu_baseline)."""
    import time
    L = timing_lib(variant)
    A = _f(A)
    n = A.shape[0]
    d = np.zeros(n)
    e = np.zeros(max(n - 1, 1))
    t0 = time.perf_counter()
    if kind == "O1":
        tau = np.zeros(max(n - 1, 1))
        L.oracle_sytd2(n, _p(A), max(n, 1), _p(d), _p(e), _p(tau))
    else:
        tau1 = np.zeros(n)
        L.oracle_sbr_naive(n, b, _p(A), max(n, 1), _p(tau1))
        tot = L.oracle_bc_total_steps(n, b)
        V2 = np.zeros(max(tot * b, 1))
        tau2 = np.zeros(max(tot, 1))
        L.oracle_bc_naive(n, b, _p(A), max(n, 1), _p(d), _p(e), _p(V2), _p(tau2), 0)
    return time.perf_counter() - t0


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        L.oracle_house.restype = _D
        L.oracle_house.argtypes = [_I, _P, _I, ctypes.POINTER(_D)]
        L.oracle_sytd2.argtypes = [_I, _P, _I, _P, _P, _P]
        L.oracle_sbr_naive.argtypes = [_I, _I, _P, _I, _P]
        L.oracle_panel_qr.argtypes = [_I, _I, _P, _I, _P]
        L.oracle_wy.argtypes = [_I, _I, _P, _I, _P, _P, _I]
        L.oracle_zy.argtypes = [_I, _I, _P, _I, _P, _I, _P, _I, _P, _I]
        L.oracle_syr2k_lower.argtypes = [_I, _I, _P, _I, _P, _I, _P, _I]
        L.oracle_dbbr.argtypes = [_I, _I, _I, _P, _I, _P]
        L.oracle_bc_steps.restype = _I
        L.oracle_bc_steps.argtypes = [_I, _I, _I]
        L.oracle_bc_total_steps.restype = _I
        L.oracle_bc_total_steps.argtypes = [_I, _I]
        L.oracle_bc_naive.argtypes = [_I, _I, _P, _I, _P, _P, _P, _P, ctypes.c_int]
        L.oracle_bc_wavefront.argtypes = [_I, _I, _P, _I, _P, _P, _P, _P, _I]
        L.oracle_bc_r7.argtypes = [_I, _I, _P, _I, _P, _P, _P, _P, _I]
        L.oracle_sbr_backtransform.argtypes = [_I, _I, _P, _I, _P, ctypes.c_int, _I, _P, _I]
        L.oracle_bc_backtransform.argtypes = [_I, _I, _P, _P, ctypes.c_int, _I, _P, _I]
        L.oracle_form_q.argtypes = [_I, _I, _P, _I, _P, _P, _P, _P, _I]
        L.oracle_sturm_eig.argtypes = [_I, _P, _P, _P]
        L.oracle_sturm_count.restype = _I
        L.oracle_sturm_count.argtypes = [_I, _P, _P, _D, _D]
        L.oracle_jacobi_eig.restype = ctypes.c_int
        L.oracle_jacobi_eig.argtypes = [_I, _P, _I, _P]
        _lib = L
    return _lib


def _f(a):
    """Fortran-ordered float64 copy."""
    return np.array(a, dtype=np.float64, order="F", copy=True)


def _p(a):
    return None if a is None else a.ctypes.data


def house(x):
    """R1 / P:86-88: returns (v, tau, beta) with v[0] = 1 and (I - tau v v^T) x = beta e_1."""
    x = np.array(x, dtype=np.float64, copy=True)
    beta = _D()
    tau = lib().oracle_house(len(x), _p(x), 1, ctypes.byref(beta))
    v = x.copy()
    if len(v):
        v[0] = 1.0
    return v, tau, beta.value


def sytd2(A):
    """O1: returns (d, e, tau, Aout) for symmetric A (lower referenced)."""
    A = _f(A)
    n = A.shape[0]
    d = np.zeros(n)
    e = np.zeros(max(n - 1, 0))
    tau = np.zeros(max(n - 1, 0))
    lib().oracle_sytd2(n, _p(A), max(n, 1), _p(d), _p(e), _p(tau))
    return d, e, tau, A


def sbr_naive(A, b):
    """O2a: returns (Aout, tau1): band of width b in the lower band, SBR vectors below it."""
    A = _f(A)
    n = A.shape[0]
    tau1 = np.zeros(n)
    lib().oracle_sbr_naive(n, b, _p(A), max(n, 1), _p(tau1))
    return A, tau1


def dbbr(A, b, k):
    """Algorithm 1 with readings R4: returns (Aout, tau1)."""
    A = _f(A)
    n = A.shape[0]
    tau1 = np.zeros(n)
    lib().oracle_dbbr(n, b, k, _p(A), max(n, 1), _p(tau1))
    return A, tau1


def panel_qr(P):
    P = _f(P)
    m, w = P.shape
    tau = np.zeros(min(m, w))
    lib().oracle_panel_qr(m, w, _p(P), max(m, 1), _p(tau))
    return P, tau


def wy(V, tau):
    """P:96-104 recurrence: W with H_1...H_k = I - W V^T (V unit lower trapezoidal, below diagonal)."""
    V = _f(V)
    m, kk = V.shape
    W = np.zeros((m, kk), order="F")
    tau = np.ascontiguousarray(tau, dtype=np.float64)
    lib().oracle_wy(m, kk, _p(V), max(m, 1), _p(tau), _p(W), max(m, 1))
    return W


def zy(A, W, Y):
    """Eq. (1): Z = A W - 1/2 Y W^T A W (A symmetric, lower referenced)."""
    A, W, Y = _f(A), _f(W), _f(Y)
    m, kk = W.shape
    Z = np.zeros((m, kk), order="F")
    lib().oracle_zy(m, kk, _p(A), max(m, 1), _p(W), max(m, 1), _p(Y), max(m, 1), _p(Z), max(m, 1))
    return Z


def syr2k_lower(C, Y, Z):
    C, Y, Z = _f(C), _f(Y), _f(Z)
    m, kk = Y.shape
    lib().oracle_syr2k_lower(m, kk, _p(C), max(m, 1), _p(Y), max(m, 1), _p(Z), max(m, 1))
    return C


def bc_steps(n, b, s):
    return lib().oracle_bc_steps(n, b, s)


def bc_total_steps(n, b):
    return lib().oracle_bc_total_steps(n, b)


def bc_naive(A, b, full=False, want_v=True):
    """O2b: returns (d, e, V2, tau2) from the lower band of A (A itself is not modified)."""
    A = _f(A)
    n = A.shape[0]
    d = np.zeros(n)
    e = np.zeros(max(n - 1, 0))
    tot = bc_total_steps(n, b)
    V2 = np.zeros(max(tot * b, 1)) if want_v else None
    tau2 = np.zeros(max(tot, 1)) if want_v else None
    lib().oracle_bc_naive(n, b, _p(A), max(n, 1), _p(d), _p(e), _p(V2), _p(tau2), 1 if full else 0)
    if want_v:
        V2, tau2 = V2[: tot * b], tau2[:tot]
    return d, e, V2, tau2


def bc_wavefront(A, b, lag):
    """O2b in the pipelined wavefront order with the given lag (R9): returns (d, e, V2, tau2)."""
    A = _f(A)
    n = A.shape[0]
    d = np.zeros(n)
    e = np.zeros(max(n - 1, 0))
    tot = bc_total_steps(n, b)
    V2 = np.zeros(max(tot * b, 1))
    tau2 = np.zeros(max(tot, 1))
    lib().oracle_bc_wavefront(n, b, _p(A), max(n, 1), _p(d), _p(e), _p(V2), _p(tau2), lag)
    return d, e, V2[: tot * b], tau2[:tot]


def bc_r7(A, b, lag=0):
    """O2c: the chase with R7's step grouping (lower triangle only); lag 0 sweep-major, lag >= 1 wavefront."""
    A = _f(A)
    n = A.shape[0]
    d = np.zeros(n)
    e = np.zeros(max(n - 1, 0))
    tot = bc_total_steps(n, b)
    V2 = np.zeros(max(tot * b, 1))
    tau2 = np.zeros(max(tot, 1))
    lib().oracle_bc_r7(n, b, _p(A), max(n, 1), _p(d), _p(e), _p(V2), _p(tau2), lag)
    return d, e, V2[: tot * b], tau2[:tot]


def sbr_backtransform(A_sbr, tau1, b, C, trans=False):
    """C <- Q1 C (or Q1^T C) from the SBR vectors below the band of A_sbr (sec. 4.3), one reflector at a time."""
    A_sbr = _f(A_sbr)
    C = _f(C)
    n, ncols = C.shape
    tau1 = np.ascontiguousarray(tau1, dtype=np.float64)
    lib().oracle_sbr_backtransform(n, b, _p(A_sbr), max(n, 1), _p(tau1), 1 if trans else 0, ncols, _p(C), max(n, 1))
    return C


def bc_backtransform(V2, tau2, b, C, trans=False):
    """C <- Q2 C (or Q2^T C) from the bulge-chasing reflectors (R7 layout), one reflector at a time."""
    C = _f(C)
    n, ncols = C.shape
    V2 = np.ascontiguousarray(V2, dtype=np.float64)
    tau2 = np.ascontiguousarray(tau2, dtype=np.float64)
    lib().oracle_bc_backtransform(n, b, _p(V2), _p(tau2), 1 if trans else 0, ncols, _p(C), max(n, 1))
    return C


def form_q(n, b, A_sbr=None, tau1=None, V2=None, tau2=None):
    """Dense Q = Q1 Q2 (reading R2)."""
    Q = np.zeros((n, n), order="F")
    A_sbr = None if A_sbr is None else _f(A_sbr)
    tau1 = None if tau1 is None else np.ascontiguousarray(tau1, dtype=np.float64)
    V2 = None if V2 is None else np.ascontiguousarray(V2, dtype=np.float64)
    tau2 = None if tau2 is None else np.ascontiguousarray(tau2, dtype=np.float64)
    lib().oracle_form_q(n, b, _p(A_sbr), max(n, 1), _p(tau1), _p(V2), _p(tau2), _p(Q), max(n, 1))
    return Q


def sturm_eig(d, e):
    d = np.ascontiguousarray(d, dtype=np.float64)
    e = np.ascontiguousarray(e, dtype=np.float64)
    n = len(d)
    w = np.zeros(n)
    lib().oracle_sturm_eig(n, _p(d), _p(e) if n > 1 else _p(np.zeros(1)), _p(w))
    return w


def sturm_count(d, e, x, pivmin=2.2250738585072014e-308):
    d = np.ascontiguousarray(d, dtype=np.float64)
    e = np.ascontiguousarray(e, dtype=np.float64)
    return lib().oracle_sturm_count(len(d), _p(d), _p(e) if len(d) > 1 else _p(np.zeros(1)), float(x), pivmin)


def jacobi_eig(A):
    """Cyclic Jacobi; A is symmetrised from its lower triangle first."""
    A = np.array(A, dtype=np.float64)
    L = np.tril(A)
    A = _f(L + np.tril(A, -1).T)
    n = A.shape[0]
    w = np.zeros(n)
    sweeps = lib().oracle_jacobi_eig(n, _p(A), max(n, 1), _p(w))
    return w, sweeps


def tridiagonalize(A, b, k=None):
    """The whole two-stage method on the CPU: DBBR (Alg. 1) then bulge chasing.

    Returns (d, e, Aout, tau1, V2, tau2).  k = None uses the naive column-wise SBR (O2a)."""
    if k is None:
        Aout, tau1 = sbr_naive(A, b)
    else:
        Aout, tau1 = dbbr(A, b, k)
    d, e, V2, tau2 = bc_naive(Aout, b)
    return d, e, Aout, tau1, V2, tau2
