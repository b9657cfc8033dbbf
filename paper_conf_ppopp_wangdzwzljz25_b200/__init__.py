"""Thin Python binding of libtrid.so (include/trid.h) — argument marshalling only.

Every step of the method runs in the CUDA library; this module only passes device pointers, sizes and
torch's current CUDA stream through ctypes, and allocates workspaces with torch (PyTorch is the
memory/stream plumbing, not the product).  There is no CPU fallback: if libtrid.so is missing or no
CUDA device is present, every call raises.

Layout: the C-ABI is column-major.  A row-major torch tensor ``X`` of shape (c, r) with unit inner
stride is the column-major r x c matrix with leading dimension ``X.stride(0)``; i.e. torch passes
X^T.  For the symmetric input A that is the same matrix, but the library's LOWER triangle is torch's
UPPER triangle, and results stored "below the band" appear above torch's diagonal.  ``lower_view``
returns the logical column-major matrix as a torch view.
"""
from __future__ import annotations

import ctypes
import os

import torch

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TRID_LIB_PATH") or os.path.join(HERE, "libtrid.so")   # override: A/B timing tools

_lib = None
_I64 = ctypes.c_int64
_INT = ctypes.c_int
_P = ctypes.c_void_p
_SZ = ctypes.c_size_t


class TridError(RuntimeError):
    pass


def lib():
    """Load libtrid.so (build it first with ``python -m paper_conf_ppopp_wangdzwzljz25_b200.build``)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise TridError(f"libtrid.so not built at {LIB_PATH}; run __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        L.trid_status_string.restype = ctypes.c_char_p
        L.trid_status_string.argtypes = [_INT]
        L.trid_version.restype = ctypes.c_char_p
        L.trid_last_error_string.restype = ctypes.c_char_p
        L.trid_default_k.restype = _INT
        L.trid_default_k.argtypes = [_I64, _INT]
        L.trid_bc_total_steps.restype = _I64
        L.trid_bc_total_steps.argtypes = [_I64, _INT]
        L.trid_sbr_dbbr_bufsize.argtypes = [_I64, _INT, _INT, _INT, ctypes.POINTER(_SZ)]
        L.trid_bulge_chase_bufsize.argtypes = [_I64, _INT, ctypes.POINTER(_SZ), ctypes.POINTER(_I64),
                                               ctypes.POINTER(_I64)]
        L.trid_sytrd_2stage_bufsize.argtypes = [_I64, _INT, _INT, _INT, ctypes.POINTER(_SZ), ctypes.POINTER(_I64),
                                                ctypes.POINTER(_I64)]
        L.trid_sbr_dbbr.argtypes = [_I64, _P, _I64, _INT, _INT, _INT, _P, _P, _SZ, _P]
        L.trid_bulge_chase.argtypes = [_I64, _INT, _P, _I64, _P, _P, _P, _P, _P, _SZ, _P]
        L.trid_sytrd_2stage.argtypes = [_I64, _P, _I64, _INT, _INT, _INT, _P, _P, _P, _P, _P, _P, _SZ, _P]
        L.trid_panel_qr_bufsize.argtypes = [_I64, _INT, ctypes.POINTER(_SZ)]
        L.trid_panel_qr.argtypes = [_I64, _INT, _P, _I64, _P, _P, _I64, _P, _I64, _P, _SZ, _P]
        L.trid_syr2k_lower.argtypes = [_I64, _I64, _P, _I64, _P, _I64, _P, _I64, _P]
        L.trid_zy_bufsize.argtypes = [_I64, _INT, ctypes.POINTER(_SZ)]
        L.trid_zy.argtypes = [_I64, _INT, _P, _I64, _P, _I64, _P, _I64, _P, _I64, _P, _SZ, _P]
        L.trid_bulge_chase_band.argtypes = [_I64, _INT, _P, _I64, _P, _P, _P, _P, _P, _SZ, _P]
        L.trid_sbr_backtransform_bufsize.argtypes = [_I64, _INT, _INT, _I64, ctypes.POINTER(_SZ)]
        L.trid_sbr_backtransform.argtypes = [_I64, _INT, _INT, _P, _I64, _P, _INT, _I64, _P, _I64, _P, _SZ, _P]
        L.trid_bc_backtransform.argtypes = [_I64, _INT, _P, _P, _INT, _I64, _P, _I64, _P]
        L.trid_stebz_bufsize.argtypes = [_I64, ctypes.POINTER(_SZ)]
        L.trid_stebz.argtypes = [_I64, _P, _P, _P, _P, _SZ, _P]
        L.trid_syevals_2stage_bufsize.argtypes = [_I64, _INT, _INT, _INT, ctypes.POINTER(_SZ)]
        L.trid_syevals_2stage.argtypes = [_I64, _P, _I64, _INT, _INT, _INT, _P, _P, _SZ, _P]
        L.trid_comm_unique_id.argtypes = [ctypes.c_char_p]
        L.trid_comm_init_nccl.argtypes = [ctypes.c_char_p, _INT, _INT, ctypes.POINTER(_P)]
        L.trid_comm_init_local.argtypes = [_INT, ctypes.POINTER(_P)]
        L.trid_comm_destroy.argtypes = [_P]
        L.trid_comm_size.argtypes = [_P]
        L.trid_comm_rank.argtypes = [_P]
        L.trid_mg_local_cols.restype = _I64
        L.trid_mg_local_cols.argtypes = [_I64, _INT, _INT, _INT]
        L.trid_sbr_dbbr_mg_bufsize.argtypes = [_I64, _INT, _INT, _INT, _INT, _INT, ctypes.POINTER(_SZ)]
        L.trid_sbr_dbbr_mg.argtypes = [_P, _I64, _P, _I64, _INT, _INT, _INT, _INT, _P, _P, _SZ, _P]
        L.trid_band_gather.argtypes = [_P, _I64, _INT, _P, _I64, _INT, _INT, _P, _I64, _P]
        for name in ("trid_bulge_chase_band", "trid_comm_unique_id", "trid_comm_init_nccl", "trid_comm_init_local",
                     "trid_comm_destroy", "trid_comm_size", "trid_comm_rank", "trid_sbr_dbbr_mg_bufsize",
                     "trid_sbr_dbbr_mg", "trid_band_gather"):
            getattr(L, name).restype = _INT
        L.trid_profile_begin.restype = _INT
        L.trid_profile_end.restype = _INT
        L.trid_profile_end.argtypes = [_P, _P, _INT]
        L.trid_kernel_launches.restype = _I64
        for name in ("trid_sbr_backtransform_bufsize", "trid_sbr_backtransform", "trid_bc_backtransform",
                     "trid_stebz_bufsize", "trid_stebz", "trid_syevals_2stage_bufsize", "trid_syevals_2stage",
                     "trid_sbr_dbbr_bufsize", "trid_bulge_chase_bufsize", "trid_sytrd_2stage_bufsize",
                     "trid_sbr_dbbr", "trid_bulge_chase", "trid_sytrd_2stage", "trid_panel_qr_bufsize",
                     "trid_panel_qr", "trid_syr2k_lower", "trid_zy_bufsize", "trid_zy"):
            getattr(L, name).restype = _INT
        _lib = L
    return _lib


EXPORTS = ("trid_status_string", "trid_last_error_string", "trid_version", "trid_default_k", "trid_bc_total_steps", "trid_sbr_dbbr_bufsize",
           "trid_bulge_chase_bufsize", "trid_sytrd_2stage_bufsize", "trid_sbr_dbbr", "trid_bulge_chase",
           "trid_sytrd_2stage", "trid_panel_qr_bufsize", "trid_panel_qr", "trid_syr2k_lower", "trid_zy_bufsize",
           "trid_zy", "trid_profile_begin", "trid_profile_end", "trid_kernel_launches", "trid_bulge_chase_band",
           "trid_comm_unique_id", "trid_comm_init_nccl", "trid_comm_init_local", "trid_comm_destroy", "trid_comm_size",
           "trid_comm_rank", "trid_mg_local_cols", "trid_sbr_dbbr_mg_bufsize", "trid_sbr_dbbr_mg", "trid_band_gather",
           "trid_stebz_bufsize", "trid_stebz", "trid_syevals_2stage_bufsize", "trid_syevals_2stage",
           "trid_sbr_backtransform_bufsize", "trid_sbr_backtransform", "trid_bc_backtransform")

PROF_CLASSES = ("panel_qr", "wy", "symm", "zy", "next_panel", "syr2k", "bulge_chase", "stebz", "sbr_backtransform",
                "bc_backtransform")
SBR_CLASSES = ("panel_qr", "wy", "symm", "zy", "next_panel", "syr2k")


def profile_begin():
    _check(lib().trid_profile_begin(), "trid_profile_begin")


def profile_end():
    """Returns {class: (ms, calls)} for the stages launched since profile_begin()."""
    import numpy as np
    ms = np.zeros(len(PROF_CLASSES))
    calls = np.zeros(len(PROF_CLASSES), dtype=np.int64)
    _check(lib().trid_profile_end(ms.ctypes.data, calls.ctypes.data, len(PROF_CLASSES)), "trid_profile_end")
    return {c: (float(ms[i]), int(calls[i])) for i, c in enumerate(PROF_CLASSES)}


def kernel_launches() -> int:
    return int(lib().trid_kernel_launches())


def _check(status: int, what: str):
    if status != 0:
        msg = f"{what}: {lib().trid_status_string(status).decode()} ({status})"
        if status == 1:
            msg += ": " + lib().trid_last_error_string().decode()
        raise TridError(msg)


def _dev(t: torch.Tensor, name: str):
    if not isinstance(t, torch.Tensor) or not t.is_cuda or t.dtype != torch.float64:
        raise TridError(f"{name} must be a CUDA float64 tensor")
    return t.data_ptr()


def _ld(t: torch.Tensor, rows: int) -> int:
    """Leading dimension of the column-major view of storage tensor t (shape (cols, >=rows))."""
    if t.dim() == 1:
        return max(rows, 1)
    if t.stride(1) != 1:
        raise TridError("storage tensor must have unit inner stride")
    return t.stride(0)


def _stream():
    return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)


def _workspace(nbytes: int, device) -> torch.Tensor:
    return torch.empty(max(int(nbytes), 256), dtype=torch.uint8, device=device)


def lower_view(A: torch.Tensor) -> torch.Tensor:
    """Logical column-major matrix of a storage tensor (a transposed view; element (i, j) = A[j, i])."""
    return A.mT


def default_k(n: int, b: int) -> int:
    return lib().trid_default_k(n, b)


def bc_total_steps(n: int, b: int) -> int:
    return lib().trid_bc_total_steps(n, b)


def sbr_dbbr_bufsize(n, b, nb, k=0):
    out = _SZ()
    _check(lib().trid_sbr_dbbr_bufsize(n, b, nb, k, ctypes.byref(out)), "trid_sbr_dbbr_bufsize")
    return out.value


def bulge_chase_bufsize(n, b):
    out, v2, t2 = _SZ(), _I64(), _I64()
    _check(lib().trid_bulge_chase_bufsize(n, b, ctypes.byref(out), ctypes.byref(v2), ctypes.byref(t2)),
           "trid_bulge_chase_bufsize")
    return out.value, v2.value, t2.value


def sytrd_2stage_bufsize(n, b, nb, k=0):
    out, v2, t2 = _SZ(), _I64(), _I64()
    _check(lib().trid_sytrd_2stage_bufsize(n, b, nb, k, ctypes.byref(out), ctypes.byref(v2), ctypes.byref(t2)),
           "trid_sytrd_2stage_bufsize")
    return out.value, v2.value, t2.value


def sbr_dbbr(A: torch.Tensor, b: int, nb: int | None = None, k: int = 0, tau1=None, work=None):
    """Stage 1 in place on A (n x n storage tensor).  Returns tau1 (n)."""
    n = A.shape[0]
    nb = nb or b
    tau1 = tau1 if tau1 is not None else torch.empty(n, dtype=torch.float64, device=A.device)
    nbytes = sbr_dbbr_bufsize(n, b, nb, k)
    work = work if work is not None else _workspace(nbytes, A.device)
    _check(lib().trid_sbr_dbbr(n, _dev(A, "A"), _ld(A, n), b, nb, k, _dev(tau1, "tau1"), work.data_ptr(),
                               work.numel(), _stream()), "trid_sbr_dbbr")
    return tau1


def bulge_chase(A: torch.Tensor, b: int, want_vectors: bool = True, work=None, out=None):
    """Stage 2 from A's lower band.  Returns (d, e, V2, tau2) (V2/tau2 None in eigenvalues-only mode)."""
    n = A.shape[0]
    nbytes, v2len, t2len = bulge_chase_bufsize(n, b)
    dev = A.device
    if out is None:
        d = torch.empty(n, dtype=torch.float64, device=dev)
        e = torch.empty(max(n - 1, 1), dtype=torch.float64, device=dev)
        V2 = torch.empty(max(v2len, 1), dtype=torch.float64, device=dev) if want_vectors else None
        tau2 = torch.empty(max(t2len, 1), dtype=torch.float64, device=dev) if want_vectors else None
    else:
        d, e, V2, tau2 = out
    work = work if work is not None else _workspace(nbytes, dev)
    _check(lib().trid_bulge_chase(n, b, _dev(A, "A"), _ld(A, n), _dev(d, "d"), _dev(e, "e"),
                                  V2.data_ptr() if V2 is not None else None,
                                  tau2.data_ptr() if tau2 is not None else None,
                                  work.data_ptr(), work.numel(), _stream()), "trid_bulge_chase")
    return d, e[: max(n - 1, 0)], (V2[:v2len] if V2 is not None else None), (tau2[:t2len] if tau2 is not None else None)


def sytrd_2stage(A: torch.Tensor, b: int, nb: int | None = None, k: int = 0, want_vectors: bool = True,
                 work=None, out=None):
    """Both stages in place on A.  Returns (d, e, tau1, V2, tau2)."""
    n = A.shape[0]
    nb = nb or b
    nbytes, v2len, t2len = sytrd_2stage_bufsize(n, b, nb, k)
    dev = A.device
    if out is None:
        d = torch.empty(n, dtype=torch.float64, device=dev)
        e = torch.empty(max(n - 1, 1), dtype=torch.float64, device=dev)
        tau1 = torch.empty(max(n, 1), dtype=torch.float64, device=dev)
        V2 = torch.empty(max(v2len, 1), dtype=torch.float64, device=dev) if want_vectors else None
        tau2 = torch.empty(max(t2len, 1), dtype=torch.float64, device=dev) if want_vectors else None
    else:
        d, e, tau1, V2, tau2 = out
    work = work if work is not None else _workspace(nbytes, dev)
    _check(lib().trid_sytrd_2stage(n, _dev(A, "A"), _ld(A, n), b, nb, k, _dev(d, "d"), _dev(e, "e"),
                                   _dev(tau1, "tau1"), V2.data_ptr() if V2 is not None else None,
                                   tau2.data_ptr() if tau2 is not None else None, work.data_ptr(), work.numel(),
                                   _stream()), "trid_sytrd_2stage")
    return (d, e[: max(n - 1, 0)], tau1[:n], (V2[:v2len] if V2 is not None else None),
            (tau2[:t2len] if tau2 is not None else None))


def panel_qr(P: torch.Tensor):
    """Panel QR of the column-major m x w matrix stored in P (shape (w, m)).  Returns (tau, T, Y) where T and
    Y are storage tensors (shapes (w, w) and (kk, m))."""
    w, m = P.shape
    kk = min(m, w)
    dev = P.device
    tau = torch.zeros(max(kk, 1), dtype=torch.float64, device=dev)
    T = torch.zeros((w, w), dtype=torch.float64, device=dev)
    Y = torch.zeros((max(kk, 1), max(m, 1)), dtype=torch.float64, device=dev)
    out = _SZ()
    _check(lib().trid_panel_qr_bufsize(m, w, ctypes.byref(out)), "trid_panel_qr_bufsize")
    work = _workspace(out.value, dev)
    _check(lib().trid_panel_qr(m, w, _dev(P, "P"), _ld(P, m), _dev(tau, "tau"), _dev(T, "T"), w, _dev(Y, "Y"),
                               max(m, 1), work.data_ptr(), work.numel(), _stream()), "trid_panel_qr")
    return tau[:kk], T, Y


def syr2k_lower(C: torch.Tensor, Y: torch.Tensor, Z: torch.Tensor):
    """C -= Y Z^T + Z Y^T on the column-major lower triangle; C storage (m, m), Y/Z storage (kk, m)."""
    m = C.shape[0]
    kk = Y.shape[0]
    _check(lib().trid_syr2k_lower(m, kk, _dev(C, "C"), _ld(C, m), _dev(Y, "Y"), _ld(Y, m), _dev(Z, "Z"), _ld(Z, m),
                                  _stream()), "trid_syr2k_lower")
    return C


def zy(A: torch.Tensor, W: torch.Tensor, Y: torch.Tensor):
    """Z = A W - 1/2 Y W^T A W (Eq. (1)); A storage (m, m) lower-referenced, W/Y storage (w, m)."""
    m = A.shape[0]
    w = W.shape[0]
    Z = torch.empty((w, m), dtype=torch.float64, device=A.device)
    out = _SZ()
    _check(lib().trid_zy_bufsize(m, w, ctypes.byref(out)), "trid_zy_bufsize")
    work = _workspace(out.value, A.device)
    _check(lib().trid_zy(m, w, _dev(A, "A"), _ld(A, m), _dev(W, "W"), _ld(W, m), _dev(Y, "Y"), _ld(Y, m),
                         _dev(Z, "Z"), m, work.data_ptr(), work.numel(), _stream()), "trid_zy")
    return Z


def bulge_chase_band(AB: torch.Tensor, n: int, b: int, want_vectors: bool = True, work=None, out=None):
    """Stage 2 from LAPACK lower band storage: AB storage tensor of shape (n, ldab) (column-major ldab x n,
    AB[j, i-j] = B(i, j)).  Returns (d, e, V2, tau2)."""
    ldab = _ld(AB, b + 1)
    nbytes, v2len, t2len = bulge_chase_bufsize(n, b)
    dev = AB.device
    if out is None:
        d = torch.empty(max(n, 1), dtype=torch.float64, device=dev)
        e = torch.empty(max(n - 1, 1), dtype=torch.float64, device=dev)
        V2 = torch.empty(max(v2len, 1), dtype=torch.float64, device=dev) if want_vectors else None
        tau2 = torch.empty(max(t2len, 1), dtype=torch.float64, device=dev) if want_vectors else None
    else:
        d, e, V2, tau2 = out
    work = work if work is not None else _workspace(nbytes, dev)
    _check(lib().trid_bulge_chase_band(n, b, _dev(AB, "AB"), ldab, _dev(d, "d"), _dev(e, "e"),
                                       V2.data_ptr() if V2 is not None else None,
                                       tau2.data_ptr() if tau2 is not None else None,
                                       work.data_ptr(), work.numel(), _stream()), "trid_bulge_chase_band")
    return d[:n], e[: max(n - 1, 0)], (V2[:v2len] if V2 is not None else None), (tau2[:t2len] if tau2 is not None else None)


# ------------------------------------------------------------------ back-transformations
def sbr_backtransform(S: torch.Tensor, tau1: torch.Tensor, b: int, C: torch.Tensor, trans: bool = False, k: int = 0,
                      work=None):
    """C <- Q1 C (or Q1^T C) in place.  S: the storage tensor of A after stage 1 (its lower part holds the SBR
    vectors); C: storage tensor of the column-major n x ncols matrix (shape (ncols, n))."""
    n = S.shape[0]
    ncols = C.shape[0]
    out = _SZ()
    _check(lib().trid_sbr_backtransform_bufsize(n, b, k, ncols, ctypes.byref(out)), "trid_sbr_backtransform_bufsize")
    work = work if work is not None else _workspace(out.value, C.device)
    _check(lib().trid_sbr_backtransform(n, b, k, _dev(S, "A"), _ld(S, n), _dev(tau1, "tau1"), 1 if trans else 0,
                                        ncols, _dev(C, "C"), _ld(C, n), work.data_ptr(), work.numel(), _stream()),
           "trid_sbr_backtransform")
    return C


def bc_backtransform(V2, tau2, n: int, b: int, C: torch.Tensor, trans: bool = False):
    """C <- Q2 C (or Q2^T C) in place; C storage tensor of shape (ncols, n)."""
    ncols = C.shape[0]
    _check(lib().trid_bc_backtransform(n, b, V2.data_ptr() if V2 is not None else None,
                                       tau2.data_ptr() if tau2 is not None else None, 1 if trans else 0, ncols,
                                       _dev(C, "C"), _ld(C, n), _stream()), "trid_bc_backtransform")
    return C


# ------------------------------------------------------------------ eigenvalues
def stebz(d: torch.Tensor, e: torch.Tensor, w=None, work=None):
    """Eigenvalues of tridiag(e, d, e), ascending (Sturm bisection on the GPU)."""
    n = d.numel()
    out = _SZ()
    _check(lib().trid_stebz_bufsize(n, ctypes.byref(out)), "trid_stebz_bufsize")
    w = w if w is not None else torch.empty(max(n, 1), dtype=torch.float64, device=d.device)
    work = work if work is not None else _workspace(out.value, d.device)
    _check(lib().trid_stebz(n, _dev(d, "d"), _dev(e, "e") if e.numel() else None, _dev(w, "w"), work.data_ptr(),
                            work.numel(), _stream()), "trid_stebz")
    return w[:n]


def syevals_2stage(A: torch.Tensor, b: int, nb: int | None = None, k: int = 0, w=None, work=None):
    """Eigenvalues of the symmetric A (overwritten) by DBBR + eigenvalues-only BC + Sturm bisection."""
    n = A.shape[0]
    nb = nb or b
    out = _SZ()
    _check(lib().trid_syevals_2stage_bufsize(n, b, nb, k, ctypes.byref(out)), "trid_syevals_2stage_bufsize")
    w = w if w is not None else torch.empty(max(n, 1), dtype=torch.float64, device=A.device)
    work = work if work is not None else _workspace(out.value, A.device)
    _check(lib().trid_syevals_2stage(n, _dev(A, "A"), _ld(A, n), b, nb, k, _dev(w, "w"), work.data_ptr(),
                                     work.numel(), _stream()), "trid_syevals_2stage")
    return w[:n]


# ------------------------------------------------------------------ multi-GPU stage 1
class Comm:
    """A libtrid communicator handle (NCCL rank or local virtual rank)."""

    def __init__(self, handle: int):
        self.handle = ctypes.c_void_p(handle)

    @property
    def size(self) -> int:
        return lib().trid_comm_size(self.handle)

    @property
    def rank(self) -> int:
        return lib().trid_comm_rank(self.handle)

    def destroy(self):
        if self.handle:
            _check(lib().trid_comm_destroy(self.handle), "trid_comm_destroy")
            self.handle = ctypes.c_void_p(0)


def comm_local(nranks: int):
    """nranks virtual ranks sharing this process and the current device (drive each from its own thread)."""
    arr = (_P * nranks)()
    _check(lib().trid_comm_init_local(nranks, arr), "trid_comm_init_local")
    return [Comm(arr[q]) for q in range(nranks)]


def comm_nccl(group=None) -> Comm:
    """NCCL communicator over the ranks of a torch.distributed process group (one GPU per rank, the current
    CUDA device); the 128-byte unique id is created on rank 0 and broadcast through the group."""
    import torch.distributed as dist
    rank, size = dist.get_rank(group), dist.get_world_size(group)
    dev = "cuda" if dist.get_backend(group) == "nccl" else "cpu"
    buf = torch.zeros(128, dtype=torch.uint8, device=dev)
    if rank == 0:
        idb = ctypes.create_string_buffer(128)
        _check(lib().trid_comm_unique_id(idb), "trid_comm_unique_id")
        buf.copy_(torch.frombuffer(bytearray(idb.raw), dtype=torch.uint8))
    dist.broadcast(buf, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
    idb = ctypes.create_string_buffer(bytes(buf.cpu().numpy().tobytes()), 128)
    h = _P()
    _check(lib().trid_comm_init_nccl(idb, size, rank, ctypes.byref(h)), "trid_comm_init_nccl")
    return Comm(h.value)


def mg_local_cols(n: int, colblock: int, nranks: int, rank: int) -> int:
    return int(lib().trid_mg_local_cols(n, colblock, nranks, rank))


def sbr_dbbr_mg_bufsize(n, b, nb, k, nranks, rank):
    out = _SZ()
    _check(lib().trid_sbr_dbbr_mg_bufsize(n, b, nb, k, nranks, rank, ctypes.byref(out)), "trid_sbr_dbbr_mg_bufsize")
    return out.value


def sbr_dbbr_mg(comm: Comm, A_local: torch.Tensor, n: int, b: int, nb: int | None = None, k: int = 0, tau1=None,
                work=None):
    """Stage 1 on this rank's block-cyclic columns (storage tensor of shape (nq, >= n): local column x is row
    x).  Collective over the communicator.  Returns tau1 (n)."""
    nb = nb or b
    g, q = comm.size, comm.rank
    tau1 = tau1 if tau1 is not None else torch.empty(max(n, 1), dtype=torch.float64, device=A_local.device)
    nbytes = sbr_dbbr_mg_bufsize(n, b, nb, k, g, q)
    work = work if work is not None else _workspace(nbytes, A_local.device)
    ldA = _ld(A_local, n) if A_local.numel() else max(n, 1)
    _check(lib().trid_sbr_dbbr_mg(comm.handle, n, A_local.data_ptr() if A_local.numel() else None, ldA, b, b, nb, k,
                                  _dev(tau1, "tau1"), work.data_ptr(), work.numel(), _stream()), "trid_sbr_dbbr_mg")
    return tau1[:n]


def band_gather(comm: Comm, A_local: torch.Tensor, n: int, b: int, root: int = 0, AB=None):
    """Band of the block-cyclic matrix to `root` in LAPACK lower band storage (returned as a storage tensor
    of shape (n, b+1)); collective.  Only root's result holds the band."""
    AB = AB if AB is not None else torch.empty((max(n, 1), b + 1), dtype=torch.float64, device=A_local.device)
    ldA = _ld(A_local, n) if A_local.numel() else max(n, 1)
    _check(lib().trid_band_gather(comm.handle, n, b, A_local.data_ptr() if A_local.numel() else None, ldA, b, root,
                                  _dev(AB, "AB"), _ld(AB, b + 1), _stream()), "trid_band_gather")
    return AB
