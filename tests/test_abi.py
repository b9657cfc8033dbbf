"""C-ABI checks that need no GPU: the library loads, exports every symbol include/trid.h declares,
and the host-side argument checks / workspace queries behave as documented."""
import ctypes
import os
import re

import pytest

import paper_conf_ppopp_wangdzwzljz25_b200 as trid

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    src = open(os.path.join(ROOT, "include", "trid.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(trid_[a-z0-9_]+)\s*\(", src)))


def test_header_exports_all_symbols():
    syms = header_symbols()
    assert len(syms) >= 15
    L = trid.lib()
    for s in syms:
        assert hasattr(L, s), s
    assert set(syms) == set(trid.EXPORTS)


def test_version_and_status_strings():
    L = trid.lib()
    assert b"sm_100a" in L.trid_version()
    assert L.trid_status_string(0) == b"success"
    assert L.trid_status_string(-3) == b"invalid argument 3"
    assert L.trid_status_string(3) == b"workspace too small"


def test_default_k_and_step_counts():
    assert trid.default_k(32768, 32) == 1024
    assert trid.default_k(32768, 64) == 1024
    assert trid.default_k(100, 96) == 960
    assert trid.default_k(100, 2048 // 2) == 1024
    import oracle
    for n, b in [(256, 32), (257, 32), (10, 3), (8192, 64), (3, 2), (50, 49), (60, 100)]:
        assert trid.bc_total_steps(n, b) == oracle.bc_total_steps(n, b)
    assert trid.bc_total_steps(100, 1) == 0


def test_bufsize_queries_and_argument_checks():
    L = trid.lib()
    sz = ctypes.c_size_t()
    assert L.trid_sbr_dbbr_bufsize(-1, 32, 8, 0, ctypes.byref(sz)) == -1
    assert L.trid_sbr_dbbr_bufsize(256, 0, 8, 0, ctypes.byref(sz)) == -2
    assert L.trid_sbr_dbbr_bufsize(256, 32, 7, 0, ctypes.byref(sz)) == -3
    assert L.trid_sbr_dbbr_bufsize(256, 32, 8, 48, ctypes.byref(sz)) == -4
    assert L.trid_sbr_dbbr_bufsize(256, 512, 8, 0, ctypes.byref(sz)) == 4
    assert L.trid_sbr_dbbr_bufsize(256, 32, 8, 0, ctypes.byref(sz)) == 0 and sz.value > 0
    nb, v2, t2 = trid.bulge_chase_bufsize(256, 32)
    assert v2 == 1136 * 32 and t2 == 1136 and nb >= 256 * 64 * 8
    # entry points reject bad arguments on the host before touching CUDA
    assert L.trid_sbr_dbbr(-1, None, 1, 32, 8, 0, None, None, 0, None) == -1
    assert L.trid_sbr_dbbr(10, None, 10, 4, 2, 0, None, None, 0, None) == -2
    assert L.trid_sbr_dbbr(10, 1, 5, 4, 2, 0, None, None, 0, None) == -3
    assert L.trid_bulge_chase(10, 0, 1, 10, None, None, None, None, None, 0, None) == -4
    assert L.trid_sytrd_2stage(10, 1, 10, 4, 3, 0, None, None, None, None, None, None, 0, None) == -5
    assert L.trid_syr2k_lower(5, 2, 1, 4, 1, 5, 1, 5, None) == -4
    # n == 0 is a legal no-op
    assert L.trid_bulge_chase(0, 4, None, 1, None, None, None, None, None, 0, None) == 0
    assert L.trid_syr2k_lower(0, 0, None, 1, None, 1, None, 1, None) == 0


def test_library_has_no_cpu_fallback():
    """The product path has no CPU implementation: it rejects host tensors outright."""
    import torch
    A = torch.zeros(8, 8, dtype=torch.float64)
    with pytest.raises(trid.TridError):
        trid.sytrd_2stage(A, 2)


def test_sass_uses_dmma():
    """The contraction kernels are FP64 tensor-core (DMMA) code for sm_100a."""
    import subprocess
    out = subprocess.run(["cuobjdump", "-sass", trid.LIB_PATH], capture_output=True, text=True).stdout
    assert "DMMA" in out
    assert "sm_100a" in subprocess.run(["cuobjdump", "-lelf", trid.LIB_PATH], capture_output=True,
                                       text=True).stdout
