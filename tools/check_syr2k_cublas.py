import os, sys, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_wangdzwzljz25_b200 as trid
import trid_gen
from tools.syr2k_study import _load
n, k = 2048, 64
dev = torch.device("cuda:0")
C0 = trid_gen.random_symmetric(n, 7, device=dev)
Y = torch.rand((k, n), dtype=torch.float64, device=dev) * 2 - 1
Z = torch.rand((k, n), dtype=torch.float64, device=dev) * 2 - 1
ref = C0.mT - Y.mT @ Z - Z.mT @ Y   # logical
C1 = C0.clone(); trid.syr2k_lower(C1, Y, Z)
cublas = _load("libcublas.so.12"); h = ctypes.c_void_p(); cublas.cublasCreate_v2(ctypes.byref(h))
cublas.cublasSetStream_v2(h, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
cublas.cublasDsyr2k_v2.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.POINTER(ctypes.c_double), ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p, ctypes.c_int, ctypes.POINTER(ctypes.c_double), ctypes.c_void_p, ctypes.c_int]
C2 = C0.clone()
st = cublas.cublasDsyr2k_v2(h, 0, 0, n, k, ctypes.byref(ctypes.c_double(-1.0)), ctypes.c_void_p(Y.data_ptr()), n, ctypes.c_void_p(Z.data_ptr()), n, ctypes.byref(ctypes.c_double(1.0)), ctypes.c_void_p(C2.data_ptr()), n)
torch.cuda.synchronize()
L = lambda X: torch.tril(X)
print("status", st, "ours-ref", float(torch.max(torch.abs(L(C1.mT) - L(ref)))), "cublas-ref", float(torch.max(torch.abs(L(C2.mT) - L(ref)))), "ours-cublas", float(torch.max(torch.abs(L(C1.mT) - L(C2.mT)))), "changed", float(torch.max(torch.abs(L(C1.mT) - L(C0.mT)))))
