import os, time, torch, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import trid_gen
print({k: v for k, v in os.environ.items() if "INJECT" in k or "NSIGHT" in k or "NV_" in k or "CUDA" in k})
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
A = trid_gen.random_symmetric(n, 3001, device="cuda:0")
for lib in ("magma", "cusolver"):
    try:
        torch.backends.cuda.preferred_linalg_library(lib)
        t = time.time()
        w = torch.linalg.eigvalsh(A)
        torch.cuda.synchronize()
        print(lib, "ok", time.time() - t, float(w[0]), float(w[-1]))
    except Exception as e:
        print(lib, "fail", str(e)[:200])
