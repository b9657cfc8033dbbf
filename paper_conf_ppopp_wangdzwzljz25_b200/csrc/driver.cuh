// driver.cuh — host-side pieces of the DBBR driver shared by the single-GPU (api.cu) and the multi-GPU
// (mg.cu) drivers.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace trid {

// Z builder after the SYMM (a3): X -= Y_< (Z_<^T W) + Z_< (Y_<^T W) (R4e), S = W^T X, Z_p = X - 1/2 Y_p S.
// U (ld ldu >= 2*nprev) receives [Z_<^T W; Y_<^T W].  folded: the corrections were applied inside the SYMM launch
// (zy_panel); only S and Z are formed.
cudaError_t zy_tail(int64_t m, int kk, const double* Wp, int64_t ldw, const double* Yp, const double* Yprev,
                    const double* Zprev, int64_t ldyz, int64_t nprev, double* Zp, double* X, int64_t ldx, double* U,
                    int64_t ldu, double* S, int64_t lds, double* part, int64_t part_elems,
                    unsigned* sem, cudaStream_t st, bool folded = false);

// Band pack into compact BC storage from "element (c+o, c) at X[o + c*cs]" (full A: cs = lda+1; LAPACK lower
// band storage: cs = ldab).
cudaError_t bulge_chase_cs(int64_t n, int b, const double* X, int64_t cs, double* d, double* e, double* V2,
                           double* tau2, void* work, cudaStream_t st);

}  // namespace trid
