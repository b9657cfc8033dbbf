// eig.cuh — eigenvalues of a symmetric tridiagonal matrix by Sturm bisection (eig.cu).
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

namespace trid {
size_t stebz_work_bytes(int64_t n);
// w[0..n) = eigenvalues of tridiag(e, d, e), ascending.  work: stebz_work_bytes(n) bytes, 256-byte aligned.
cudaError_t stebz(int64_t n, const double* d, const double* e, double* w, void* work, cudaStream_t st);
}  // namespace trid
