// backtrans.cuh — the back-transformations C <- Q1 C / Q2 C (backtrans.cu).
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

namespace trid {
// T factors (dlarft forward columnwise) of the ceil(kg/b) b-column panels of a reflector block from their Gram
// matrices G (b x b each, ld b, consecutive) and tau: T panels b x b, ld b, consecutive.
cudaError_t tfactor_from_gram(int b, int kg, const double* G, const double* tau, double* T, cudaStream_t st);
int sbr_bt_default_k(int b);
size_t sbr_backtransform_work_bytes(int64_t n, int b, int k, int64_t ncols);
cudaError_t sbr_backtransform(int64_t n, int b, int k, const double* A, int64_t lda, const double* tau1, int trans,
                              int64_t ncols, double* C, int64_t ldc, void* work, cudaStream_t st);
int bc_bt_nb(int b);
cudaError_t bc_backtransform(int64_t n, int b, const double* V2, const double* tau2, int trans, int64_t ncols,
                             double* C, int64_t ldc, cudaStream_t st);
}  // namespace trid
