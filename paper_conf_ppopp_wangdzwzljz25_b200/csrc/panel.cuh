// panel.cuh — host launchers for the panel QR (panel_qr.cu) and the bulge chase (bulge.cu).
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

namespace trid {

// Panel QR + T + explicit Y (see panel_qr.cu).  red: panel_red_bytes(w) bytes; bar: 256 words (zeroed by the launcher).
size_t panel_red_bytes(int w);
cudaError_t panel_qr(int64_t m, int w, double* P, int64_t ldp, double* tau, double* T, int64_t ldt, double* Y,
                     int64_t ldy, double* red, unsigned* bar, cudaStream_t st);

// Register-resident, cluster-reduced panel QR (panel_reg.cu) for w in {16, 32, 64}, m <= 36864.
bool panel_reg_supported(int64_t m, int w);
size_t panel_reg_gpart_bytes(int w);
cudaError_t panel_qr_reg(int64_t m, int w, double* P, int64_t ldp, double* tau, double* T, int64_t ldt, double* Y,
                         int64_t ldy, double* gpart, unsigned* bar, cudaStream_t st);

// Bulge chasing (see bulge.cu).
int bc_ldab(int64_t n, int b);
int64_t bc_total_steps(int64_t n, int b);
size_t bc_work_bytes(int64_t n, int b);
cudaError_t bulge_chase(int64_t n, int b, const double* A, int64_t lda, double* d, double* e, double* V2,
                        double* tau2, void* work, cudaStream_t st);

}  // namespace trid
