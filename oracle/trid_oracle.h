/* oracle/trid_oracle.h — TEST INFRASTRUCTURE ONLY (never linked into the product library).
 *
 * Plain, slow, obviously-correct CPU reference for the two-stage FP64 tridiagonalization of
 * Wang et al., "Improving Tridiagonalization Performance on GPU Architectures", PPoPP'25
 * (/root/reference/PAPER.md, cited as P:<line>).  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may call it.  It shares no code, header,
 * table or helper with the CUDA path under paper_conf_ppopp_wangdzwzljz25_b200/csrc.
 *
 * Conventions: column-major, element (i,j) of a matrix with leading
 * dimension ld lives at X[j*ld + i]; symmetric matrices are referenced through their LOWER
 * triangle; all arithmetic is IEEE binary64; 0-based indices.
 */
#ifndef TRID_ORACLE_H
#define TRID_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Householder reflector, P:86-88 (sec. 2.1) with the LAPACK dlarfg sign convention (reading R1).
 * x[0] = alpha, x[k*incx] (k>=1) the rest.  On return x[k*incx] (k>=1) holds v[k] (v[0] = 1 implicit),
 * *beta the new leading entry, and the return value is tau; H = I - tau v v^T, H x = beta e_1. */
double oracle_house(int64_t len, double* x, int64_t incx, double* beta);

/* O1: unblocked one-stage tridiagonalization (LAPACK dsytd2, uplo='L'), the "definition" of
 * A = Q T Q^T.  d[n], e[n-1], tau[n-1]; V overwrites A below the subdiagonal. */
void oracle_sytd2(int64_t n, double* A, int64_t lda, double* d, double* e, double* tau);

/* O2a: naive column-wise successive band reduction to bandwidth b (sec. 2.3): for every
 * column c = 0..n-b-2 one reflector on rows c+b..n-1, applied from the left to the panel columns
 * c+1..c+b-1 and two-sided to the trailing matrix.  tau1[n] (zeros past n-b-2). */
void oracle_sbr_naive(int64_t n, int64_t b, double* A, int64_t lda, double* tau1);

/* Householder QR of an m x w panel (Alg. 1 line 5), column by column.  tau[min(m,w)]. */
void oracle_panel_qr(int64_t m, int64_t w, double* P, int64_t ldp, double* tau);

/* WY accumulation by the paper's recurrence: from V (m x kk unit lower trapezoidal,
 * stored below the diagonal of V with implicit unit diagonal) and tau, build W (m x kk) so that
 * H_1 H_2 ... H_kk = I - W V^T. */
void oracle_wy(int64_t m, int64_t kk, const double* V, int64_t ldv, const double* tau, double* W, int64_t ldw);

/* Eq. (1): Z = A W - 1/2 Y W^T A W with A (m x m symmetric, lower), W, Y (m x kk). */
void oracle_zy(int64_t m, int64_t kk, const double* A, int64_t lda, const double* W, int64_t ldw,
               const double* Y, int64_t ldy, double* Z, int64_t ldz);

/* syr2k, lower triangle only: C -= Y Z^T + Z Y^T (Alg. 1 line 15; Fig. 7).  Strict upper untouched. */
void oracle_syr2k_lower(int64_t m, int64_t kk, double* C, int64_t ldc, const double* Y, int64_t ldy,
                        const double* Z, int64_t ldz);

/* Algorithm 1 (DBBR) step by step with readings R4: outer blocks of width k, panels of
 * width b; z from the implicitly-updated trailing matrix; next-panel update (l.8-12) for all but the
 * last panel of a block; deferred syr2k (l.15) from the end of the block's last panel.  k % b == 0. */
void oracle_dbbr(int64_t n, int64_t b, int64_t k, double* A, int64_t lda, double* tau1);

/* Number of bulge-chasing steps of sweep s (reading R7) and the total over all sweeps. */
int64_t oracle_bc_steps(int64_t n, int64_t b, int64_t s);
int64_t oracle_bc_total_steps(int64_t n, int64_t b);

/* O2b: naive sweep-major bulge chasing (sec. 2.4, Fig. 3, Alg. 2; step indexing R7).  Reads the band
 * (diagonal + b subdiagonals) from A's lower triangle, does not modify A.  d[n], e[n-1];
 * V2[total*b] / tau2[total] in the R7 layout (may be NULL).  full != 0 applies every reflector to the
 * whole dense matrix instead of the band window (slow; used to pin the window). */
void oracle_bc_naive(int64_t n, int64_t b, const double* A, int64_t lda, double* d, double* e,
                     double* V2, double* tau2, int full);

/* O2b in the paper's pipelined order (reading R9), run serially: time slot t runs
 * step t - lag*s of every sweep s that has it, highest s first.  Same outputs as oracle_bc_naive. */
void oracle_bc_wavefront(int64_t n, int64_t b, const double* A, int64_t lda, double* d, double* e,
                         double* V2, double* tau2, int64_t lag);

/* O2c: the chase with reading R7's step grouping (a step owns columns R_m; the next reflector is generated
 * and left-applied inside the step), lower triangle only.  lag = 0 sweep-major, lag >= 1 the wavefront order
 * above.  Same outputs as oracle_bc_naive up to rounding; lag 2 reproduces lag 0 bit for bit (R9). */
void oracle_bc_r7(int64_t n, int64_t b, const double* A, int64_t lda, double* d, double* e, double* V2,
                  double* tau2, int64_t lag);

/* Dense Q = Q1 Q2 (reading R2): Q1 = prod_c H_c from the SBR vectors below the band of A_sbr and
 * tau1 (may be NULL: Q1 = I); Q2 = product of the bulge-chasing reflectors in sweep-major order
 * (V2/tau2 may be NULL: Q2 = I). */
void oracle_form_q(int64_t n, int64_t b, const double* A_sbr, int64_t lda, const double* tau1,
                   const double* V2, const double* tau2, double* Q, int64_t ldq);

/* SBR back-transformation (sec. 4.3): C <- Q1 C (trans 0) or Q1^T C (trans 1), one reflector at
 * a time (the definition the paper's Alg. 3 regroups).  C n x ncols. */
void oracle_sbr_backtransform(int64_t n, int64_t b, const double* A, int64_t lda, const double* tau1, int trans,
                              int64_t ncols, double* C, int64_t ldc);

/* BC back-transformation: C <- Q2 C (trans 0) or Q2^T C (trans 1), one reflector at a time. */
void oracle_bc_backtransform(int64_t n, int64_t b, const double* V2, const double* tau2, int trans, int64_t ncols,
                             double* C, int64_t ldc);

/* Eigenvalues of the symmetric tridiagonal T = tridiag(e, d, e) by Sturm-sequence bisection
 * (gate G3), ascending into w[n]. */
void oracle_sturm_eig(int64_t n, const double* d, const double* e, double* w);

/* Number of eigenvalues of T strictly below x (Sturm count with LAPACK dlaebz pivmin guard). */
int64_t oracle_sturm_count(int64_t n, const double* d, const double* e, double x, double pivmin);

/* Cyclic Jacobi eigenvalues of a dense symmetric matrix (Golub & Van Loan, sec. 8.5); A (full storage,
 * both triangles read) is overwritten; ascending eigenvalues into w[n].  Returns the sweep count. */
int oracle_jacobi_eig(int64_t n, double* A, int64_t lda, double* w);

#ifdef __cplusplus
}
#endif
#endif
