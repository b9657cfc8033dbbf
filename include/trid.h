/* include/trid.h — C-ABI of libtrid.so: two-stage FP64 symmetric tridiagonalization on B200 (sm_100a).
 *
 * Method: Wang et al., "Improving Tridiagonalization Performance on GPU Architectures", PPoPP'25.
 * Citations P:<line> are lines of that paper's text; R<k> are the readings listed in
 * DESIGN.md (where the paper is silent, ambiguous or garbled).
 *
 * Problem: A in R^{n x n} symmetric  ->  A = Q T Q^T, T tridiagonal, Q orthogonal
 * (the paper writes A = Q^{-1} T Q; its Q is our Q^T, reading R2).
 *   stage 1 (Alg. 1, DBBR): full -> band of bandwidth b, Q1 = prod_c (I - tau1[c] v_c v_c^T)
 *   stage 2 (Alg. 2, BC):   band -> tridiagonal,       Q2 = prod_{s,m} (I - tau2 v v^T)
 *   Q = Q1 Q2.
 *
 * Conventions for every entry point:
 *   - All array pointers are DEVICE pointers (cudaMalloc / torch CUDA tensors) unless stated otherwise.
 *   - Column-major (Fortran) storage: element (i, j) of A is A[i + j*lda].  Symmetric matrices are
 *     referenced through their LOWER triangle only; the strict upper triangle is never read or written
 *     (reading R6).  A row-major torch (n, n) tensor passed with lda = n is therefore seen transposed:
 *     for symmetric input that is the same matrix, and our lower triangle is torch's upper triangle.
 *   - Sizes are 64-bit.  Every call is asynchronous and stream-ordered on `stream`; the library never
 *     allocates device memory and never synchronizes the host.  The caller owns every buffer.
 *   - Workspaces come from the matching *_bufsize query (host-only).  Calls are reentrant across
 *     streams when each call has its own workspace.
 *   - Errors: argument checks happen on the host before any launch and return -i for the i-th invalid
 *     argument (LAPACK `info` convention).  CUDA launch errors return TRID_ERR_CUDA.  Faults inside
 *     kernels surface at the caller's next synchronization (as in cuBLAS).  NaN/Inf inputs are not
 *     checked and propagate.  No exceptions cross the ABI.
 */
#ifndef TRID_H
#define TRID_H

#include <stddef.h>
#include <stdint.h>
#include <cuda_runtime.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
  TRID_SUCCESS = 0,
  TRID_ERR_CUDA = 1,        /* a CUDA runtime call or launch failed */
  TRID_ERR_NCCL = 2,        /* an NCCL call failed (multi-GPU stage 1); see trid_last_error_string() */
  TRID_ERR_WORKSPACE = 3,   /* dwork_bytes smaller than the *_bufsize result */
  TRID_ERR_UNSUPPORTED = 4  /* a valid but unsupported configuration (e.g. b > TRID_MAX_B) */
};

#define TRID_MAX_B 256      /* largest band width / panel width supported */

/* Human-readable status ("success", "invalid argument 3", ...).  Static storage, never NULL. */
const char* trid_status_string(int status);

/* Description of the last CUDA failure that produced TRID_ERR_CUDA ("no error" if none).  Static storage,
 * process-global, overwritten by the next failure. */
const char* trid_last_error_string(void);

/* Library version string, e.g. "trid-b200 0.1 sm_100a". */
const char* trid_version(void);

/* Default outer block k for DBBR: the largest multiple of b that is <= max(b, 1024) (P:442 uses
 * b = 32, k = 1024; reading R5). */
int trid_default_k(int64_t n, int b);

/* Number of bulge-chasing steps of the whole chase (reading R7): sum_{s=0}^{n-3} (floor((n-3-s)/b)+1)
 * for b >= 2, else 0.  V2 holds b doubles per step, tau2 one. */
int64_t trid_bc_total_steps(int64_t n, int b);

/* ---- workspace queries (host only; no allocation; no CUDA call) -------------------------------- */
int trid_sbr_dbbr_bufsize(int64_t n, int b, int nb, int k, size_t* dwork_bytes);
int trid_bulge_chase_bufsize(int64_t n, int b, size_t* dwork_bytes, int64_t* v2_len, int64_t* tau2_len);
int trid_sytrd_2stage_bufsize(int64_t n, int b, int nb, int k, size_t* dwork_bytes, int64_t* v2_len,
                              int64_t* tau2_len);

/* ---- stage 1: double-blocking band reduction (Alg. 1; readings R4a-f) ----------------
 * In : A (n x n, lda >= max(1,n)), lower triangle = the symmetric input.
 * Out: the diagonal and the b sub-diagonals of A hold the band B; below the band,
 *      A(c+b+1 : n-1, c) holds the SBR Householder vector of column c (unit entry at row c+b implicit),
 *      tau1[c] its scalar (tau1[c] = 0 for c >= n-b-1).  tau1 has n entries.
 * b  : band width = panel width, 1 <= b <= TRID_MAX_B.
 * nb : inner block of the panel QR (R5), 1 <= nb <= b, b % nb == 0 (performance knob; same result up to rounding).
 *      Panels of width b <= 64 are factored whole by the register kernel; wider panels (b % 16 == 0) in blocked form
 *      with 64-column inner blocks (the register kernel's widest), other b by the general kernel.
 * k  : outer block = syr2k rank, k == 0 -> trid_default_k(n, b); else k >= b, k % b == 0.
 * b >= n-1 is a legal no-op (tau1 = 0).  dwork: trid_sbr_dbbr_bufsize bytes, 256-byte aligned. */
int trid_sbr_dbbr(int64_t n, double* A, int64_t lda, int b, int nb, int k, double* tau1,
                  void* dwork, size_t dwork_bytes, cudaStream_t stream);

/* ---- stage 2: bulge chasing on the GPU (sec. 2.4 Fig. 3, Alg. 2; readings R7-R9) -------
 * In : band B of bandwidth b in A's lower band (diagonal + b sub-diagonals), as left by
 *      trid_sbr_dbbr.  Entries below the band are ignored.  A is not modified.
 * Out: d[n], e[n-1] with T = tridiag(e, d, e) (reading R8); V2[trid_bc_total_steps(n,b) * b] and
 *      tau2[trid_bc_total_steps(n,b)] hold the BC reflectors: step m of sweep s stores its vector
 *      (v[0] = 1 explicit, zero padded to b) at V2 + (S(s)+m)*b and its scalar at tau2[S(s)+m],
 *      S(s) = sum_{s'<s} steps(s'); it acts on rows s+1+m*b .. min(s+(m+1)*b, n-1) (reading R7).
 *      V2 == NULL && tau2 == NULL selects eigenvalues-only mode.
 * Sweeps run concurrently, pipelined at lag 2 by release/acquire progress counters (R9); the result
 * is bitwise identical to the sweep-major order of the same kernel (debug env TRID_BC_SERIAL=1 runs that order;
 * tests/test_gpu_parity.py::test_bulge_chase_serial_equals_parallel_bitwise).  b <= 64: one CTA per sweep;
 * 64 < b <= 128: one CTA per sweep (trapezoid window in shared memory), 128 < b <= 256: a cluster of 4. */
int trid_bulge_chase(int64_t n, int b, const double* A, int64_t lda, double* d, double* e, double* V2,
                     double* tau2, void* dwork, size_t dwork_bytes, cudaStream_t stream);

/* ---- both stages: A = Q T Q^T with Q = Q1 Q2 (Q1 from tau1 and the vectors below A's band, Q2 from
 * V2/tau2).  k = 0 -> trid_default_k.  Argument meanings as above. */
int trid_sytrd_2stage(int64_t n, double* A, int64_t lda, int b, int nb, int k, double* d, double* e,
                      double* tau1, double* V2, double* tau2, void* dwork, size_t dwork_bytes,
                      cudaStream_t stream);

/* ---- eigenvalues of T (the eigenvalues-only EVD of P:446-448) ------------------------
 * trid_stebz: w[0..n) = the eigenvalues of T = tridiag(e, d, e) in ascending order, by Sturm-sequence bisection
 * (LAPACK dstebz/dlaebz definition: count of negative pivots of T - xI with the pivmin guard, Gershgorin start,
 * stop at width <= 2 eps max(|lo|,|hi|) + pivmin; the gate G3's definition).  d[n], e[n-1], w[n] device arrays;
 * d/e are not modified.  dwork: trid_stebz_bufsize bytes.  Accuracy: each w[k] is within 2 eps |w[k]| + pivmin
 * of an exact eigenvalue of T (bisection on exact Sturm counts; Kahan's count is backward stable). */
int trid_stebz_bufsize(int64_t n, size_t* dwork_bytes);
int trid_stebz(int64_t n, const double* d, const double* e, double* w, void* dwork, size_t dwork_bytes,
               cudaStream_t stream);

/* trid_syevals_2stage: eigenvalues of the symmetric A (lower triangle, overwritten as by trid_sytrd_2stage) by
 * DBBR + eigenvalues-only bulge chasing (no V2) + trid_stebz; w[n] ascending.  dwork: trid_syevals_2stage_bufsize
 * bytes (holds d, e, tau1 and the stage workspaces).  Argument meanings as trid_sytrd_2stage. */
int trid_syevals_2stage_bufsize(int64_t n, int b, int nb, int k, size_t* dwork_bytes);
int trid_syevals_2stage(int64_t n, double* A, int64_t lda, int b, int nb, int k, double* w, void* dwork,
                        size_t dwork_bytes, cudaStream_t stream);

/* ---- back-transformations: eigenvectors of A from those of T -------------------------
 * trid_sbr_backtransform: C <- Q1 C (trans = 0) or Q1^T C (trans = 1) for the n x ncols matrix C (ld ldc), Q1 from
 * the SBR vectors below A's band and tau1 as left by trid_sbr_dbbr / trid_sytrd_2stage (b, A, lda, tau1 exactly as
 * passed there).  Method: sec. 4.3 Alg. 3 and sec. 5.3: the per-panel W blocks are merged
 * recursively, W = [W1 | W2 - W1 Y1^T W2], into groups of k reflector columns (k = 0 -> 2048; else k >= b,
 * k % b == 0), each applied as one block reflector with DMMA contractions.  A and tau1 are not modified.
 * dwork: trid_sbr_backtransform_bufsize bytes (2 n k + k ncols doubles plus small buffers). */
int trid_sbr_backtransform_bufsize(int64_t n, int b, int k, int64_t ncols, size_t* dwork_bytes);
int trid_sbr_backtransform(int64_t n, int b, int k, const double* A, int64_t lda, const double* tau1, int trans,
                           int64_t ncols, double* C, int64_t ldc, void* dwork, size_t dwork_bytes, cudaStream_t stream);

/* trid_bc_backtransform: C <- Q2 C (trans = 0) or Q2^T C (trans = 1), Q2 from V2/tau2 as returned by
 * trid_bulge_chase (same n and b; R7 layout).  Blocks of consecutive sweeps are regrouped by step (only reflectors
 * on disjoint rows are reordered: the product is Q2 exactly) and applied to 32-column slabs of C, one CTA each.
 * No workspace.  V2/tau2 may be NULL only when the chase stores no reflector (n < 3 or b < 2). */
int trid_bc_backtransform(int64_t n, int b, const double* V2, const double* tau2, int trans, int64_t ncols, double* C,
                          int64_t ldc, cudaStream_t stream);

/* ---- stage 2 from LAPACK lower band storage (dsbtrd-style input): AB[(i-j) + j*ldab] = B(i, j) for
 * 0 <= i-j <= b, ldab >= b+1 (the layout trid_band_gather produces).  Otherwise as trid_bulge_chase. */
int trid_bulge_chase_band(int64_t n, int b, const double* AB, int64_t ldab, double* d, double* e, double* V2,
                          double* tau2, void* dwork, size_t dwork_bytes, cudaStream_t stream);

/* ---- multi-GPU stage 1 ------------------------------------------------
 * One rank per GPU (one process each, NCCL), or — for testing the sharded arithmetic on one device —
 * g "local" virtual ranks in one process, each driven from its own host thread with its own stream.
 * Layout: the n x n matrix is 1D block-cyclic over column blocks of width colblock = b: global column
 * block B lives on rank B % g; rank q stores its columns contiguously in order (local column x) as
 * full-height columns, A_local(i, x) = A(i, c(x)), lda_local >= n; only entries with i >= c(x) (the
 * lower triangle) are referenced.  trid_mg_local_cols gives the local column count.
 * Communicator calls are collective over the ranks; a failing rank leaves the others waiting (as NCCL). */
typedef struct trid_comm* trid_comm_t;
/* 128-byte NCCL unique id (call on one rank, distribute out of band, e.g. torch.distributed.broadcast). */
int trid_comm_unique_id(unsigned char id[128]);
/* NCCL communicator (libnccl.so.2 resolved at run time; the current CUDA device is the rank's GPU). */
int trid_comm_init_nccl(const unsigned char id[128], int nranks, int rank, trid_comm_t* comm);
/* nranks (<= 16) virtual ranks sharing this process and device: comms[q] is rank q. */
int trid_comm_init_local(int nranks, trid_comm_t* comms);
int trid_comm_destroy(trid_comm_t comm);
int trid_comm_size(trid_comm_t comm);
int trid_comm_rank(trid_comm_t comm);
/* number of columns rank `rank` of `nranks` stores (block-cyclic, blocks of colblock); -1 on bad args */
int64_t trid_mg_local_cols(int64_t n, int colblock, int nranks, int rank);
int trid_sbr_dbbr_mg_bufsize(int64_t n, int b, int nb, int k, int nranks, int rank, size_t* dwork_bytes);
/* Alg. 1 with the per-panel exchange of SURVEY 8(e): the panel owner's [Y_p | T | tau] is broadcast,
 * the partial X = A_blk W_p over each rank's stored entries plus the rank's row slice of the implicit-update
 * corrections (R4e) is all-reduced (sum), S and Z_p are formed redundantly, the next-panel update runs on the
 * next panel's owner, the syr2k on every rank's own columns.
 * Out: as trid_sbr_dbbr, in the block-cyclic layout (band + SBR vectors in each owner's columns);
 * tau1[n] complete on every rank.  colblock must equal b. */
int trid_sbr_dbbr_mg(trid_comm_t comm, int64_t n, double* A_local, int64_t lda_local, int colblock, int b, int nb,
                     int k, double* tau1, void* dwork, size_t dwork_bytes, cudaStream_t stream);
/* Gather the band (diagonal + b sub-diagonals) to `root` in LAPACK lower band storage AB (ldab >= b+1,
 * ldab x n doubles, a device buffer on EVERY rank — it is the send buffer; only root's holds the band on
 * return).  Collective (a sum-reduce of disjoint column sets). */
int trid_band_gather(trid_comm_t comm, int64_t n, int b, const double* A_local, int64_t lda_local, int colblock,
                     int root, double* AB, int64_t ldab, cudaStream_t stream);

/* ---- profiling (host-side, optional; used by bench.py) ------------------------------------------
 * trid_profile_begin(): from now on every hot-path stage launched by the library is bracketed by a pair
 * of CUDA events recorded on the stream it runs on.  trid_profile_end(ms, calls, nclass) synchronizes
 * those events and returns, per stage class, the summed elapsed milliseconds and the number of stage
 * instances; classes: 0 panel QR (a1/a2), 1 W = Y T, 2 SYMM X = A W (a3), 3 Z-builder corrections and
 * Z = X - 1/2 Y W^T X (a3), 4 next-panel update (a4), 5 deferred syr2k (a5), 6 bulge chase incl. band
 * pack and d/e extraction (a6/a7), 7 Sturm bisection (trid_stebz), 8 SBR back-transformation, 9 BC
 * back-transformation.  Either pointer may be NULL.  Process-global state (not reentrant).
 * trid_kernel_launches(): total number of CUDA kernels this library has launched in the process. */
int trid_profile_begin(void);
int trid_profile_end(double* ms, int64_t* calls, int nclass);
int64_t trid_kernel_launches(void);

/* ---- hot-path building blocks, exposed for unit parity tests ------------ */

/* a1+a2: Householder QR of the m x w panel P (ld ldp), in place: R in the upper triangle, V below it
 * (unit diagonal implicit), tau[min(m,w)]; T (w x w, ld ldt, upper triangular, dlarft forward
 * columnwise) and Y (m x min(m,w), ld ldy: V made explicit with unit diagonal and zeros above) such
 * that H_1 ... H_kk = I - Y T Y^T.  w <= TRID_MAX_B.  Workspace: trid_panel_qr_bufsize. */
int trid_panel_qr_bufsize(int64_t m, int w, size_t* dwork_bytes);
int trid_panel_qr(int64_t m, int w, double* P, int64_t ldp, double* tau, double* T, int64_t ldt,
                  double* Y, int64_t ldy, void* dwork, size_t dwork_bytes, cudaStream_t stream);

/* a5 / a4: C -= Y Z^T + Z Y^T on the lower triangle of the m x m matrix C (strict upper untouched);
 * Y, Z are m x kk.  The DMMA syr2k of Alg. 1 l.15 (Fig. 7); its tiles are staged by TMA tensor copies when the
 * operands are 16-byte aligned with even leading dimensions and m is even (else by cp.async; same bits). */
int trid_syr2k_lower(int64_t m, int64_t kk, double* C, int64_t ldc, const double* Y, int64_t ldy,
                     const double* Z, int64_t ldz, cudaStream_t stream);

/* a3: X = A W for A (m x m symmetric, lower referenced, ld lda) and W (m x w), then
 * Z = X - 1/2 Y (W^T X) (Eq. (1)).  Workspace: trid_zy_bufsize. */
int trid_zy_bufsize(int64_t m, int w, size_t* dwork_bytes);
int trid_zy(int64_t m, int w, const double* A, int64_t lda, const double* W, int64_t ldw, const double* Y,
            int64_t ldy, double* Z, int64_t ldz, void* dwork, size_t dwork_bytes, cudaStream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* TRID_H */
