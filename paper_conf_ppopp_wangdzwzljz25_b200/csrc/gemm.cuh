// gemm.cuh — FP64 DMMA contraction engine (host launchers).  See gemm.cu.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace trid {

enum { OP_N = 0, OP_T = 1 };
enum { TILE_128x128 = 0, TILE_128x64 = 1, TILE_64x64 = 2 };

// C = alpha * sum_seg op(A_seg) op(B_seg) + beta * Cin, M x N, column-major.
//   op(A) = A   : A is M x K  (element (m,k) at A[m + k*lda])        OP_N
//   op(A) = A^T : A is K x M  (element (k,m) at A[k + m*lda])        OP_T
//   op(B) = B   : B is K x N  (element (k,n) at B[k + n*ldb])        OP_N
//   op(B) = B^T : B is N x K  (element (n,k) at B[n + k*ldb])        OP_T
// lower != 0: only elements with row + diag_off >= col are written (tiles wholly above are skipped).
// tri != 0  : blockIdx.x enumerates the lower-triangular tiles of a square tiling (syr2k, Fig. 7).
// splits > 1: deterministic split-K; partial z goes to part + z*part_stride (ld part_ld), then
//             reduce_partials() forms C in fixed order.
struct GemmArgs {
  int64_t M = 0, N = 0;
  int nseg = 1;
  // gemm() only, segment 0: rows >= msplit of op(A) are rows (row - msplit) of A2m (same ld) -- two
  // stacked operands [op(A); op(A2m)] in one launch
  const double* A2m = nullptr;
  int64_t msplit = INT64_MAX;
  const double* A[2] = {nullptr, nullptr};
  int64_t lda[2] = {1, 1};
  const double* B[2] = {nullptr, nullptr};
  int64_t ldb[2] = {1, 1};
  int64_t K[2] = {0, 0};
  double alpha = 1.0, beta = 0.0;
  const double* Cin = nullptr;
  int64_t ldcin = 1;
  double* C = nullptr;
  int64_t ldc = 1;
  int lower = 0;
  int64_t diag_off = 0;
  int tri = 0;
  int splits = 1;
  double* part = nullptr;
  int64_t part_ld = 1, part_stride = 0;
  // gemm() only: per-tile arrival counters (zero on entry, left zero on exit, >= tiles entries); when set, the
  // last split of each tile reduces the partials in fixed order (no separate reduction launch)
  unsigned* sem = nullptr;
  // multi-GPU column map for the lower epilogue mask (gemm_ws only): C's column x is global column
  // cmap(x) = ((x+mg_lofs)/mg_cb*mg_g + mg_q)*mg_cb + (x+mg_lofs)%mg_cb - mg_gofs; mg_g <= 1: identity.
  int mg_g = 1, mg_q = 0, mg_cb = 1;
  int64_t mg_lofs = 0, mg_gofs = 0;
};

// 1D block-cyclic column map of one rank
struct MgMap {
  int g = 1, q = 0, cb = 1;
  int64_t lofs = 0, gofs = 0;
};

// Launch; when a.splits > 1 also launches the reduction.  Returns the first CUDA error.
cudaError_t gemm(GemmArgs a, int opA, int opB, int tile, cudaStream_t st);

// Choose a split count so the grid fills the machine for a tall reduction (K >> M, N).
int pick_splits(int64_t M, int64_t N, int64_t K, int tile, int64_t max_part_elems);

// Warp-specialized persistent engine (gemm_ws.cu): tiles 128x128 (N > 64) / 128x64.  gemm_ws: op(A) = A.
cudaError_t gemm_ws(GemmArgs a, int opB, cudaStream_t st);
cudaError_t gemm_ws_op(GemmArgs a, int opA, int opB, cudaStream_t st);
// C (M x N) = alpha op(A) op(B) + beta Cin (ld lda/ldb/ldc), deterministic split-K over part (part_elems doubles)
// A2 != nullptr (opA == OP_T): rows >= msplit of op(A) come from A2 (the stacked [op(A); op(A2)], same ld)
cudaError_t gemm_ws_mm(int opA, int opB, int64_t M, int64_t N, int64_t K, double alpha, const double* A, int64_t lda,
                       const double* B, int64_t ldb, double beta, double* C, int64_t ldc, double* part,
                       int64_t part_elems, cudaStream_t st, const double* A2 = nullptr, int64_t msplit = 0);
// nc: columns of each of the two correction segments folded into the SYMM's K axis (0: none)
int64_t symm_ws_splits(int64_t m, int64_t w, int64_t nc = 0);
int ws_skinny_splits(int64_t M, int64_t N, int64_t K);
int64_t symm_ws_part_elems(int64_t m, int64_t w, int64_t nc = 0);
cudaError_t symm_ws(int64_t m, int64_t w, const double* A, int64_t lda, const double* W, int64_t ldw, double* X,
                    int64_t ldx, double* part, int64_t part_elems, cudaStream_t st, int64_t nc = 0,
                    const double* CA0 = nullptr, const double* CB0 = nullptr, const double* CA1 = nullptr,
                    const double* CB1 = nullptr, int64_t ldca = 0, int64_t ldcb = 0);

// Multi-GPU SYMM partials over a rank's local trailing columns (nqt of them, A_loc rows = global rows).
int64_t symm_mg_part_elems(int64_t m, int64_t w, int64_t nqt);
cudaError_t symm_mg_rows(int64_t m, int64_t w, int64_t nqt, const double* Aloc, int64_t lda, const double* Wloc,
                         int64_t ldwl, double* X, int64_t ldx, const MgMap& mp, double* part, int64_t part_elems,
                         cudaStream_t st);
cudaError_t symm_mg_cols(int64_t m, int64_t w, int64_t nqt, const double* Aloc, int64_t lda, const double* W,
                         int64_t ldw, double* Xl, int64_t ldxl, const MgMap& mp, double* part, int64_t part_elems,
                         cudaStream_t st);

}  // namespace trid
