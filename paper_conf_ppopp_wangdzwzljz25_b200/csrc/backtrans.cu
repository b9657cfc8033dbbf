// backtrans.cu — the back-transformations: applying Q1 (SBR) and Q2 (BC) of
// A = Q T Q^T, Q = Q1 Q2 (reading R2), to an n x ncols matrix C.  With C = the eigenvectors of T this is the
// eigenvector back-transformation of the two-stage EVD.
//
// ---- Q1: DBBR back-transformation (sec. 4.3 Alg. 3, sec. 5.3 Fig. 13) ----------------
// Q1 = H_0 ... H_{n-b-2}; reflector c acts on rows c+b.. with v_c = (1, A(c+b+1:, c)), tau1[c].  The reflector
// columns are taken in groups of k (the paper's k = 2048).  Per group [c0, c0+kg):
//   1. Y (m x kg, m = n-c0-b) explicit from A (unit diagonal, zeros above: a staircase);
//   2. per panel of b columns: Gram G = Y_p^T Y_p (DMMA), T_p by the dlarft recurrence (one CTA per panel),
//      W_p = Y_p T_p (DMMA)  -- the b-wide blocks W_i of Fig. 13;
//   3. Alg. 3's merge W = [W_1 | W_2 - W_1 (Y_1^T W_2)] applied level by level (widths b, 2b, ... < kg): two
//      DMMA contractions per pair (Fig. 13: "batched GEMM ... until the size of W_i grows to n x k");
//   4. the group as ONE block reflector I - W Y^T: X = Y^T C (kg x ncols), C -= W X (DMMA, K = kg).
// Q1 C applies the groups last to first (I - W Y^T); Q1^T C first to last (I - Y W^T).  All contractions run on
// the warp-specialized DMMA engine (gemm_ws.cu) with deterministic split-K.
//
// ---- Q2: BC back-transformation (the paper's open problem) --------------------
// Q2 = prod_s prod_m H_{s,m} (sweep-major, R7 layout).  For a block of nb consecutive sweeps [s0, s0+nb) the
// product is G_M ... G_1 G_0 with G_m = H_{s0,m} H_{s0+1,m} ... H_{s0+nb-1,m}: two reflectors of the block whose
// rows overlap always satisfy m' <= m for s < s' (rows s+1+mb.. and s'+1+m'b.. overlap iff |s'-s+(m'-m)b| < b),
// so this order keeps every overlapping pair in sweep-major order and only commutes disjoint ones.  Group G_m
// touches rows [s0+1+mb, s0+nb-1+(m+1)b] (R = b+nb-1 rows).  Q2 C = B_0 (B_1 (... (B_last C))), B = G_M..G_0.
// Kernel: one CTA per 32-column slab of C; per sweep block (last to first) it slides down the rows group by group
// (G_0 first): the group's window rows are loaded from the slab into registers (a warp holds 4 columns; its 8 row
// lanes per column hold interleaved row pairs, so every access is 16 consecutive rows), its nb reflectors (from V2,
// staged once per group in shared memory in window shape, zero-padded) are applied one at a time -- partial dot over
// the thread's rows (two chains), 3 warp shuffles, rank-1 update in registers -- and stored back.  One pass over the slab per sweep block: C traffic n^2 ncols 16 / nb
// bytes, 4 n^2 ncols / 2 useful flops on the FP64 pipe (DFMA; B200's DFMA and DMMA peaks are equal).
#include "common.cuh"
#include "gemm.cuh"
#include "prof.cuh"
#include "backtrans.cuh"

#include <stdlib.h>

namespace trid {

// ================================================================================ Q1 (SBR)
// Y(i, t) = 1 (i == t), A(o+i, c0+t) (i > t), 0 (i < t);  i in [0, m), t in [0, kg)
__global__ void bt_build_y_kernel(int64_t m, int kg, const double* A, int64_t lda, double* Y, int64_t ldy) {
  const int64_t total = m * kg;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = idx % m, t = idx / m;
    Y[i + t * ldy] = i == t ? 1.0 : (i > t ? A[i + t * lda] : 0.0);
  }
}

// One CTA per panel: T (bp x bp, upper, ld b) from the Gram G = Y_p^T Y_p (ld b) and tau (dlarft forward
// columnwise): T(i,i) = tau_i, T(0:i, i) = -tau_i T(0:i, 0:i) G(0:i, i).
__global__ void bt_tfactor_kernel(int b, int kg, const double* G, const double* tau, double* T) {
  const int p = blockIdx.x, t0 = p * b;
  const int bp = (kg - t0) < b ? (kg - t0) : b;
  const double* Gp = G + (size_t)p * b * b;
  double* ts = T + (size_t)p * b * b;   // built in place (L1/L2-resident, b^3/3 flops)
  for (int idx = threadIdx.x; idx < b * b; idx += blockDim.x) ts[idx] = 0.0;
  __syncthreads();
  for (int i = 0; i < bp; ++i) {
    const double ti = tau[t0 + i];
    for (int r = threadIdx.x; r < b; r += blockDim.x) {
      double v = 0.0;
      if (r < i) {
        double acc = 0.0;
        for (int q = r; q < i; ++q) acc += ts[r + q * b] * Gp[q + i * b];
        v = -ti * acc;
      } else if (r == i) {
        v = ti;
      }
      ts[r + i * b] = v;
    }
    __syncthreads();
  }
}

cudaError_t tfactor_from_gram(int b, int kg, const double* G, const double* tau, double* T, cudaStream_t st) {
  const int np = (kg + b - 1) / b;
  bt_tfactor_kernel<<<np, 128, 0, st>>>(b, kg, G, tau, T);
  count_launches(1);
  return cudaGetLastError();
}

namespace {
size_t a256(size_t x) { return (x + 255) / 256 * 256; }

// C (M x N) = alpha op(A) op(B) + beta Cin on the DMMA engine (gemm_ws_mm, split-K when the grid is small)
cudaError_t mm(int opA, int opB, int64_t M, int64_t N, int64_t K, double alpha, const double* A, int64_t lda,
               const double* B, int64_t ldb, double beta, double* C, int64_t ldc, double* part, int64_t part_elems,
               cudaStream_t st) {
  return gemm_ws_mm(opA, opB, M, N, K, alpha, A, lda, B, ldb, beta, C, ldc, part, part_elems, st);
}

struct SbrBtWork {
  double *Y, *W, *X, *G, *T, *S, *part;
  int64_t part_elems;
  size_t bytes;
};
SbrBtWork carve_sbr_bt(void* base, int64_t n, int b, int k, int64_t ncols) {
  SbrBtWork w;
  char* p = (char*)base;
  size_t off = 0;
  auto take = [&](size_t cnt) {
    double* q = p ? (double*)(p + off) : nullptr;
    off += a256(sizeof(double) * cnt);
    return q;
  };
  w.Y = take((size_t)n * k);
  w.W = take((size_t)n * k);
  w.X = take((size_t)k * (ncols > 0 ? ncols : 1));
  w.G = take((size_t)k * b);   // k/b panels of b x b
  w.T = take((size_t)k * b);
  w.S = take((size_t)(k / 2 + b) * (k / 2 + b));
  w.part_elems = (int64_t)8 << 20;   // 64 MB of split-K partials
  w.part = take((size_t)w.part_elems);
  w.bytes = off;
  return w;
}
}  // namespace

int sbr_bt_default_k(int b) {
  int k = (2048 / b) * b;   // k = 2048
  return k < b ? b : k;
}

size_t sbr_backtransform_work_bytes(int64_t n, int b, int k, int64_t ncols) {
  return carve_sbr_bt(nullptr, n, b, k, ncols).bytes;
}

cudaError_t sbr_backtransform(int64_t n, int b, int k, const double* A, int64_t lda, const double* tau1, int trans,
                              int64_t ncols, double* C, int64_t ldc, void* work, cudaStream_t st) {
  const int64_t nref = n - b - 1;   // reflector columns 0 .. n-b-2
  if (nref <= 0 || ncols <= 0) return cudaSuccess;
  SbrBtWork w = carve_sbr_bt(work, n, b, k, ncols);
  const int64_t ngroups = (nref + k - 1) / k;
  const int64_t ld = n;
  cudaError_t e;
  for (int64_t gi = 0; gi < ngroups; ++gi) {
    const int64_t g = trans ? gi : ngroups - 1 - gi;
    const int64_t c0 = g * k;
    const int kg = (int)((nref - c0) < k ? (nref - c0) : k);
    const int64_t o = c0 + b, m = n - o;
    const int np = (kg + b - 1) / b;
    // 1. explicit Y (staircase), W = 0
    {
      int blocks = (int)((m * kg + 255) / 256);
      if (blocks > 16 * num_sms()) blocks = 16 * num_sms();
      bt_build_y_kernel<<<blocks, 256, 0, st>>>(m, kg, A + o + c0 * lda, lda, w.Y, ld);
      count_launches(1);
      if ((e = cudaGetLastError()) != cudaSuccess) return e;
      if ((e = cudaMemset2DAsync(w.W, sizeof(double) * ld, 0, sizeof(double) * m, kg, st)) != cudaSuccess) return e;
    }
    // 2. per panel: Gram, T (dlarft), W_p = Y_p T_p
    for (int p = 0; p < np; ++p) {
      const int t0 = p * b, bp = (kg - t0) < b ? (kg - t0) : b;
      const double* Yp = w.Y + t0 + (int64_t)t0 * ld;
      if ((e = mm(OP_T, OP_N, bp, bp, m - t0, 1.0, Yp, ld, Yp, ld, 0.0, w.G + (size_t)p * b * b, b, w.part,
                  w.part_elems, st)) != cudaSuccess)
        return e;
    }
    bt_tfactor_kernel<<<np, 128, 0, st>>>(b, kg, w.G, tau1 + c0, w.T);
    count_launches(1);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    for (int p = 0; p < np; ++p) {
      const int t0 = p * b, bp = (kg - t0) < b ? (kg - t0) : b;
      if ((e = mm(OP_N, OP_N, m - t0, bp, bp, 1.0, w.Y + t0 + (int64_t)t0 * ld, ld, w.T + (size_t)p * b * b, b,
                  0.0, w.W + t0 + (int64_t)t0 * ld, ld, w.part, w.part_elems, st)) != cudaSuccess)
        return e;
    }
    // 3. Alg. 3 merge, level by level: W_R -= W_L (Y_L^T W_R)
    for (int wl = b; wl < kg; wl *= 2) {
      for (int t0 = 0; t0 + wl < kg; t0 += 2 * wl) {
        const int tr = t0 + wl, wr = (kg - tr) < wl ? (kg - tr) : wl;
        // S (wl x wr) = Y(tr:, t0:t0+wl)^T W(tr:, tr:tr+wr)   (W_R is zero above row tr)
        if ((e = mm(OP_T, OP_N, wl, wr, m - tr, 1.0, w.Y + tr + (int64_t)t0 * ld, ld, w.W + tr + (int64_t)tr * ld,
                    ld, 0.0, w.S, wl, w.part, w.part_elems, st)) != cudaSuccess)
          return e;
        // W(t0:, tr:tr+wr) -= W(t0:, t0:t0+wl) S   (W_L is zero above row t0)
        if ((e = mm(OP_N, OP_N, m - t0, wr, wl, -1.0, w.W + t0 + (int64_t)t0 * ld, ld, w.S, wl, 1.0,
                    w.W + t0 + (int64_t)tr * ld, ld, w.part, w.part_elems, st)) != cudaSuccess)
          return e;
      }
    }
    // 4. C(o:, :) -= W (Y^T C)   or   C(o:, :) -= Y (W^T C)
    const double* L1 = trans ? w.W : w.Y;
    const double* L2 = trans ? w.Y : w.W;
    if ((e = mm(OP_T, OP_N, kg, ncols, m, 1.0, L1, ld, C + o, ldc, 0.0, w.X, kg, w.part, w.part_elems, st)) !=
        cudaSuccess)
      return e;
    if ((e = mm(OP_N, OP_N, m, ncols, kg, -1.0, L2, ld, w.X, kg, 1.0, C + o, ldc, w.part, w.part_elems, st)) !=
        cudaSuccess)
      return e;
  }
  return cudaSuccess;
}

// ================================================================================ Q2 (BC)
__host__ __device__ inline int64_t bt_steps(int64_t n, int b, int64_t s) {
  if (b < 2 || s < 0 || s > n - 3) return 0;
  return (n - 3 - s) / b + 1;
}
__host__ __device__ inline int64_t bt_F(int64_t x, int b) {   // sum_{u=0}^{x} (floor(u/b) + 1)
  if (x < 0) return 0;
  const int64_t q = x / b, r = x - q * b;
  return (int64_t)b * q * (q - 1) / 2 + q * (r + 1) + x + 1;
}
__host__ __device__ inline int64_t bt_offset(int64_t n, int b, int64_t s) {   // S(s), reading R7
  if (b < 2) return 0;
  return bt_F(n - 3, b) - bt_F(n - 3 - s, b);
}

constexpr int BT_NT = 256;   // 8 warps x 4 column lanes: 32 columns per CTA (16-column CTAs measured slower)

// QR rows per thread; the group window holds 8*QR >= b + nb - 1 rows.
__device__ __forceinline__ void bt_cp8(double* dst, const double* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}

template <int QR, int CC>
__global__ void __launch_bounds__(BT_NT, 1) bc_bt_kernel(int64_t n, int b, int nb, const double* __restrict__ V2,
                                                        const double* __restrict__ tau2, int trans, int64_t ncols,
                                                        double* C, int64_t ldc) {
  constexpr int RW = 8 * QR;   // window rows
  constexpr int NP = QR / 2;   // row pairs per thread: thread (rg, cl) holds rows 16 p + 2 rg + {0, 1}, p < NP, of
                               // its CC columns -- the 8 row-group lanes of a column cover 16 consecutive rows
  constexpr int COLS = (BT_NT / 8) * CC;   // columns per CTA: (BT_NT / 32) warps x 4 column lanes x CC per thread
  // two buffers of the group's reflectors in window shape, Vw[j][r] = v_j[r - j] (zero outside [j, j+b): the zero
  // rows are written once, the b rows of vector j are refilled per group by cp.async), nb x RW each; 2 x nb taus;
  // the block's per-sweep V2 offsets S(s0+j) and step counts
  extern __shared__ __align__(16) double sv[];
  double* stau = sv + 2 * (size_t)nb * RW;
  int64_t* soff = reinterpret_cast<int64_t*>(stau + 2 * nb);
  int64_t* sst = soff + nb;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int rg = lane >> 2, cl = lane & 3;
  double* Cc[CC];
  bool colok[CC];
#pragma unroll
  for (int u = 0; u < CC; ++u) {
    const int64_t col = (int64_t)blockIdx.x * COLS + (warp * 4 + cl) * CC + u;
    colok[u] = col < ncols;
    Cc[u] = C + (colok[u] ? col : 0) * ldc;
  }
  const int64_t nsw = n - 2;   // sweeps 0 .. n-3
  const int64_t nblk = (nsw + nb - 1) / nb;
  constexpr int NWB = BT_NT / 32;
  for (int i = threadIdx.x; i < 2 * nb * RW; i += BT_NT) sv[i] = 0.0;
  for (int64_t bi = 0; bi < nblk; ++bi) {
    const int64_t blk = trans ? bi : nblk - 1 - bi;
    const int64_t s0 = blk * nb;
    const int nbb = (int)((nsw - s0) < nb ? (nsw - s0) : nb);
    const int64_t M = bt_steps(n, b, s0);   // groups of the block (sweep s0 has the most steps)
    __syncthreads();   // previous block done with soff / the buffers
    for (int j = threadIdx.x; j < nbb; j += BT_NT) {
      soff[j] = bt_offset(n, b, s0 + j);
      sst[j] = bt_steps(n, b, s0 + j);
    }
    __syncthreads();
    // group gi's reflectors into buffer gi & 1 (asynchronous; its existence decides the tau slot only: a missing
    // step gets tau = 0 and is skipped, whatever the buffer holds)
    auto stage = [&](int64_t gi) {
      const int64_t m = trans ? M - 1 - gi : gi;
      double* buf = sv + (size_t)(gi & 1) * nb * RW;
      double* tb = stau + (gi & 1) * nb;
      for (int j = warp; j < nbb; j += NWB) {
        const bool ex = m < sst[j];
        if (ex) {
          const double* src = V2 + (soff[j] + m) * b;
          double* dst = buf + (size_t)j * RW + j;
          for (int i = lane; i < b; i += 32) bt_cp8(dst + i, src + i);
          if (lane == 0) bt_cp8(tb + j, tau2 + soff[j] + m);
        } else if (lane == 0) {
          tb[j] = 0.0;
        }
      }
      asm volatile("cp.async.commit_group;\n" ::: "memory");
    };
    stage(0);
    for (int64_t gi = 0; gi < M; ++gi) {
      const int64_t m = trans ? M - 1 - gi : gi;
      const int64_t w0 = s0 + 1 + m * b;   // first row of the group window
      if (gi + 1 < M) {
        stage(gi + 1);
        asm volatile("cp.async.wait_group 1;\n" ::: "memory");
      } else {
        asm volatile("cp.async.wait_group 0;\n" ::: "memory");
      }
      __syncthreads();   // group gi's reflectors visible to all
      const double* vbuf = sv + (size_t)(gi & 1) * nb * RW;
      const double* tbuf = stau + (gi & 1) * nb;
      // the window rows of this thread: w0 + 16 p + 2 rg + h, for each of its CC columns
      double x[CC][QR];
#pragma unroll
      for (int u = 0; u < CC; ++u)
#pragma unroll
        for (int p = 0; p < NP; ++p)
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int64_t r = w0 + 16 * p + 2 * rg + h;
            x[u][2 * p + h] = (colok[u] && r < n) ? Cc[u][r] : 0.0;
          }
      // G_m C applies H_{s0+nbb-1,m} first;  G_m^T C applies H_{s0,m} first
      for (int jj = 0; jj < nbb; ++jj) {
        const int j = trans ? jj : nbb - 1 - jj;
        const double tau = tbuf[j];
        if (tau == 0.0) continue;
        const double2* vj = reinterpret_cast<const double2*>(vbuf + (size_t)j * RW + 2 * rg);
        double vv[QR];
#pragma unroll
        for (int p = 0; p < NP; ++p) {
          const double2 t = vj[8 * p];   // rows 16 p + 2 rg, +1
          vv[2 * p] = t.x;
          vv[2 * p + 1] = t.y;
        }
        double d[CC];
#pragma unroll
        for (int u = 0; u < CC; ++u) {
          double d0 = 0.0, d1 = 0.0;
#pragma unroll
          for (int p = 0; p < NP; ++p) {
            d0 = fma(vv[2 * p], x[u][2 * p], d0);
            d1 = fma(vv[2 * p + 1], x[u][2 * p + 1], d1);
          }
          d[u] = d0 + d1;
        }
#pragma unroll
        for (int u = 0; u < CC; ++u) d[u] += __shfl_xor_sync(0xffffffffu, d[u], 4);
#pragma unroll
        for (int u = 0; u < CC; ++u) d[u] += __shfl_xor_sync(0xffffffffu, d[u], 8);
#pragma unroll
        for (int u = 0; u < CC; ++u) d[u] += __shfl_xor_sync(0xffffffffu, d[u], 16);
#pragma unroll
        for (int u = 0; u < CC; ++u) {
          const double td = tau * d[u];
#pragma unroll
          for (int q = 0; q < QR; ++q) x[u][q] = fma(-td, vv[q], x[u][q]);
        }
      }
#pragma unroll
      for (int u = 0; u < CC; ++u)
#pragma unroll
        for (int p = 0; p < NP; ++p)
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int64_t r = w0 + 16 * p + 2 * rg + h;
            if (colok[u] && r < n) Cc[u][r] = x[u][2 * p + h];
          }
      __syncthreads();   // every warp is done with buffer gi & 1 before stage(gi + 2) refills it
    }
  }
}

// window rows RW = 8 QR: about b + 32, so a block holds ~33 sweeps and a reflector (b rows) covers most of the
// window (round 2 first used 2b rows: half of every dot and update multiplied zeros, ncu: FP64 pipe 28 % busy for
// 10 % useful flops)
static int bc_bt_qr(int b) { return b <= 32 ? 8 : (b <= 64 ? 12 : (b <= 128 ? 20 : 36)); }
static int bc_bt_rw(int b) { return 8 * bc_bt_qr(b); }

int bc_bt_nb(int b) {
  // window RW = 8*QR rows >= b + nb - 1; two buffers of nb staged window-shaped vectors (2 nb x RW doubles) fit in
  // 200 KB of shared memory
  const int rw = bc_bt_rw(b);
  int nb = rw - b + 1;
  const int cap = (int)(200 * 1024 / (16 * (size_t)rw)) - 2;
  if (nb > cap) nb = cap;
  static const char* ne = getenv("TRID_BT_NB");   // A/B: sweeps per block
  if (ne && atoi(ne) >= 1 && atoi(ne) < nb) nb = atoi(ne);
  return nb < 1 ? 1 : nb;
}

cudaError_t bc_backtransform(int64_t n, int b, const double* V2, const double* tau2, int trans, int64_t ncols,
                             double* C, int64_t ldc, cudaStream_t st) {
  if (n < 3 || b < 2 || ncols <= 0) return cudaSuccess;
  const int nb = bc_bt_nb(b);
  const size_t smem = sizeof(double) * (2 * (size_t)nb * bc_bt_rw(b) + 2 * (size_t)nb) + 2 * sizeof(int64_t) * nb;
  // one column per thread; TRID_BT_CC=2 (A/B, b <= 64) gives each thread two columns -- two independent reflector
  // chains per warp -- measured slower at n = 8192 (345 vs 317 ms: half the CTAs, same per-reflector latency)
  static const char* ce = getenv("TRID_BT_CC");
  const int cc = (ce && atoi(ce) == 2 && b <= 64) ? 2 : 1;
  const int cols = (BT_NT / 8) * cc;
  const int64_t grid = (ncols + cols - 1) / cols;
  const int qr = bc_bt_qr(b);
  const void* fn = qr == 8 ? (cc == 2 ? (const void*)bc_bt_kernel<8, 2> : (const void*)bc_bt_kernel<8, 1>)
                 : qr == 12 ? (cc == 2 ? (const void*)bc_bt_kernel<12, 2> : (const void*)bc_bt_kernel<12, 1>)
                 : qr == 20 ? (const void*)bc_bt_kernel<20, 1> : (const void*)bc_bt_kernel<36, 1>;
  static DeviceOnce attrs[6];
  const int ai = qr == 8 ? (cc == 2 ? 0 : 1) : qr == 12 ? (cc == 2 ? 2 : 3) : qr == 20 ? 4 : 5;
  cudaError_t e = attrs[ai]([&] {
    return cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
  });
  if (e != cudaSuccess) return e;
  if (qr == 8 && cc == 2)
    bc_bt_kernel<8, 2><<<(unsigned)grid, BT_NT, smem, st>>>(n, b, nb, V2, tau2, trans, ncols, C, ldc);
  else if (qr == 8)
    bc_bt_kernel<8, 1><<<(unsigned)grid, BT_NT, smem, st>>>(n, b, nb, V2, tau2, trans, ncols, C, ldc);
  else if (qr == 12 && cc == 2)
    bc_bt_kernel<12, 2><<<(unsigned)grid, BT_NT, smem, st>>>(n, b, nb, V2, tau2, trans, ncols, C, ldc);
  else if (qr == 12)
    bc_bt_kernel<12, 1><<<(unsigned)grid, BT_NT, smem, st>>>(n, b, nb, V2, tau2, trans, ncols, C, ldc);
  else if (qr == 20)
    bc_bt_kernel<20, 1><<<(unsigned)grid, BT_NT, smem, st>>>(n, b, nb, V2, tau2, trans, ncols, C, ldc);
  else
    bc_bt_kernel<36, 1><<<(unsigned)grid, BT_NT, smem, st>>>(n, b, nb, V2, tau2, trans, ncols, C, ldc);
  count_launches(1);
  return cudaGetLastError();
}

}  // namespace trid
