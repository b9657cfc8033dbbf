// gemm.cu — FP64 DMMA contraction engine for the DBBR hot path.
//
// One templated CTA-tile mainloop (cp.async 3-stage smem ring, DMMA m16n8k8 f64 from padded smem
// fragments) serves:
//   * the deferred syr2k  C -= Y Z^T + Z Y^T, lower triangle only, triangular tile grid  (Alg. 1 l.15,
//     Fig. 7: independent square tiles, reorderable)
//   * the next-panel update                                                    (Alg. 1 l.8-12)
//   * W = Y T, corrections and Z = X - 1/2 Y (W^T X)                            (Eq. (1))
// (the SYMM X = A W of the Z builder runs on the warp-specialized engine, gemm_ws.cu)
// Padded smem strides (4 mod 16 doubles) keep 64-bit DMMA fragment loads bank-conflict free.
#include "common.cuh"
#include "gemm.cuh"
#include "prof.cuh"

namespace trid {

constexpr int BK = 16;
constexpr int STAGES = 3;

// Leading dimensions are == 4 (mod 16) doubles: a 64-bit fragment load is served per half-warp
// (4 rows g x 4 k-lanes t); stride 4 (mod 16) puts those 16 addresses on 16 distinct bank pairs.
template <int BM, int OPA>
struct ATile {
  static constexpr int LD = OPA == OP_N ? BM + 4 : BK + 4;
  static constexpr int ELEMS = OPA == OP_N ? BK * (BM + 4) : BM * (BK + 4);
  __device__ static __forceinline__ int idx(int r, int k) { return OPA == OP_N ? k * LD + r : r * LD + k; }
};
template <int BN, int OPB>
struct BTile {
  static constexpr int LD = OPB == OP_T ? BN + 4 : BK + 4;
  static constexpr int ELEMS = OPB == OP_T ? BK * (BN + 4) : BN * (BK + 4);
  __device__ static __forceinline__ int idx(int k, int c) { return OPB == OP_T ? k * LD + c : c * LD + k; }
};

template <int BM, int BN>
constexpr int stage_elems_max() {
  return (ATile<BM, OP_N>::ELEMS > ATile<BM, OP_T>::ELEMS ? ATile<BM, OP_N>::ELEMS : ATile<BM, OP_T>::ELEMS) +
         (BTile<BN, OP_N>::ELEMS > BTile<BN, OP_T>::ELEMS ? BTile<BN, OP_N>::ELEMS : BTile<BN, OP_T>::ELEMS);
}

// MASK: 0 none; 1 keep (k <= row)  [SYMM row strip incl. diagonal]; 2 keep (k > row) [SYMM column strip]
template <int BM, int BN, int NT, int OPA, int OPB, int MASK>
__device__ __forceinline__ void load_stage(double* As, double* Bs, const double* A, int64_t lda, const double* B,
                                           int64_t ldb, int64_t m0, int64_t n0, int64_t M, int64_t N, int64_t k0,
                                           int64_t kend, const double* A2 = nullptr, int64_t msplit = INT64_MAX) {
  const int tid = threadIdx.x;
#pragma unroll
  for (int e = tid; e < BM * BK; e += NT) {
    int r, kk;
    if (OPA == OP_N) { r = e % BM; kk = e / BM; } else { kk = e % BK; r = e / BK; }
    const int64_t row = m0 + r, k = k0 + kk;
    bool p = row < M && k < kend;
    if (MASK == 1) p = p && (k <= row);
    if (MASK == 2) p = p && (k > row);
    const double* src = A;
    if (p) {
      // rows >= msplit come from A2 (row - msplit): two stacked operands in one launch
      const double* Ab = row < msplit ? A : A2;
      const int64_t rr = row < msplit ? row : row - msplit;
      src = OPA == OP_N ? Ab + rr + k * lda : Ab + k + rr * lda;
    }
    cp_async8(As + ATile<BM, OPA>::idx(r, kk), src, p);
  }
#pragma unroll
  for (int e = tid; e < BN * BK; e += NT) {
    int c, kk;
    if (OPB == OP_T) { c = e % BN; kk = e / BN; } else { kk = e % BK; c = e / BK; }
    const int64_t col = n0 + c, k = k0 + kk;
    const bool p = col < N && k < kend;
    const double* src = B;
    if (p) src = OPB == OP_N ? B + k + col * ldb : B + col + k * ldb;
    cp_async8(Bs + BTile<BN, OPB>::idx(kk, c), src, p);
  }
}

// Accumulate op(A)[m0:m0+BM, kbeg:kend] * op(B)[kbeg:kend, n0:n0+BN] into acc.
template <int BM, int BN, int WGM, int WGN, int OPA, int OPB, int MASK>
__device__ __forceinline__ void mainloop(double (&acc)[BM / WGM / 16][BN / WGN / 8][4], double* smem, const double* A,
                                         int64_t lda, const double* B, int64_t ldb, int64_t m0, int64_t n0,
                                         int64_t M, int64_t N, int64_t kbeg, int64_t kend,
                                         const double* A2 = nullptr, int64_t msplit = INT64_MAX) {
  constexpr int NT = WGM * WGN * 32;
  constexpr int WTM = BM / WGM, WTN = BN / WGN;
  constexpr int MT = WTM / 16, NTL = WTN / 8;
  constexpr int AE = ATile<BM, OPA>::ELEMS, BE = BTile<BN, OPB>::ELEMS;
  if (kend <= kbeg) return;
  const int ntile = (int)((kend - kbeg + BK - 1) / BK);
  double* As = smem;
  double* Bs = smem + STAGES * AE;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int wm = warp % WGM, wn = warp / WGM;
  const int g = lane >> 2, t = lane & 3;
  __syncthreads();  // previous users of smem are done
#pragma unroll
  for (int s = 0; s < STAGES - 1; ++s) {
    if (s < ntile)
      load_stage<BM, BN, NT, OPA, OPB, MASK>(As + s * AE, Bs + s * BE, A, lda, B, ldb, m0, n0, M, N, kbeg + s * BK,
                                             kend, A2, msplit);
    cp_async_commit();
  }
  for (int it = 0; it < ntile; ++it) {
    cp_async_wait<STAGES - 2>();
    __syncthreads();
    const int nxt = it + STAGES - 1;
    if (nxt < ntile) {
      const int st = nxt % STAGES;
      load_stage<BM, BN, NT, OPA, OPB, MASK>(As + st * AE, Bs + st * BE, A, lda, B, ldb, m0, n0, M, N,
                                             kbeg + (int64_t)nxt * BK, kend, A2, msplit);
    }
    cp_async_commit();
    const double* Ast = As + (it % STAGES) * AE;
    const double* Bst = Bs + (it % STAGES) * BE;
    // k4 sub-steps outermost: the MT*NTL accumulators are independent between two uses, so the
    // DMMA pipe never waits on its own previous result (SASS DMMA.8x8x4 latency ~13-26 cycles).
#pragma unroll
    for (int ks = 0; ks < BK; ks += 4) {
      double a0[MT], a1[MT], bf[NTL];
#pragma unroll
      for (int mt = 0; mt < MT; ++mt) {
        const int rr = wm * WTM + mt * 16 + g;
        a0[mt] = Ast[ATile<BM, OPA>::idx(rr, ks + t)];
        a1[mt] = Ast[ATile<BM, OPA>::idx(rr + 8, ks + t)];
      }
#pragma unroll
      for (int nt = 0; nt < NTL; ++nt) bf[nt] = Bst[BTile<BN, OPB>::idx(ks + t, wn * WTN + nt * 8 + g)];
#pragma unroll
      for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NTL; ++nt) dmma_16x8x4(acc[mt][nt], a0[mt], a1[mt], bf[nt]);
    }
  }
  cp_async_wait<0>();
}

__device__ __forceinline__ void tri_tile(int64_t t, int& tm, int& tn) {
  int64_t r = (int64_t)((sqrt(8.0 * (double)t + 1.0) - 1.0) * 0.5);
  while (r * (r + 1) / 2 > t) --r;
  while ((r + 1) * (r + 2) / 2 <= t) ++r;
  tm = (int)r;
  tn = (int)(t - r * (r + 1) / 2);
}

template <int BM, int BN, int WGM, int WGN, int OPA, int OPB>
__global__ void __launch_bounds__(WGM* WGN * 32, (BM * BN <= 4096 ? 3 : 2)) gemm_kernel(GemmArgs a) {
  constexpr int WTM = BM / WGM, WTN = BN / WGN;
  constexpr int MT = WTM / 16, NTL = WTN / 8;
  extern __shared__ __align__(16) double smem[];
  int tm, tn;
  if (a.tri) {
    tri_tile(blockIdx.x, tm, tn);
  } else {
    tm = blockIdx.x;
    tn = blockIdx.y;
  }
  const int64_t m0 = (int64_t)tm * BM, n0 = (int64_t)tn * BN;
  if (a.lower && m0 + BM - 1 + a.diag_off < n0) return;
  double acc[MT][NTL][4];
#pragma unroll
  for (int i = 0; i < MT; ++i)
#pragma unroll
    for (int j = 0; j < NTL; ++j)
#pragma unroll
      for (int q = 0; q < 4; ++q) acc[i][j][q] = 0.0;

  // split-K over the concatenated, BK-aligned segments
  const int64_t kt0 = (a.K[0] + BK - 1) / BK, kt1 = a.nseg > 1 ? (a.K[1] + BK - 1) / BK : 0;
  const int64_t total = kt0 + kt1;
  const int z = blockIdx.z;
  const int64_t per = (total + a.splits - 1) / a.splits;
  const int64_t tb = (int64_t)z * per, te = (tb + per < total) ? tb + per : total;
  if (tb < kt0) {
    const int64_t e = te < kt0 ? te : kt0;
    const int64_t kb = tb * BK, ke = (e * BK < a.K[0]) ? e * BK : a.K[0];
    mainloop<BM, BN, WGM, WGN, OPA, OPB, 0>(acc, smem, a.A[0], a.lda[0], a.B[0], a.ldb[0], m0, n0, a.M, a.N, kb, ke,
                                            a.A2m, a.msplit);
  }
  if (te > kt0) {
    const int64_t b0 = (tb > kt0 ? tb : kt0) - kt0, e = te - kt0;
    const int64_t kb = b0 * BK, ke = (e * BK < a.K[1]) ? e * BK : a.K[1];
    mainloop<BM, BN, WGM, WGN, OPA, OPB, 0>(acc, smem, a.A[1], a.lda[1], a.B[1], a.ldb[1], m0, n0, a.M, a.N, kb, ke);
  }

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int wm = warp % WGM, wn = warp / WGM;
  const int g = lane >> 2, t = lane & 3;
#pragma unroll
  for (int mt = 0; mt < MT; ++mt)
#pragma unroll
    for (int nt = 0; nt < NTL; ++nt)
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int64_t r = m0 + wm * WTM + mt * 16 + g + (i >= 2 ? 8 : 0);
        const int64_t c = n0 + wn * WTN + nt * 8 + 2 * t + (i & 1);
        if (r < a.M && c < a.N && (!a.lower || r + a.diag_off >= c)) {
          if (a.splits > 1) {
            a.part[z * a.part_stride + r + c * a.part_ld] = acc[mt][nt][i];
          } else {
            double v = a.alpha * acc[mt][nt][i];
            if (a.beta != 0.0) v += a.beta * a.Cin[r + c * a.ldcin];
            a.C[r + c * a.ldc] = v;
          }
        }
      }
  if (a.splits > 1 && a.sem) {
    // the last split to finish this tile reduces all partials in fixed order z = 0..splits-1 (deterministic;
    // saves the separate reduction launch).  The counter is reset for the next launch.
    __shared__ int s_last;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned* cnt = a.sem + (a.tri ? (int64_t)blockIdx.x : (int64_t)blockIdx.y * gridDim.x + blockIdx.x);
      const unsigned prev = atomicAdd(cnt, 1u);
      s_last = prev == (unsigned)a.splits - 1u;
      if (s_last) *cnt = 0u;
    }
    __syncthreads();
    if (s_last) {
      __threadfence();
      for (int e = threadIdx.x; e < BM * BN; e += WGM * WGN * 32) {
        const int64_t r = m0 + e % BM, c = n0 + e / BM;
        if (r >= a.M || c >= a.N || (a.lower && r + a.diag_off < c)) continue;
        double sum = 0.0;
        for (int q = 0; q < a.splits; ++q) sum += __ldcg(a.part + q * a.part_stride + r + c * a.part_ld);
        double v = a.alpha * sum;
        if (a.beta != 0.0) v += a.beta * a.Cin[r + c * a.ldcin];
        a.C[r + c * a.ldc] = v;
      }
    }
  }
}

__global__ void reduce_partials_kernel(GemmArgs a) {
  const int64_t total = a.M * a.N;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = idx % a.M, c = idx / a.M;
    if (a.lower && r + a.diag_off < c) continue;
    // fixed order z = 0..splits-1; 8 independent loads in flight per batch (the adds stay in order, so the
    // result is bitwise that of the plain loop, without one L2 round trip per split)
    double s = 0.0;
    const double* pp = a.part + r + c * a.part_ld;
    int z = 0;
    for (; z + 8 <= a.splits; z += 8) {
      double q[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) q[u] = pp[(int64_t)(z + u) * a.part_stride];
#pragma unroll
      for (int u = 0; u < 8; ++u) s += q[u];
    }
    for (; z < a.splits; ++z) s += pp[(int64_t)z * a.part_stride];
    double v = a.alpha * s;
    if (a.beta != 0.0) v += a.beta * a.Cin[r + c * a.ldcin];
    a.C[r + c * a.ldc] = v;
  }
}

template <int BM, int BN, int WGM, int WGN, int OPA, int OPB>
static cudaError_t launch_tile(const GemmArgs& a, cudaStream_t st) {
  constexpr int NT = WGM * WGN * 32;
  constexpr size_t smem = sizeof(double) * STAGES * (ATile<BM, OPA>::ELEMS + BTile<BN, OPB>::ELEMS);
  static DeviceOnce attr;
  cudaError_t e0 = attr([&] {
    return cudaFuncSetAttribute(gemm_kernel<BM, BN, WGM, WGN, OPA, OPB>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)smem);
  });
  if (e0 != cudaSuccess) return e0;
  const int64_t tm = (a.M + BM - 1) / BM, tn = (a.N + BN - 1) / BN;
  dim3 grid;
  GemmArgs b = a;
  if (a.tri && BM == BN) {
    grid = dim3((unsigned)(tm * (tm + 1) / 2), 1, (unsigned)a.splits);
  } else {
    b.tri = 0;   // rectangular grid; tiles wholly above the diagonal exit at once (a.lower)
    grid = dim3((unsigned)tm, (unsigned)tn, (unsigned)a.splits);
  }
  gemm_kernel<BM, BN, WGM, WGN, OPA, OPB><<<grid, NT, smem, st>>>(b);
  count_launches(1);
  return cudaGetLastError();
}

// All tiles: 128 threads (2 x 2 warps), BK = 16, 3 stages, 2-3 CTAs per SM -- the shape cuBLAS's
// FP64 DGEMM uses on this part (cutlass_80_tensorop_d884gemm_64x128_16x3, DMMA pipe 96% busy).
template <int OPA, int OPB>
static cudaError_t launch_ops(const GemmArgs& a, int tile, cudaStream_t st) {
  switch (tile) {
    case TILE_128x128: return launch_tile<64, 128, 2, 2, OPA, OPB>(a, st);   // "wide": 64 x 128
    case TILE_128x64: return launch_tile<128, 64, 2, 2, OPA, OPB>(a, st);
    default: return launch_tile<64, 64, 2, 2, OPA, OPB>(a, st);
  }
}

cudaError_t gemm(GemmArgs a, int opA, int opB, int tile, cudaStream_t st) {
  if (a.M <= 0 || a.N <= 0) return cudaSuccess;
  if (a.K[0] <= 0 && (a.nseg < 2 || a.K[1] <= 0)) {
    // pure scaling: C = beta * Cin (K == 0); reuse the reduction kernel with zero splits
    GemmArgs r = a;
    r.splits = 0;
    reduce_partials_kernel<<<592, 256, 0, st>>>(r);
    count_launches(1);
    return cudaGetLastError();
  }
  if (a.splits < 1) a.splits = 1;
  cudaError_t e;
  if (opA == OP_N && opB == OP_N) e = launch_ops<OP_N, OP_N>(a, tile, st);
  else if (opA == OP_N && opB == OP_T) e = launch_ops<OP_N, OP_T>(a, tile, st);
  else if (opA == OP_T && opB == OP_N) e = launch_ops<OP_T, OP_N>(a, tile, st);
  else e = launch_ops<OP_T, OP_T>(a, tile, st);
  if (e != cudaSuccess || a.splits == 1 || a.sem) return e;
  int64_t total = a.M * a.N;
  int blocks = (int)((total + 127) / 128);   // small outputs (b x b, k x b): spread over many SMs
  if (blocks > 4 * num_sms() * 8) blocks = 4 * num_sms() * 8;
  reduce_partials_kernel<<<blocks, 128, 0, st>>>(a);
  count_launches(1);
  return cudaGetLastError();
}

int pick_splits(int64_t M, int64_t N, int64_t K, int tile, int64_t max_part_elems) {
  const int bm = tile == TILE_128x64 ? 128 : 64, bn = tile == TILE_128x128 ? 128 : 64;
  const int64_t tiles = ((M + bm - 1) / bm) * ((N + bn - 1) / bn);
  const int64_t target = 2 * kNumSMsB200;   // fixed: the split count decides the summation order
  int64_t s = (target + tiles - 1) / tiles;
  const int64_t maxk = (K + 255) / 256;  // keep >= 256 of K per split
  if (s > maxk) s = maxk;
  if (s * M * N > max_part_elems) s = max_part_elems / (M * N);
  if (s < 1) s = 1;
  if (s > 128) s = 128;
  return (int)s;
}

}  // namespace trid
