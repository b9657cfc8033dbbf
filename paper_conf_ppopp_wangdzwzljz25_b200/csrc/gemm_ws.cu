// gemm_ws.cu — warp-specialized persistent FP64 DMMA contraction engine (the big DBBR contractions).
//
// Why: on sm_100a a DMMA.8x8x4 occupies its SMSP's FP64 tensor path for 16 cycles and the compiler
// encodes that cadence into the issuing warp (stall 15 + NOP), so ONE warp saturates an SMSP and any
// moment where all warps of an SMSP block (CTA barriers, cp.async waits, prologue/epilogue) idles the
// pipe (measured: 72% DMMA-busy with the synchronous 3-stage kernel vs 96% for cuBLAS).  Here:
//   * 1 producer warp streams A/B K-tiles into a STAGES-deep shared-memory ring with cp.async (16-byte
//     when the operands are 16-byte aligned, else 8-byte) and signals full[slot] with
//     cp.async.mbarrier.arrive.noinc; it refills a slot after the consumers' empty[slot] arrivals;
//   * CWM x CWN consumer warps (2 per SMSP) wait only on full[slot]; there is no CTA-wide barrier;
//   * the grid is persistent: each CTA walks work units (tile, split) with stride gridDim.x, so the
//     producer prefetches the next unit while the consumers run the epilogue.
//   * NT contractions on 128 x 128 tiles (the deferred syr2k): producer thread 0 alone stages each operand tile with
//     ONE tensor copy (TMA, cp.async.bulk.tensor.2d from FP64 tensor maps, box {BM + 4, BK}) straight into the
//     padded, bank-conflict-free layout (TRID_WS_TMA=1: one bulk copy per k-row; 0: cp.async);
//   * the SYMM: its m-inner A tiles (row strip, correction operands) by tensor copies registered with expect_tx next
//     to the cp.async producer's noinc arrivals on the same slot barrier (the k-inner operands stay on cp.async);
//   * 128 x 128, 128 x 64 and (N <= 32) 128 x 32 tiles;
//   * epilogue: a thread's Cin values are loaded in batches before any store (Cin may alias C);
//   * triangular unit order grouped in bands of 8 tile rows (L2 reuse of the Y/Z strips: DRAM 65 -> 15 GB).
// A unit's K range is a list of up to two segments; each segment has its own A/B pointers, leading
// dimensions, A access mode (N: m-inner, T: k-inner) and triangle mask (the SYMM row/column strips).
#include "common.cuh"
#include "gemm.cuh"
#include "prof.cuh"

#include <cuda.h>
#include <cudaTypedefs.h>
#include <stdlib.h>

#include <stdint.h>
#include <stdio.h>

#include <mutex>
#include <string>
#include <unordered_map>

namespace trid {

namespace ws {

constexpr int BK = 16;

template <int BM, int BN>
struct Cfg {
  static constexpr int A_LD_N = BM + 4;   // A m-inner:  As[k][m]
  static constexpr int A_LD_T = BK + 4;   // A k-inner:  As[m][k]
  static constexpr int A_ELEMS = (BK * A_LD_N > BM * A_LD_T) ? BK * A_LD_N : BM * A_LD_T;
  static constexpr int B_LD_T = BN + 4;   // B n-inner:  Bs[k][n]   (op(B) = B^T, B is N x K)
  static constexpr int B_LD_N = BK + 4;   // B k-inner:  Bs[n][k]   (op(B) = B,   B is K x N)
  static constexpr int B_ELEMS = (BK * B_LD_T > BN * B_LD_N) ? BK * B_LD_T : BN * B_LD_N;
  static constexpr int STAGE = A_ELEMS + B_ELEMS;
  static constexpr int STAGES = (210 * 1024 / (8 * STAGE)) > 6 ? 6 : (210 * 1024 / (8 * STAGE));
  static constexpr size_t SMEM = sizeof(double) * (size_t)STAGES * STAGE + 16 * STAGES + 64;
};

struct Seg {
  const double* A;
  const double* B;
  int64_t lda, ldb;
  int64_t kb, ke;   // K range [kb, ke)
  int opa;          // OP_N / OP_T
  int mask;         // 0 none, 1 keep k <= row, 2 keep k > row (global row = m0 + r)
  int mapk, mapr;   // multi-GPU: compare cmap(k) / cmap(row) instead of k / row (block-cyclic local columns)
  int seg;          // GEMM segment index (selects the segment's tensor maps)
};

struct WsArgs {
  int64_t M, N;
  int opa;                  // GEMM segments: OP_N (A is M x K) / OP_T (A is K x M)
  int opb;                  // OP_N / OP_T for every segment
  int nseg;                 // GEMM: 1 or 2 segments over the split's K range
  const double* A[2];
  const double* B[2];
  int64_t lda[2], ldb[2], K[2];
  int symm;                 // 1: SYMM X = Asym W (A lower referenced), segments derived per tile
  // symm == 1 only: ncorr > 0 appends two GEMM K-segments CA[i] (M x ncorr, op N, ld ldca) x CB[i] (ncorr x N,
  // op N, ld ldcb) to every row block's K axis (the Z builder's corrections, R4e), chunked across the splits
  int64_t ncorr, ldca, ldcb;
  const double* CA[2];
  const double* CB[2];
  double alpha, beta;
  const double* Cin;
  int64_t ldcin;
  double* C;
  int64_t ldc;
  int lower;
  int64_t diag_off;
  int tri;                  // lower-triangular tile enumeration (BM == BN)
  int tgroup;               // tri: rows per band of the grouped unit order (<= 1: row-major)
  int tiles_m, tiles_n, splits;
  int64_t units;
  double* part;             // split partials: part + z*part_stride, ld part_ld
  int64_t part_ld, part_stride;
  int vec16;                // operands 16-byte aligned (base pointers and leading dimensions even)
  // multi-GPU column map (1D block-cyclic, mg_g ranks, blocks of mg_cb columns, this rank mg_q): local
  // column x (relative to local column mg_lofs) is global column cmap(x) (relative to global mg_gofs).
  // mg_g <= 1: identity.  Used by the lower epilogue mask (C's columns are local) and the SYMM modes 2/3.
  int mg_g, mg_q, mg_cb;
  int64_t mg_lofs, mg_gofs;
  // TMA-staged operands (GEMM segments with A op N and B op T, 128 x 128 tiles, vec16, even M and N: the
  // deferred syr2k): tma = 1: the producer stages every k-row of a tile with one bulk copy (cp.async.bulk) per
  // operand; tma = 2: one tensor copy (cp.async.bulk.tensor.2d) per operand and stage, from the segment's tensor
  // maps tmA / tmB (FP64, dims {rows, K}, box {BM + 4, BK}: the box lands as the padded [BK][BM + 4] stage layout;
  // rows past M / N and k past K are zero-filled by the copy engine)
  int tma;
  CUtensorMap tmA[2], tmB[2];
  // GEMM segment 0 with A op T only, when A2 != nullptr: rows >= msplit of op(A) are rows (row - msplit) of A2 (same
  // ld): two stacked operands [op(A); op(A2)] sharing B in one launch (the Z builder's U = [Z_<^T W; Y_<^T W])
  const double* A2;
  int64_t msplit;
  // symm_tma (SYMM, A op N K-tiles only): the m-inner A tiles of the row strip (A, dims {m, m}) and of the
  // correction segments (CA[i], dims {m, ncorr}) are staged by one tensor copy each (box {BM + 4, BK}, lands as the
  // padded [BK][BM + 4] stage); the transposed column strip, W and CB keep the cp.async producer
  int symm_tma;
  CUtensorMap tmSA, tmSC[2];
};

template <bool MG>
__device__ __forceinline__ int64_t cmap(const WsArgs& a, int64_t x) {
  if (!MG) return x;
  const int64_t X = x + a.mg_lofs, blk = X / a.mg_cb;
  return (blk * a.mg_g + a.mg_q) * a.mg_cb + (X - blk * a.mg_cb) - a.mg_gofs;
}
// number of local columns x in [0, kt) with cmap(x) <= r
template <bool MG>
__device__ __forceinline__ int64_t kcount(const WsArgs& a, int64_t r, int64_t kt) {
  if (r < 0) return 0;
  int64_t c;
  if (!MG) {
    c = r + 1;
  } else {
    const int64_t G = r + a.mg_gofs, B = G / a.mg_cb, w = G - B * a.mg_cb;
    const int64_t nbl = B > a.mg_q ? (B - a.mg_q + a.mg_g - 1) / a.mg_g : 0;
    c = nbl * a.mg_cb + ((B % a.mg_g) == a.mg_q ? w + 1 : 0) - a.mg_lofs;
  }
  return c < 0 ? 0 : (c > kt ? kt : c);
}

__device__ __forceinline__ void tri_unit(int64_t t, int& tm, int& tn) {
  int64_t r = (int64_t)((sqrt(8.0 * (double)t + 1.0) - 1.0) * 0.5);
  while (r * (r + 1) / 2 > t) --r;
  while ((r + 1) * (r + 2) / 2 <= t) ++r;
  tm = (int)r;
  tn = (int)(t - r * (r + 1) / 2);
}

template <int BM, int BN>
__device__ __forceinline__ void unit_geom(const WsArgs& a, int64_t u, int64_t& m0, int64_t& n0, int& z) {
  const int64_t tiles = a.tri ? (int64_t)a.tiles_m * (a.tiles_m + 1) / 2 : (int64_t)a.tiles_m * a.tiles_n;
  z = (int)(u / tiles);
  const int64_t t = u - (int64_t)z * tiles;
  int tm, tn;
  if (a.tri) {
    tri_unit(t, tm, tn);
    if (a.tgroup > 1) {
      // grouped order (L2 reuse): the rows of a band of tgroup tile rows are walked column by column, so the
      // ~148 units in flight touch ~tgroup A strips and ~148 / tgroup B strips instead of one A strip and 148
      // B strips.  The band of unit t is the band of its row-major position (bands hold whole rows).
      const int R0 = tm / a.tgroup * a.tgroup;
      const int nr = (a.tiles_m - R0) < a.tgroup ? (a.tiles_m - R0) : a.tgroup;
      int64_t o = t - (int64_t)R0 * (R0 + 1) / 2;
      if (o < (int64_t)R0 * nr) {
        tn = (int)(o / nr);
        tm = R0 + (int)(o % nr);
      } else {
        o -= (int64_t)R0 * nr;
        int c = R0;
        while (o >= R0 + nr - c) {
          o -= R0 + nr - c;
          ++c;
        }
        tn = c;
        tm = c + (int)o;
      }
    }
  } else {
    tm = (int)(t % a.tiles_m);
    tn = (int)(t / a.tiles_m);
  }
  m0 = (int64_t)tm * BM;
  n0 = (int64_t)tn * BN;
}

// Segments of unit u (identical in producer and consumers).
template <int BM, int BN, bool MG>
__device__ __forceinline__ int unit_segs(const WsArgs& a, int64_t m0, int z, Seg& s0, Seg& s1) {
  if (MG && a.symm >= 2) {
    // multi-GPU SYMM partial over this rank's local columns (mode 2: rows = global, K = local columns,
    // keep cmap(k) <= row; mode 3: rows = local columns, K = global rows, keep k > cmap(row))
    const int64_t rl = (m0 + BM < a.M ? m0 + BM : a.M) - 1;
    int64_t lo, hi;
    if (a.symm == 2) {
      lo = 0;
      hi = kcount<MG>(a, rl, a.K[0]);
    } else {
      lo = (cmap<MG>(a, m0) + 1) / BK * BK;
      hi = a.K[0];
    }
    if (hi <= lo) return 0;
    const int64_t chunk = (hi - lo + a.splits - 1) / a.splits;
    const int64_t cz = (chunk + BK - 1) / BK * BK;
    const int64_t k0 = lo + (int64_t)z * cz, k1 = (k0 + cz < hi) ? k0 + cz : hi;
    if (k1 <= k0) return 0;
    s0 = a.symm == 2 ? Seg{a.A[0], a.B[0], a.lda[0], a.ldb[0], k0, k1, OP_N, 1, 1, 0}
                     : Seg{a.A[0], a.B[0], a.lda[0], a.ldb[0], k0, k1, OP_T, 2, 0, 1};
    return 1;
  }
  if (a.symm) {
    // K chunk z of the strip (+ correction segments): [k0, k1); row strip (k <= row) then column strip (k > row)
    const int64_t ktot = a.K[0] + 2 * a.ncorr;
    const int64_t chunk = (ktot + a.splits - 1) / a.splits;
    const int64_t cz = (chunk + BK - 1) / BK * BK;
    const int64_t k0 = (int64_t)z * cz, k1 = (k0 + cz < a.K[0]) ? k0 + cz : a.K[0];
    if (k0 >= a.K[0]) return 0;
    const int64_t e1 = (k1 < m0 + BM) ? k1 : m0 + BM;
    const int64_t s2 = (k0 > m0) ? k0 : m0;
    const Seg row{a.A[0], a.B[0], a.lda[0], a.ldb[0], k0, e1, OP_N, 1, 0, 0};
    const Seg col{a.A[0], a.B[0], a.lda[0], a.ldb[0], s2, k1, OP_T, 2, 0, 0};
    if (e1 > k0) {
      s0 = row;
      s1 = col;
      return k1 > s2 ? 2 : 1;
    }
    s0 = col;
    return k1 > s2 ? 1 : 0;
  }
  const int64_t kt0 = (a.K[0] + BK - 1) / BK, kt1 = a.nseg > 1 ? (a.K[1] + BK - 1) / BK : 0;
  const int64_t total = kt0 + kt1;
  const int64_t per = (total + a.splits - 1) / a.splits;
  const int64_t tb = (int64_t)z * per, te = (tb + per < total) ? tb + per : total;
  int64_t kb0 = 0, ke0 = 0, kb1 = 0, ke1 = 0;
  if (tb < kt0) {
    const int64_t e = te < kt0 ? te : kt0;
    kb0 = tb * BK;
    ke0 = (e * BK < a.K[0]) ? e * BK : a.K[0];
  }
  if (te > kt0) {
    const int64_t b0 = (tb > kt0 ? tb : kt0) - kt0, e = te - kt0;
    kb1 = b0 * BK;
    ke1 = (e * BK < a.K[1]) ? e * BK : a.K[1];
  }
  const Seg g0{a.A[0], a.B[0], a.lda[0], a.ldb[0], kb0, ke0, a.opa, 0, 0, 0};
  const Seg g1{a.A[1], a.B[1], a.lda[1], a.ldb[1], kb1, ke1, a.opa, 0, 0, 0, 1};
  if (ke0 > kb0) {
    s0 = g0;
    s1 = g1;
    return ke1 > kb1 ? 2 : 1;
  }
  s0 = g1;
  return ke1 > kb1 ? 1 : 0;
}

// Correction segment i (0, 1) of unit chunk z (symm == 1, ncorr > 0): the part of [m + i ncorr, m + (i+1) ncorr)
// inside the chunk, in the segment's own k coordinates.
__device__ __forceinline__ bool corr_seg(const WsArgs& a, int z, int i, Seg& sg) {
  const int64_t ktot = a.K[0] + 2 * a.ncorr;
  const int64_t chunk = (ktot + a.splits - 1) / a.splits;
  const int64_t cz = (chunk + BK - 1) / BK * BK;
  const int64_t k0 = (int64_t)z * cz, k1 = (k0 + cz < ktot) ? k0 + cz : ktot;
  const int64_t s0 = a.K[0] + i * a.ncorr, s1 = s0 + a.ncorr;
  const int64_t b0 = k0 > s0 ? k0 : s0, e0 = k1 < s1 ? k1 : s1;
  if (e0 <= b0) return false;
  sg = Seg{a.CA[i], a.CB[i], a.ldca, a.ldcb, b0 - s0, e0 - s0, OP_N, 0, 0, 0, 2 + i};
  return true;
}

__device__ __forceinline__ void cp16(double* dst, const double* src, int bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(smem_u32(dst)), "l"(src), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void cp8(double* dst, const double* src, int bytes) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(smem_u32(dst)), "l"(src), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void cp_arrive_noinc(uint64_t* bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, unsigned bytes) {
  asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// 2D tensor copy global -> shared (TMA), completing on an mbarrier; c0 = innermost (row) coordinate
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, int c0, int c1, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];\n" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}

// ---- producer fast paths (16-byte aligned operands, no triangle mask): per-thread offsets are fixed,
// every copy of a stage is one address add + one cp.async with compile-time shared-memory offsets.
// NP producer threads (pt in [0, NP)).  m-inner tile (A op N / B op T): R rows (H = R/2 pairs) x BK.
template <int R, int LD, int NP>
__device__ __forceinline__ void load_minner16(double* T, const double* base, int64_t ld, int64_t r0, int64_t rmax,
                                              int64_t k0, int64_t kend, int pt) {
  constexpr int H = R / 2;
  constexpr int NCP = H * BK / NP;
  static_assert(NP % H == 0 || H % NP == 0, "producer mapping");
  constexpr int Q = H % NP == 0 ? H / NP : 1;          // row groups per thread when H >= NP
  constexpr int KS = NP % H == 0 ? NP / H : 0;         // k rows advanced per copy when NP >= H
  const int rp = NP % H == 0 ? pt % H : pt;            // base pair
  const int kb = NP % H == 0 ? pt / H : 0;
  int bytes_q[Q];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const int64_t row = r0 + 2 * (rp + NP * q);
    bytes_q[q] = row + 1 < rmax ? 16 : (row < rmax ? 8 : 0);
  }
  const bool kfull = k0 + BK <= kend;
#pragma unroll
  for (int i = 0; i < NCP; ++i) {
    const int q = i % Q;
    const int kk = (NP % H == 0) ? kb + KS * i : i / Q;
    int bytes = bytes_q[q];
    if (!kfull && k0 + kk >= kend) bytes = 0;
    const int rr = 2 * (rp + NP * q);
    const double* sp = base + r0 + rr + (k0 + kk) * ld;
    cp16(T + kk * LD + rr, bytes ? sp : base, bytes);
  }
}
// k-inner tile (A op T / B op N): R rows of BK contiguous k (BK/2 = 8 pairs per row).
template <int R, int LD, int NP>
__device__ __forceinline__ void load_kinner16(double* T, const double* base, int64_t ld, int64_t r0, int64_t rmax,
                                              int64_t k0, int64_t kend, int pt, const double* base2 = nullptr,
                                              int64_t msplit = INT64_MAX) {
  constexpr int NCP = R * (BK / 2) / NP;
  constexpr int RS = NP / (BK / 2);
  const int kk = 2 * (pt % (BK / 2)), rl = pt / (BK / 2);
  const int kbytes = k0 + kk + 1 < kend ? 16 : (k0 + kk < kend ? 8 : 0);
#pragma unroll
  for (int i = 0; i < NCP; ++i) {
    const int rr = rl + RS * i;
    const int64_t row = r0 + rr;
    const int bytes = row < rmax ? kbytes : 0;
    const double* rp = row < msplit ? base + row * ld : base2 + (row - msplit) * ld;
    cp16(T + rr * LD + kk, bytes ? rp + k0 + kk : base, bytes);
  }
}

// Producer: one K-tile of A and B into stage buffers (NP threads).
template <int BM, int BN, int NP, bool MG>
__device__ __forceinline__ void load_tile(const WsArgs& a, const Seg& s, int64_t k0, int64_t m0, int64_t n0,
                                          double* As, double* Bs, int pt, bool skip_a = false) {
  using C = Cfg<BM, BN>;
  const int64_t kend = s.ke;
  // the triangle masks only bite on K-tiles that overlap the diagonal block [m0, m0 + BM)
  // (with the multi-GPU map: compare cmap(k) / cmap(row); cmap is monotone)
  auto km = [&](int64_t k) { return MG && s.mapk ? cmap<MG>(a, k) : k; };
  auto rm = [&](int64_t r) { return MG && s.mapr ? cmap<MG>(a, r) : r; };
  const bool unmasked = s.mask == 0 || (s.mask == 1 && km(k0 + BK - 1) <= rm(m0)) ||
                        (s.mask == 2 && km(k0) > rm(m0 + BM - 1));
  const bool v16 = a.vec16 && unmasked;
  // ---- A
  if (skip_a) {
    // staged by a tensor copy (the SYMM's row strip / correction operands, see ws_kernel)
  } else if (v16) {
    if (s.opa == OP_N) load_minner16<BM, C::A_LD_N, NP>(As, s.A, s.lda, m0, a.M, k0, kend, pt);
    else if (s.seg == 0 && a.A2)
      load_kinner16<BM, C::A_LD_T, NP>(As, s.A, s.lda, m0, a.M, k0, kend, pt, a.A2, a.msplit);
    else load_kinner16<BM, C::A_LD_T, NP>(As, s.A, s.lda, m0, a.M, k0, kend, pt);
  } else if (s.opa == OP_N) {   // A(m, k) at A[m + k*lda], tile As[k][m]
    for (int e = pt; e < BM * BK; e += NP) {
      const int r = e % BM, kk = e / BM;
      const int64_t row = m0 + r, k = k0 + kk;
      bool p = row < a.M && k < kend;
      if (s.mask == 1) p = p && (km(k) <= rm(row));
      if (s.mask == 2) p = p && (km(k) > rm(row));
      cp8(As + kk * C::A_LD_N + r, p ? s.A + row + k * s.lda : s.A, p ? 8 : 0);
    }
  } else {                      // op(A)(m, k) = A[k + m*lda], tile As[m][k]
    for (int e = pt; e < BM * BK; e += NP) {
      const int kk = e % BK, r = e / BK;
      const int64_t row = m0 + r, k = k0 + kk;
      bool p = row < a.M && k < kend;
      if (s.mask == 1) p = p && (km(k) <= rm(row));
      if (s.mask == 2) p = p && (km(k) > rm(row));
      const double* rp = (s.seg == 0 && a.A2 && row >= a.msplit) ? a.A2 + (row - a.msplit) * s.lda : s.A + row * s.lda;
      cp8(As + r * C::A_LD_T + kk, p ? rp + k : s.A, p ? 8 : 0);
    }
  }
  // ---- B
  if (a.vec16) {
    if (a.opb == OP_T) load_minner16<BN, C::B_LD_T, NP>(Bs, s.B, s.ldb, n0, a.N, k0, kend, pt);
    else load_kinner16<BN, C::B_LD_N, NP>(Bs, s.B, s.ldb, n0, a.N, k0, kend, pt);
  } else if (a.opb == OP_T) {   // B is N x K: B[n + k*ldb], tile Bs[k][n]
    for (int e = pt; e < BN * BK; e += NP) {
      const int c = e % BN, kk = e / BN;
      const int64_t col = n0 + c, k = k0 + kk;
      const bool p = col < a.N && k < kend;
      cp8(Bs + kk * C::B_LD_T + c, p ? s.B + col + k * s.ldb : s.B, p ? 8 : 0);
    }
  } else {                      // B is K x N: B[k + n*ldb], tile Bs[n][k]
    for (int e = pt; e < BN * BK; e += NP) {
      const int kk = e % BK, c = e / BK;
      const int64_t col = n0 + c, k = k0 + kk;
      const bool p = col < a.N && k < kend;
      cp8(Bs + c * C::B_LD_N + kk, p ? s.B + k + col * s.ldb : s.B, p ? 8 : 0);
    }
  }
}

// Consumer: 4 k4-steps of one stage into the warp's accumulators.
template <int BM, int BN, int WTM, int WTN, int OPA, int OPB>
__device__ __forceinline__ void mma_stage(double (&acc)[WTM / 16][WTN / 8][4], const double* As, const double* Bs,
                                          int wm0, int wn0, int g, int t) {
  using C = Cfg<BM, BN>;
  constexpr int MT = WTM / 16, NT = WTN / 8;
#pragma unroll
  for (int ks = 0; ks < BK; ks += 4) {
    double a0[MT], a1[MT], bf[NT];
#pragma unroll
    for (int mt = 0; mt < MT; ++mt) {
      const int r = wm0 + mt * 16 + g;
      if (OPA == OP_N) {
        a0[mt] = As[(ks + t) * C::A_LD_N + r];
        a1[mt] = As[(ks + t) * C::A_LD_N + r + 8];
      } else {
        a0[mt] = As[r * C::A_LD_T + ks + t];
        a1[mt] = As[(r + 8) * C::A_LD_T + ks + t];
      }
    }
#pragma unroll
    for (int nt = 0; nt < NT; ++nt) {
      const int c = wn0 + nt * 8 + g;
      bf[nt] = OPB == OP_T ? Bs[(ks + t) * C::B_LD_T + c] : Bs[c * C::B_LD_N + ks + t];
    }
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
      for (int nt = 0; nt < NT; ++nt) dmma_16x8x4(acc[mt][nt], a0[mt], a1[mt], bf[nt]);
  }
}

constexpr int NPW = 4;   // producer warps (one warpgroup, so setmaxnreg can shrink it)
// Register budget of the 384-thread kernel: launched at 168 regs/thread (64512 per CTA); the producer
// warpgroup drops to 96 and the two consumer warpgroups rise to 200: 128*96 + 256*200 = 63488 <= 64512
// (an increase the freed registers cannot cover blocks setmaxnreg.inc forever).

template <int BM, int BN, int CWM, int CWN, int OPB, bool MG>
__global__ void __launch_bounds__((CWM * CWN + NPW) * 32, 1) ws_kernel(const __grid_constant__ WsArgs a) {
  using C = Cfg<BM, BN>;
  constexpr int NCW = CWM * CWN;
  constexpr int WTM = BM / CWM, WTN = BN / CWN;
  constexpr int MT = WTM / 16, NT = WTN / 8;
  constexpr int STAGES = C::STAGES;
  extern __shared__ __align__(128) double smem[];   // 128-byte aligned stages (tensor copies)
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + (size_t)STAGES * C::STAGE);
  uint64_t* empty = full + STAGES;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], a.tma ? 32 : NPW * 32);   // one arrive per producer thread (TMA: warp 0 only)
      mbar_init(&empty[s], NCW);  // one arrive per consumer warp
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();

  if (warp >= NCW) {
    // ======================= producer warpgroup =======================
    if (NCW == 8) asm volatile("setmaxnreg.dec.sync.aligned.u32 96;\n" ::: "memory");
    const int pt = threadIdx.x - NCW * 32;
    if constexpr (!MG && OPB == OP_T && BM == 128 && BN == 128) {
      if (a.tma) {
        // TMA staging: producer warp 0 alone; per stage, lane 0 issues one bulk copy per k-row of A and of B (the
        // tile's rows of one column: contiguous, 16-byte multiple since M and N are even) straight into the padded
        // stage rows the consumers' DMMA fragment loads expect (no bank conflicts; 32 copies of <= 1 KB per stage
        // instead of 128 threads x 16 cp.async).  Rows past M / N and k past the segment end are zeroed by the
        // warp with generic stores (fenced to the async proxy: the next use of the slot may be a bulk copy).
        // full[slot] expects 32 arrivals: lane 0's expect_tx + 31 plain arrives (each releases its own stores).
        if (pt >= 32) return;
        uint32_t kt = 0;
        for (int64_t u = blockIdx.x; u < a.units; u += gridDim.x) {
          int64_t m0, n0;
          int z;
          unit_geom<BM, BN>(a, u, m0, n0, z);
          if (a.lower && m0 + BM - 1 + a.diag_off < n0) continue;
          Seg s0, s1;
          const int ns = unit_segs<BM, BN, MG>(a, m0, z, s0, s1);
          const int rm = (int)(a.M - m0 < BM ? a.M - m0 : BM), rn = (int)(a.N - n0 < BN ? a.N - n0 : BN);
          auto run = [&](const Seg& sgm) {
            for (int64_t k0 = sgm.kb; k0 < sgm.ke; k0 += BK, ++kt) {
              const int slot = kt % STAGES;
              const uint32_t use = kt / STAGES;
              if (use > 0) mbar_wait(&empty[slot], (use - 1) & 1u);
              double* As = smem + (size_t)slot * C::STAGE;
              double* Bs = As + C::A_ELEMS;
              if (a.tma == 2) {
                // one tensor copy per operand: box {BM + 4, BK} at (row m0 / n0, k0) of the segment's maps
                if (pt == 0) {
                  mbar_arrive_expect_tx(&full[slot], (unsigned)(2 * BK * (BM + 4) * 8));
                  tma_load_2d(As, &a.tmA[sgm.seg], (int)m0, (int)k0, &full[slot]);
                  tma_load_2d(Bs, &a.tmB[sgm.seg], (int)n0, (int)k0, &full[slot]);
                } else {
                  mbar_arrive(&full[slot]);
                }
                continue;
              }
              const int kc = (int)((sgm.ke - k0) < BK ? (sgm.ke - k0) : BK);
              if (kc < BK || rm < BM || rn < BN) {
                for (int kk = 0; kk < BK; ++kk) {
                  const int ra = kk < kc ? rm : 0, rb = kk < kc ? rn : 0;
                  for (int r = ra + pt; r < BM; r += 32) As[kk * C::A_LD_N + r] = 0.0;
                  for (int r = rb + pt; r < BN; r += 32) Bs[kk * C::B_LD_T + r] = 0.0;
                }
                asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
              }
              if (pt == 0) {
                mbar_arrive_expect_tx(&full[slot], (unsigned)(kc * (rm + rn) * 8));
                for (int kk = 0; kk < kc; ++kk) {
                  bulk_g2s(As + kk * C::A_LD_N, sgm.A + m0 + (k0 + kk) * sgm.lda, rm * 8, &full[slot]);
                  bulk_g2s(Bs + kk * C::B_LD_T, sgm.B + n0 + (k0 + kk) * sgm.ldb, rn * 8, &full[slot]);
                }
              } else {
                mbar_arrive(&full[slot]);
              }
            }
          };
          if (ns > 0) run(s0);
          if (ns > 1) run(s1);
        }
        return;
      }
    }
    uint32_t kt = 0;   // global K-tile counter (ring position)
    for (int64_t u = blockIdx.x; u < a.units; u += gridDim.x) {
      int64_t m0, n0;
      int z;
      unit_geom<BM, BN>(a, u, m0, n0, z);
      if (a.lower && m0 + BM - 1 + a.diag_off < cmap<MG>(a, n0)) continue;
      Seg s0, s1;
      const int ns = unit_segs<BM, BN, MG>(a, m0, z, s0, s1);
      auto run = [&](const Seg& sgm) {
        for (int64_t k0 = sgm.kb; k0 < sgm.ke; k0 += BK, ++kt) {
          const int slot = kt % STAGES;
          const uint32_t use = kt / STAGES;
          if (use > 0) mbar_wait(&empty[slot], (use - 1) & 1u);
          double* As = smem + (size_t)slot * C::STAGE;
          bool tma_a = false;
          if constexpr (!MG && OPB == OP_N && BN <= 64) {
            // SYMM: an m-inner A tile that is unmasked and not cut short inside its tensor goes by tensor copy;
            // thread 0 registers its bytes (expect_tx, no arrival) before its own noinc arrival can complete the
            // phase, so the slot cannot complete without the copy
            if (a.symm_tma && sgm.opa == OP_N) {
              const int64_t kext = sgm.seg >= 2 ? a.ncorr : a.K[0];
              const bool unm = sgm.mask == 0 || (sgm.mask == 1 && k0 + BK - 1 <= m0);
              tma_a = unm && (k0 + BK <= sgm.ke || sgm.ke == kext);
              if (tma_a && pt == 0) {
                mbar_expect_tx(&full[slot], (unsigned)((BM + 4) * BK * 8));
                tma_load_2d(As, sgm.seg >= 2 ? &a.tmSC[sgm.seg - 2] : &a.tmSA, (int)m0, (int)k0, &full[slot]);
              }
            }
          }
          load_tile<BM, BN, NPW * 32, MG>(a, sgm, k0, m0, n0, As, As + C::A_ELEMS, pt, tma_a);
          cp_arrive_noinc(&full[slot]);
        }
      };
      if (ns > 0) run(s0);
      if (ns > 1) run(s1);
      if constexpr (BN <= 64 && OPB == OP_N && !MG) {   // the SYMM instantiations only
        if (a.ncorr) {
          Seg c;
          if (corr_seg(a, z, 0, c)) run(c);
          if (corr_seg(a, z, 1, c)) run(c);
        }
      }
    }
    return;
  }
  // ======================= consumers =======================
  if (NCW == 8) asm volatile("setmaxnreg.inc.sync.aligned.u32 200;\n" ::: "memory");
  const int wm = warp % CWM, wn = warp / CWM;
  const int g = lane >> 2, t = lane & 3;
  uint32_t kt = 0;
  for (int64_t u = blockIdx.x; u < a.units; u += gridDim.x) {
    int64_t m0, n0;
    int z;
    unit_geom<BM, BN>(a, u, m0, n0, z);
    if (a.lower && m0 + BM - 1 + a.diag_off < cmap<MG>(a, n0)) continue;
    Seg s0, s1;
    const int ns = unit_segs<BM, BN, MG>(a, m0, z, s0, s1);
    double acc[MT][NT][4];
#pragma unroll
    for (int i = 0; i < MT; ++i)
#pragma unroll
      for (int j = 0; j < NT; ++j)
#pragma unroll
        for (int q = 0; q < 4; ++q) acc[i][j][q] = 0.0;
    auto run = [&](const Seg& sgm) {
      for (int64_t k0 = sgm.kb; k0 < sgm.ke; k0 += BK, ++kt) {
        const int slot = kt % STAGES;
        mbar_wait(&full[slot], (kt / STAGES) & 1u);
        const double* As = smem + (size_t)slot * C::STAGE;
        if (sgm.opa == OP_N) mma_stage<BM, BN, WTM, WTN, OP_N, OPB>(acc, As, As + C::A_ELEMS, wm * WTM, wn * WTN, g, t);
        else mma_stage<BM, BN, WTM, WTN, OP_T, OPB>(acc, As, As + C::A_ELEMS, wm * WTM, wn * WTN, g, t);
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[slot]);
      }
    };
    if (ns > 0) run(s0);
    if (ns > 1) run(s1);
    if constexpr (BN <= 64 && OPB == OP_N && !MG) {   // the SYMM instantiations only
      if (a.ncorr) {
        Seg c;
        if (corr_seg(a, z, 0, c)) run(c);
        if (corr_seg(a, z, 1, c)) run(c);
      }
    }
    // ---- epilogue.  Cin may alias C, so a load issued after a store of the same thread could not be hoisted
    // above it by the compiler (one dependent global round trip per element); the Cin values of EN
    // fragments are loaded first, then combined and stored (MT * NT / EN round trips per tile instead of 64;
    // EN bounded by the register budget next to the accumulators).
    constexpr int EN = NT >= 4 ? (MG ? 1 : 4) : NT;
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
      for (int n0t = 0; n0t < NT; n0t += EN) {
        double cin[EN][4];
        if (a.splits == 1 && a.beta != 0.0) {
#pragma unroll
          for (int q = 0; q < EN; ++q)
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const int64_t r = m0 + wm * WTM + mt * 16 + g + (i >= 2 ? 8 : 0);
              const int64_t c = n0 + wn * WTN + (n0t + q) * 8 + 2 * t + (i & 1);
              cin[q][i] = (r < a.M && c < a.N && (!a.lower || r + a.diag_off >= cmap<MG>(a, c)))
                              ? a.Cin[r + c * a.ldcin]
                              : 0.0;
            }
        }
#pragma unroll
        for (int q = 0; q < EN; ++q)
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const int nt = n0t + q;
            const int64_t r = m0 + wm * WTM + mt * 16 + g + (i >= 2 ? 8 : 0);
            const int64_t c = n0 + wn * WTN + nt * 8 + 2 * t + (i & 1);
            if (r < a.M && c < a.N && (!a.lower || r + a.diag_off >= cmap<MG>(a, c))) {
              if (a.splits > 1) {
                a.part[z * a.part_stride + r + c * a.part_ld] = acc[mt][nt][i];
              } else {
                double v = a.alpha * acc[mt][nt][i];
                if (a.beta != 0.0) v += a.beta * cin[q][i];
                a.C[r + c * a.ldc] = v;
              }
            }
          }
      }
  }
}

__global__ void ws_reduce_kernel(int64_t M, int64_t N, int splits, const double* part, int64_t part_ld,
                                 int64_t part_stride, double alpha, double beta, const double* Cin, int64_t ldcin,
                                 double* C, int64_t ldc, int lower, int64_t diag_off) {
  const int64_t total = M * N;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = idx % M, c = idx / M;
    if (lower && r + diag_off < c) continue;
    // fixed order, 8 loads in flight per batch (bitwise equal to the plain loop)
    double s = 0.0;
    const double* pp = part + r + c * part_ld;
    int z = 0;
    for (; z + 8 <= splits; z += 8) {
      double q[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) q[u] = pp[(int64_t)(z + u) * part_stride];
#pragma unroll
      for (int u = 0; u < 8; ++u) s += q[u];
    }
    for (; z < splits; ++z) s += pp[(int64_t)z * part_stride];
    double v = alpha * s;
    if (beta != 0.0) v += beta * Cin[r + c * ldcin];
    C[r + c * ldc] = v;
  }
}

template <int BM, int BN, int CWM, int CWN, int OPB, bool MG = false>
static cudaError_t launch(WsArgs& a, cudaStream_t st) {
  using C = Cfg<BM, BN>;
  static DeviceOnce attr;
  cudaError_t e0 = attr([] {
    return cudaFuncSetAttribute(ws_kernel<BM, BN, CWM, CWN, OPB, MG>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)C::SMEM);
  });
  if (e0 != cudaSuccess) return e0;
  static const char* genv = getenv("TRID_WS_GROUP");
  a.tgroup = genv ? atoi(genv) : 8;
  a.tiles_m = (int)((a.M + BM - 1) / BM);
  a.tiles_n = (int)((a.N + BN - 1) / BN);
  if (a.tri && BM != BN) a.tri = 0;
  const int64_t tiles = a.tri ? (int64_t)a.tiles_m * (a.tiles_m + 1) / 2 : (int64_t)a.tiles_m * a.tiles_n;
  a.units = tiles * a.splits;
  int64_t grid = a.units < num_sms() ? a.units : num_sms();
  if (grid < 1) return cudaSuccess;
  ws_kernel<BM, BN, CWM, CWN, OPB, MG><<<(unsigned)grid, (CWM * CWN + NPW) * 32, C::SMEM, st>>>(a);
  count_launches(1);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess || a.splits == 1) return e;
  int64_t total = a.M * a.N;
  int blocks = (int)((total + 255) / 256);
  if (blocks > 16 * num_sms()) blocks = 16 * num_sms();
  ws_reduce_kernel<<<blocks, 256, 0, st>>>(a.M, a.N, a.splits, a.part, a.part_ld, a.part_stride, a.alpha, a.beta,
                                           a.Cin, a.ldcin, a.C, a.ldc, a.lower, a.diag_off);
  count_launches(1);
  return cudaGetLastError();
}

static bool al16(const void* p) { return ((uintptr_t)p & 15) == 0; }

// 128 x 32 tiles for N <= 32 (default on; TRID_WS_NARROW=0 falls back to 128 x 64 for A/B).  Read once: the
// split counts (and hence the workspace sizes and the deterministic sums) depend on it.
static bool narrow_tiles() {
  static const bool on = !(getenv("TRID_WS_NARROW") && getenv("TRID_WS_NARROW")[0] == '0');
  return on;
}

// FP64 2D tensor map of a column-major operand X (rows x cols, leading dimension ld): dims {rows, cols}, box
// {128 + 4, BK} (the engine's padded [BK][BM + 4] stage), no swizzle, out-of-bounds elements zero-filled.  The
// driver entry point is resolved once through the runtime (no link against libcuda).
static bool encode_map(CUtensorMap* map, const double* X, int64_t rows, int64_t cols, int64_t ld, unsigned box0,
                       unsigned box1);
static bool encode_rows_map(CUtensorMap* map, const double* X, int64_t rows, int64_t cols, int64_t ld) {
  return encode_map(map, X, rows, cols, ld, 128 + 4, BK);
}
// FP64 2D tensor map of a column-major X (rows x cols, ld), box {box0 rows, box1 columns}, no swizzle, OOB zero
static bool encode_map(CUtensorMap* map, const double* X, int64_t rows, int64_t cols, int64_t ld, unsigned box0,
                       unsigned box1) {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      p = nullptr;
    return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }();
  if (!fn || rows <= 0 || cols <= 0 || rows >= (1ll << 31) || cols >= (1ll << 31)) return false;
  const cuuint64_t dims[2] = {(cuuint64_t)rows, (cuuint64_t)cols};
  const cuuint64_t strides[1] = {(cuuint64_t)ld * sizeof(double)};
  const cuuint32_t box[2] = {box0, box1};
  const cuuint32_t estr[2] = {1, 1};
  return fn(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<double*>(X), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace ws

// C = alpha * sum_seg op(A_seg) op(B_seg) + beta * Cin; tile 128x128 (wide N), 128x64 (N <= 64) or 128x32 (N <= 32,
// the b = 32 band: a 128x64 tile would multiply half zeros; warps 8x1 of 16x32).  Same
// semantics as gemm().
cudaError_t gemm_ws(GemmArgs g, int opB, cudaStream_t st) { return gemm_ws_op(g, OP_N, opB, st); }

cudaError_t gemm_ws_op(GemmArgs g, int opA, int opB, cudaStream_t st) {
  if (g.M <= 0 || g.N <= 0) return cudaSuccess;
  ws::WsArgs a{};
  a.M = g.M; a.N = g.N; a.opa = opA; a.opb = opB; a.nseg = g.nseg;
  bool v16 = true;
  for (int i = 0; i < 2; ++i) {
    a.A[i] = g.A[i]; a.B[i] = g.B[i]; a.lda[i] = g.lda[i]; a.ldb[i] = g.ldb[i]; a.K[i] = g.K[i];
    if (i < g.nseg) v16 = v16 && ws::al16(g.A[i]) && ws::al16(g.B[i]) && !(g.lda[i] & 1) && !(g.ldb[i] & 1);
  }
  a.vec16 = v16;
  a.symm = 0;
  a.alpha = g.alpha; a.beta = g.beta; a.Cin = g.Cin; a.ldcin = g.ldcin; a.C = g.C; a.ldc = g.ldc;
  a.lower = g.lower; a.diag_off = g.diag_off; a.tri = g.tri;
  a.splits = g.splits < 1 ? 1 : g.splits;
  a.mg_g = g.mg_g; a.mg_q = g.mg_q; a.mg_cb = g.mg_cb; a.mg_lofs = g.mg_lofs; a.mg_gofs = g.mg_gofs;
  if (a.mg_g > 1 && (a.tri || (a.lower && a.splits > 1) || a.mg_cb < 1)) return cudaErrorInvalidValue;
  a.part = g.part; a.part_ld = g.part_ld; a.part_stride = g.part_stride;
  a.A2 = (g.A2m && g.msplit < g.M) ? g.A2m : nullptr;
  a.msplit = g.msplit;
  if (a.A2) {   // stacked operands: A op T, one segment, no multi-GPU map
    if (opA != OP_T || g.nseg != 1 || a.mg_g > 1) return cudaErrorInvalidValue;
    a.vec16 = a.vec16 && ws::al16(g.A2m);
  }
  if (a.mg_g > 1) {   // multi-GPU column map (only the lower-masked syr2k of mg.cu uses it)
    if (opB != OP_T || opA != OP_N) return cudaErrorInvalidValue;
    return g.N <= 64 ? ws::launch<128, 64, 4, 2, OP_T, true>(a, st) : ws::launch<128, 128, 4, 2, OP_T, true>(a, st);
  }
  if (g.N <= 32 && ws::narrow_tiles()) {
    return opB == OP_T ? ws::launch<128, 32, 8, 1, OP_T>(a, st) : ws::launch<128, 32, 8, 1, OP_N>(a, st);
  }
  if (g.N <= 64) {
    return opB == OP_T ? ws::launch<128, 64, 4, 2, OP_T>(a, st) : ws::launch<128, 64, 4, 2, OP_N>(a, st);
  }
  // bulk-copy (TMA) staging for A op N / B op T on 128 x 128 tiles (the syr2k and the other NT contractions);
  // (measured: syr2k 70.7 -> 65.9 ms at n = 32768, k = 1024); env TRID_WS_TMA=0 restores the cp.async producer
  // TRID_WS_TMA: 0 cp.async producer, 1 per-row bulk copies, 2 (default) tensor maps (cp.async.bulk.tensor)
  const char* tenv = getenv("TRID_WS_TMA");   // read per call (tests toggle it)
  const int tmode = tenv ? atoi(tenv) : 2;
  a.tma = (tmode != 0) && opA == OP_N && opB == OP_T && v16 && !(g.M & 1) && !(g.N & 1);
  if (a.tma && tmode == 2) {
    bool ok = true;
    for (int i = 0; i < g.nseg && ok; ++i)
      ok = ws::encode_rows_map(&a.tmA[i], g.A[i], g.M, g.K[i], g.lda[i]) &&
           ws::encode_rows_map(&a.tmB[i], g.B[i], g.N, g.K[i], g.ldb[i]);
    a.tma = ok ? 2 : 1;   // no driver entry point: the per-row bulk copies (same staged values)
  }
  return opB == OP_T ? ws::launch<128, 128, 4, 2, OP_T>(a, st) : ws::launch<128, 128, 4, 2, OP_N>(a, st);
}

// Split-K count of a GEMM on the persistent engine from a makespan model (as for the SYMM below): units
// u = z * tiles + t walked by 148 CTAs with stride 148, unit z covering K-tiles [z per, (z + 1) per) of the
// ceil(K / 16) K-tiles; unit cost = K-tiles x 1.19 us (128 x 64 tile; 2.38 us for 128 x 128) + 2 us; + the split-K
// reduction (read s + 1, write 1 partial at 5 TB/s, + 3 us launch).  Pure function of the shape and the caps
// (deterministic sums; the workspace sizing uses it), memoized.  env TRID_SPLIT_MODEL=0 restores the former
// rule (~3 waves of units, >= 256 of K per split).
static int gemm_splits_model(int64_t M, int64_t N, int64_t K, int cap, int64_t part_cap) {
  const int64_t bn = (N <= 32 && ws::narrow_tiles()) ? 32 : (N <= 64 ? 64 : 128);
  const int64_t tiles = ((M + 127) / 128) * ((N + bn - 1) / bn);
  const double ts = bn == 32 ? 0.60 : (bn == 64 ? 1.19 : 2.38);
  const int64_t kt = (K + 15) / 16;
  double best = 1e300;
  int bs = 1;
  double load[kNumSMsB200];
  for (int64_t sp = 1; sp <= cap && sp <= kt; ++sp) {
    if (sp > 1 && sp * M * N > part_cap) break;
    const int64_t per = (kt + sp - 1) / sp;
    for (int c = 0; c < kNumSMsB200; ++c) load[c] = 0.0;
    for (int64_t u = 0; u < tiles * sp; ++u) {
      const int64_t z = u / tiles;
      int64_t k = kt - z * per;
      k = k < per ? k : per;
      load[u % kNumSMsB200] += (k > 0 ? (double)k : 0.0) * ts + 2.0;
    }
    double mk = 0.0;
    for (int c = 0; c < kNumSMsB200; ++c) mk = load[c] > mk ? load[c] : mk;
    if (sp > 1) mk += (double)(sp + 2) * (double)M * (double)N * 8.0 / 5.0e6 + 3.0;
    if (mk < best * 0.999) {
      best = mk;
      bs = (int)sp;
    }
  }
  return bs;
}
static bool split_model_on() {
  static const bool on = !(getenv("TRID_SPLIT_MODEL") && getenv("TRID_SPLIT_MODEL")[0] == '0');
  return on;
}
static int gemm_splits(int64_t M, int64_t N, int64_t K, int cap, int64_t part_cap) {
  static std::mutex mu;
  static std::unordered_map<std::string, int> memo;
  char key[96];
  snprintf(key, sizeof key, "%lld/%lld/%lld/%d/%lld", (long long)M, (long long)N, (long long)K, cap,
           (long long)part_cap);
  {
    std::lock_guard<std::mutex> lk(mu);
    auto it = memo.find(key);
    if (it != memo.end()) return it->second;
  }
  const int sp = gemm_splits_model(M, N, K, cap, part_cap);
  std::lock_guard<std::mutex> lk(mu);
  memo[key] = sp;
  return sp;
}

// C (M x N) = alpha op(A) op(B) + beta Cin with a split-K count (deterministic sums) from the makespan model,
// within part_elems partials and <= 64 splits.
cudaError_t gemm_ws_mm(int opA, int opB, int64_t M, int64_t N, int64_t K, double alpha, const double* A, int64_t lda,
                       const double* B, int64_t ldb, double beta, double* C, int64_t ldc, double* part,
                       int64_t part_elems, cudaStream_t st, const double* A2, int64_t msplit) {
  if (M <= 0 || N <= 0) return cudaSuccess;
  int64_t s;
  if (split_model_on()) {
    s = gemm_splits(M, N, K, 64, part_elems);
  } else {
    const int64_t tiles = ((M + 127) / 128) * ((N + (N <= 64 ? 63 : 127)) / (N <= 64 ? 64 : 128));
    s = (3 * kNumSMsB200 + tiles - 1) / tiles;
    const int64_t maxk = K / 256;
    if (s > maxk) s = maxk;
    if (s > 64) s = 64;
    if (s > 1 && s * M * N > part_elems) s = part_elems / (M * N);
    if (s < 1) s = 1;
  }
  GemmArgs g;
  g.M = M; g.N = N; g.K[0] = K; g.A[0] = A; g.lda[0] = lda; g.B[0] = B; g.ldb[0] = ldb;
  g.alpha = alpha; g.beta = beta; g.Cin = C; g.ldcin = ldc; g.C = C; g.ldc = ldc;
  if (A2) {
    g.A2m = A2;
    g.msplit = msplit;
  }
  g.splits = (int)s;
  g.part = part; g.part_ld = M; g.part_stride = M * N;
  return gemm_ws_op(g, opA, opB, st);
}

// Split-K for the skinny engine GEMMs (M = trailing rows, N = b, K = 2 x block columns): the makespan model with
// <= 16 splits (the former rule: ~3 waves of units, >= 256 of K per split).  Partials: splits * M * N doubles.
int ws_skinny_splits(int64_t M, int64_t N, int64_t K) {
  if (split_model_on()) return gemm_splits(M, N, K, 16, INT64_MAX);
  const int64_t tiles = ((M + 127) / 128) * ((N + (N <= 64 ? 63 : 127)) / (N <= 64 ? 64 : 128));
  int64_t sp = (3 * kNumSMsB200 + tiles - 1) / tiles;   // fixed (not the device's): sizes workspaces, fixes sums
  const int64_t maxs = K / 256;
  if (sp > maxs) sp = maxs;
  if (sp > 16) sp = 16;
  return sp < 1 ? 1 : (int)sp;
}

// Strip splits of the SYMM, chosen by a makespan model of the persistent grid (148 CTAs walking units
// u = z * tiles + t with stride 148, unit z covering the K chunk [z cz, (z + 1) cz) of the strip, cz a multiple of
// 16): unit cost = (its K + the diagonal-block overlap) / 16 stages x 1.19 us (one 128 x 64 x 16 DMMA stage at
// ~0.88 of 37 TF/s over 148 SMs) + 2 us (unit epilogue / refill); + the split-K reduction over HBM (read s + 1,
// write 1 partial, 5 TB/s).  Pure function of (m, w) and fixed constants (the workspace sizing and the
// deterministic sums use it), memoized.  The former rule (>= 8 waves, K >= 512 per split) left up to 9% of the
// last wave idle at some m (e.g. m = 28608: 1344 units = 9.08 waves).  env TRID_SYMM_WAVES=W restores it.
static int64_t symm_splits_model(int64_t m, int64_t w, int64_t nc) {
  const int64_t tm = (m + 127) / 128, rows = tm * ((w + 63) / 64);
  int64_t maxs = (m + 255) / 256 < 32 ? (m + 255) / 256 : 32;
  const int64_t maxw = (24 * kNumSMsB200 + rows - 1) / rows;   // <= ~24 waves (bounds the search)
  const double ts = (w <= 32 && ws::narrow_tiles()) ? 0.60 : 1.19;   // us per 128 x BN x 16 stage
  if (maxs > maxw) maxs = maxw;
  double best = 1e300;
  int64_t bs = 1;
  double load[kNumSMsB200];
  for (int64_t sp = 1; sp <= maxs; ++sp) {
    const int64_t kt = m + 2 * nc;   // strip + correction segments
    const int64_t chunk = (kt + sp - 1) / sp, cz = (chunk + 15) / 16 * 16;
    for (int c = 0; c < kNumSMsB200; ++c) load[c] = 0.0;
    const int64_t units = rows * sp;
    for (int64_t u = 0; u < units; ++u) {
      const int64_t z = u / rows, t = (u % rows) % tm;
      const int64_t k0 = z * cz, k1 = k0 + cz < kt ? k0 + cz : kt;
      double kk = k1 > k0 ? (double)(k1 - k0) : 0.0;
      const int64_t d0 = t * 128, d1 = d0 + 128 < m ? d0 + 128 : m;   // diagonal block, counted by both strips
      const int64_t o0 = k0 > d0 ? k0 : d0, o1 = k1 < d1 ? k1 : d1;
      if (o1 > o0) kk += (double)(o1 - o0);
      load[u % kNumSMsB200] += kk / 16.0 * ts + 2.0;
    }
    double mk = 0.0;
    for (int c = 0; c < kNumSMsB200; ++c) mk = load[c] > mk ? load[c] : mk;
    if (sp > 1) mk += (double)(sp + 2) * (double)m * (double)w * 8.0 / 5.0e6;
    if (mk < best * 0.999) {
      best = mk;
      bs = sp;
    }
  }
  return bs;
}

int64_t symm_ws_splits(int64_t m, int64_t w, int64_t nc) {
  static const char* wv = getenv("TRID_SYMM_WAVES");
  if (wv) {
    const int64_t rows = (m + 127) / 128 * ((w + 63) / 64);
    int64_t sp = (atoll(wv) * kNumSMsB200 + rows - 1) / rows;
    const int64_t maxs = (m + 511) / 512;
    if (sp > maxs) sp = maxs;
    if (sp > 32) sp = 32;
    return sp < 1 ? 1 : sp;
  }
  if (m <= 0 || w <= 0) return 1;
  static std::mutex mu;
  static std::unordered_map<int64_t, int64_t> memo;
  const int64_t key = (m * 4096 + w) * 8192 + nc;
  {
    std::lock_guard<std::mutex> lk(mu);
    auto it = memo.find(key);
    if (it != memo.end()) return it->second;
  }
  const int64_t sp = symm_splits_model(m, w, nc);
  std::lock_guard<std::mutex> lk(mu);
  memo[key] = sp;
  return sp;
}
int64_t symm_ws_part_elems(int64_t m, int64_t w, int64_t nc) {
  const int64_t sp = symm_ws_splits(m, w, nc);
  return sp > 1 ? sp * m * w : 0;
}

// X = Asym W (+ CA0 CB0 + CA1 CB1 when nc > 0) on the warp-specialized engine (row strip + transposed column strip
// per row block, then the two correction segments, all in one K axis chunked across the splits).
cudaError_t symm_ws(int64_t m, int64_t w, const double* A, int64_t lda, const double* W, int64_t ldw, double* X,
                    int64_t ldx, double* part, int64_t part_elems, cudaStream_t st, int64_t nc, const double* CA0,
                    const double* CB0, const double* CA1, const double* CB1, int64_t ldca, int64_t ldcb) {
  if (m <= 0 || w <= 0) return cudaSuccess;
  ws::WsArgs a{};
  a.M = m; a.N = w; a.opb = OP_N; a.nseg = 1; a.symm = 1;
  a.A[0] = A; a.B[0] = W; a.lda[0] = lda; a.ldb[0] = ldw; a.K[0] = m;
  a.vec16 = ws::al16(A) && ws::al16(W) && !(lda & 1) && !(ldw & 1);
  if (nc > 0) {
    a.ncorr = nc; a.CA[0] = CA0; a.CB[0] = CB0; a.CA[1] = CA1; a.CB[1] = CB1; a.ldca = ldca; a.ldcb = ldcb;
    a.vec16 = a.vec16 && ws::al16(CA0) && ws::al16(CA1) && ws::al16(CB0) && ws::al16(CB1) && !(ldca & 1) &&
              !(ldcb & 1);
  }
  a.alpha = 1.0; a.beta = 0.0; a.C = X; a.ldc = ldx;
  int64_t sp = symm_ws_splits(m, w, nc > 0 ? nc : 0);
  if (sp * m * w > part_elems) sp = part_elems / (m * w);
  if (sp < 1) sp = 1;
  a.splits = (int)sp;
  a.part = part; a.part_ld = m; a.part_stride = m * w;
  // tensor copies for the m-inner A tiles (TRID_WS_TMA: default 2 on; 0 / 1 keep cp.async for every tile)
  const char* tenv = getenv("TRID_WS_TMA");
  if ((!tenv || atoi(tenv) == 2) && a.vec16) {
    bool ok = ws::encode_map(&a.tmSA, A, m, m, lda, 128 + 4, ws::BK);
    for (int i = 0; i < 2 && ok && nc > 0; ++i) ok = ws::encode_map(&a.tmSC[i], a.CA[i], m, nc, ldca, 128 + 4, ws::BK);
    a.symm_tma = ok ? 1 : 0;
  }
  if (w <= 32 && ws::narrow_tiles()) return ws::launch<128, 32, 8, 1, OP_N>(a, st);
  return ws::launch<128, 64, 4, 2, OP_N>(a, st);
}

// ---- multi-GPU SYMM partials (block-cyclic local columns) ------------------------
static int64_t mg_splits(int64_t tiles, int64_t K) {
  int64_t sp = (8 * kNumSMsB200 + tiles - 1) / tiles;
  const int64_t maxs = (K + 511) / 512;
  if (sp > maxs) sp = maxs;
  if (sp > 32) sp = 32;
  return sp < 1 ? 1 : sp;
}
int64_t symm_mg_part_elems(int64_t m, int64_t w, int64_t nqt) {
  const int64_t tn = (w + 63) / 64;
  const int64_t s2 = mg_splits((m + 127) / 128 * tn, nqt), s3 = mg_splits((nqt + 127) / 128 * tn, m);
  const int64_t e2 = s2 > 1 ? s2 * m * w : 0, e3 = s3 > 1 ? s3 * nqt * w : 0;
  return e2 > e3 ? e2 : e3;
}
static cudaError_t symm_mg(int mode, int64_t M, int64_t w, int64_t K, const double* A, int64_t lda, const double* B,
                           int64_t ldb, double* C, int64_t ldc, const MgMap& mp, double* part, int64_t part_elems,
                           cudaStream_t st) {
  if (M <= 0 || w <= 0) return cudaSuccess;
  ws::WsArgs a{};
  a.M = M; a.N = w; a.opb = OP_N; a.nseg = 1; a.symm = mode;
  a.A[0] = A; a.B[0] = B; a.lda[0] = lda; a.ldb[0] = ldb; a.K[0] = K;
  a.vec16 = ws::al16(A) && ws::al16(B) && !(lda & 1) && !(ldb & 1);
  a.alpha = 1.0; a.beta = 0.0; a.C = C; a.ldc = ldc;
  a.mg_g = mp.g; a.mg_q = mp.q; a.mg_cb = mp.cb; a.mg_lofs = mp.lofs; a.mg_gofs = mp.gofs;
  int64_t sp = mg_splits((M + 127) / 128 * ((w + 63) / 64), K);
  if (sp * M * w > part_elems) sp = part_elems / (M * w);
  if (sp < 1) sp = 1;
  a.splits = (int)sp;
  a.part = part; a.part_ld = M; a.part_stride = M * w;
  return w <= 64 ? ws::launch<128, 64, 4, 2, OP_N, true>(a, st) : ws::launch<128, 128, 4, 2, OP_N, true>(a, st);
}
// X (m x w) = sum over local columns x with cmap(x) <= row of A_loc(row, x) W_loc(x, :)
cudaError_t symm_mg_rows(int64_t m, int64_t w, int64_t nqt, const double* Aloc, int64_t lda, const double* Wloc,
                         int64_t ldwl, double* X, int64_t ldx, const MgMap& mp, double* part, int64_t part_elems,
                         cudaStream_t st) {
  return symm_mg(2, m, w, nqt, Aloc, lda, Wloc, ldwl, X, ldx, mp, part, part_elems, st);
}
// Xl (nqt x w) = sum over global rows k > cmap(x) of A_loc(k, x) W(k, :)
cudaError_t symm_mg_cols(int64_t m, int64_t w, int64_t nqt, const double* Aloc, int64_t lda, const double* W,
                         int64_t ldw, double* Xl, int64_t ldxl, const MgMap& mp, double* part, int64_t part_elems,
                         cudaStream_t st) {
  return symm_mg(3, nqt, w, m, Aloc, lda, W, ldw, Xl, ldxl, mp, part, part_elems, st);
}

}  // namespace trid
