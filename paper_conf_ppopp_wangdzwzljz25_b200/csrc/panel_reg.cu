// panel_reg.cu — register-resident, cluster-reduced panel QR for DBBR (Alg. 1 line 5)
// with the dlarft T factor and the explicit Y = V.  Fast path for w in {16, 32, 64}.
//
// Layout: G CTAs (a multiple of 8, launched as clusters of 8) own contiguous row blocks of the m x w
// panel; inside a CTA, warp wi owns columns [wi*CPW, (wi+1)*CPW) and lane l owns rows l, l+32, ...
// so the whole panel lives in registers (RL x CPW doubles per thread).  Column t costs:
//   1. every warp forms its slots of the Gram row  sum_{r>t} x_r P(r, j)  (x = column t below row t,
//      broadcast through shared memory) with one transposed butterfly, plus the row-t values;
//   2. cluster barrier; CTA rank c reduces slots c, c+8, ... over the 8 CTAs through DSMEM (fixed
//      order) and writes the cluster partial to global memory;
//   3. ONE grid barrier (release/acquire counter);
//   4. every CTA sums the NC cluster partials in a fixed order -> identical beta/tau/w in all CTAs;
//   5. register update P(r, j) -= tau w_j v_r, T column in CTA 0's shared memory.
// Default since round 2: panel_reg2_kernel, the same scheme with two reflectors per grid barrier (look-ahead Gram
// sums of the column pair, falling back to one reflector where the look-ahead norm would cancel); 155 -> 141 ms of
// panel time per n = 32768 step.  TRID_PANEL_PAIR=0 selects panel_reg_kernel.
#include <cooperative_groups.h>

#include "common.cuh"
#include "panel.cuh"
#include "prof.cuh"

#include <stdlib.h>

namespace trid {

namespace cg = cooperative_groups;

constexpr int PR_NT = 256;   // 8 warps
constexpr int PR_CL = 4;     // cluster size (33 co-resident 4-CTA clusters at 1 CTA/SM on B200)
constexpr int PR_MAXNC = 40; // max clusters
constexpr int PR_RL = 8;     // rows per lane (rows per CTA <= 256)
constexpr int PR_NBAR = 8;   // grid-barrier counters (128 B apart)

struct PanelRegArgs {
  int64_t m;
  int w, kk;
  double* P;
  int64_t ldp;
  double* tau;
  double* T;
  int64_t ldt;
  double* Y;
  int64_t ldy;
  double* gpart;     // 2 x NC x 2w cluster partials
  unsigned* bar;     // grid barrier counter (zero at launch)
  int rows;          // rows per CTA
  long long* trace;  // debug (TRID_PANEL_TRACE=m): %globaltimer per column phase, CTAs 0 and G-1
};
__device__ __forceinline__ long long pr_gtimer() {
  long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#define PR_TRACE(k)                                                                        \
  do {                                                                                     \
    if (a.trace && tid == 0 && (g == 0 || g == G - 1) && t < 256)                          \
      a.trace[((g == 0 ? 0 : 1) * 256 + t) * 8 + (k)] = pr_gtimer();                       \
  } while (0)

// T(0:c, c) = -tau_c T(0:c, 0:c) (V(:, 0:c)^T v_c), T(c, c) = tau_c (dlarft forward columnwise);
// Dm[c*W + p] = v_c^T v_p.  Reads T columns < c (complete: a __syncthreads separates the calls).
__device__ __forceinline__ void t_column(double* Ts, const double* Dm, const double* taus, int c, int W, int tid) {
  for (int q2 = tid; q2 < W; q2 += PR_NT) {
    double v = 0.0;
    if (q2 < c) {
      double sacc = 0.0;
      for (int p = q2; p < c; ++p) sacc += Ts[q2 + p * W] * Dm[c * W + p];
      v = -taus[c] * sacc;
    } else if (q2 == c) {
      v = taus[c];
    }
    Ts[q2 + c * W] = v;
  }
}

template <int CPW>
__global__ void __launch_bounds__(PR_NT, 1) panel_reg_kernel(const __grid_constant__ PanelRegArgs a) {
  constexpr int W = 8 * CPW;
  constexpr int RS = 2 * W;
  extern __shared__ __align__(16) double sm[];
  double* xsb = sm;                   // 2 x rows of this CTA: column t (broadcast), by column parity
  double* mypart = xsb + 2 * 32 * PR_RL;   // 2 x RS   (double-buffered per column parity)
  double* tot = mypart + 2 * RS;      // RS
  double* Ts = tot + RS;              // W x W    (CTA 0)
  double* Dm = Ts + W * W;            // W x W    (CTA 0): v_t^T v_p, p < t, for the T factor
  double* taus = Dm + W * W;          // W        (CTA 0)
  double* tot2 = taus + W;            // RS       second half of the partial sums
  cg::cluster_group cl = cg::this_cluster();
  const int g = blockIdx.x, G = gridDim.x, NC = G / PR_CL;
  const int crank = (int)cl.block_rank(), cid = g / PR_CL;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int64_t rlo = (int64_t)g * a.rows;
  const int nr = (int)((rlo + a.rows <= a.m) ? a.rows : (a.m > rlo ? a.m - rlo : 0));
  const int j0 = warp * CPW;

  double P[PR_RL][CPW];
#pragma unroll
  for (int q = 0; q < PR_RL; ++q) {
    const int i = lane + 32 * q;
#pragma unroll
    for (int c = 0; c < CPW; ++c)
      P[q][c] = (i < nr && j0 + c < a.w) ? a.P[(rlo + i) + (int64_t)(j0 + c) * a.ldp] : 0.0;
  }
  // column 0 -> xs (buffer 0)
  if (warp == 0) {
#pragma unroll
    for (int q = 0; q < PR_RL; ++q) xsb[lane + 32 * q] = P[q][0];
  }
  unsigned epoch = 0;
  __syncthreads();

  for (int t = 0; t < a.kk; ++t) {
    const int par = t & 1;
    const double* xs = xsb + par * 32 * PR_RL;
    PR_TRACE(0);
    // ---- 1. Gram slots of this warp's columns over rows > t, and row-t values
    double acc[CPW];
#pragma unroll
    for (int c = 0; c < CPW; ++c) acc[c] = 0.0;
    int qt = -1;   // this lane's q holding row t, if any
#pragma unroll
    for (int q = 0; q < PR_RL; ++q) {
      const int64_t r = rlo + lane + 32 * q;
      const double x = (r > t && lane + 32 * q < nr) ? xs[lane + 32 * q] : 0.0;
      if (r == t && lane + 32 * q < nr) qt = q;
#pragma unroll
      for (int c = 0; c < CPW; ++c) acc[c] = fma(x, P[q][c], acc[c]);
    }
    // transposed butterfly: CPW values over 32 lanes
    int qb = 0;
#pragma unroll
    for (int o = 16, K = CPW; K > 1; o >>= 1, K >>= 1) {
      const bool up = (lane & o) != 0;
#pragma unroll
      for (int i = 0; i < K / 2; ++i) {
        const double send = up ? acc[i] : acc[i + K / 2];
        const double keep = up ? acc[i + K / 2] : acc[i];
        acc[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
      }
      if (up) qb += K / 2;
    }
    constexpr int LV = CPW >= 8 ? 3 : (CPW == 4 ? 2 : (CPW == 2 ? 1 : 0));
    double f = acc[0];
#pragma unroll
    for (int o = 16 >> LV; o >= 1; o >>= 1) f += __shfl_xor_sync(0xffffffffu, f, o);
    double* mp = mypart + par * RS;
    if ((lane & ((32 >> LV) - 1)) == 0) mp[j0 + qb] = f;
    // row-t values of this warp's columns (owner lane) or zero
    {
      const unsigned own = __ballot_sync(0xffffffffu, qt >= 0);
      if (own) {
        const int src = __ffs(own) - 1;
#pragma unroll
        for (int c = 0; c < CPW; ++c) {
          double vv = 0.0;
#pragma unroll
          for (int q = 0; q < PR_RL; ++q)
            if (q == qt) vv = P[q][c];
          vv = __shfl_sync(0xffffffffu, vv, src);
          if (lane == 0) mp[W + j0 + c] = vv;
        }
      } else if (lane < CPW) {
        mp[W + j0 + lane] = 0.0;
      }
    }
    // ---- 2. cluster reduction through DSMEM (fixed order over the 8 CTAs)
    PR_TRACE(1);
    cl.sync();
    PR_TRACE(2);
    {
      // thread -> (slot s = crank + 8*k, member c): 8 lanes per slot
      const int k = tid / PR_CL, c = tid % PR_CL;
      const int s = crank + PR_CL * k;
      double v = 0.0;
      if (s < RS) {
        const double* rp = cl.map_shared_rank(mypart + par * RS, c);
        v = rp[s];
      }
#pragma unroll
      for (int o = 1; o < PR_CL; o <<= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
      if (c == 0 && s < RS) __stcg(a.gpart + ((size_t)par * NC + cid) * RS + s, v);
    }
    // ---- 3. one grid barrier
    __syncthreads();
    PR_TRACE(3);
    epoch += 1;
    // grid barrier on PR_NBAR counters (128 B apart) so the G arrivals do not serialise on one L2 line
    if (tid == 0) asm volatile("red.release.gpu.global.add.u32 [%0], 1;\n" ::"l"(a.bar + 32 * (g % PR_NBAR)) : "memory");
    // CTA 0 builds the T column of the previous reflector while the other CTAs arrive (off the critical path)
    if (g == 0 && t > 0) t_column(Ts, Dm, taus, t - 1, W, tid);
    if (tid < PR_NBAR) {
      const unsigned target = epoch * (unsigned)((G - tid + PR_NBAR - 1) / PR_NBAR);
      const unsigned* cnt = a.bar + 32 * tid;
      while (ld_relaxed_u32(cnt) < target) {
      }
      (void)ld_acquire_u32(cnt);
    }
    __syncthreads();
    PR_TRACE(4);
    // ---- 4. totals over the NC cluster partials, fixed order
    {
      // 2 threads per slot: cluster partials [0, NC/2) and [NC/2, NC), each summed in order, then added
      const int s = tid % RS, hh = tid / RS, q0 = hh ? NC / 2 : 0, q1 = hh ? NC : NC / 2;
      constexpr int HALF = (PR_MAXNC + 1) / 2;
      if (tid < 2 * RS) {
        double vals[HALF];
#pragma unroll
        for (int q = 0; q < HALF; ++q)
          vals[q] = q0 + q < q1 ? __ldcg(a.gpart + ((size_t)par * NC + q0 + q) * RS + s) : 0.0;
        double v = vals[0];
#pragma unroll
        for (int q = 1; q < HALF; ++q)
          if (q0 + q < q1) v += vals[q];
        (hh ? tot2 : tot)[s] = v;
      }
    }
    __syncthreads();
    for (int s = tid; s < RS; s += PR_NT) tot[s] += tot2[s];
    __syncthreads();
    PR_TRACE(5);
    // ---- 5. reflector, update, T column
    const House h = make_house(tot[W + t], tot[t]);
    double tw[CPW];   // -tau * w_j for this warp's columns (w_j = v^T P(:, j))
#pragma unroll
    for (int c = 0; c < CPW; ++c) tw[c] = -h.tau * fma(h.scale, tot[j0 + c], tot[W + j0 + c]);
    if (j0 > t) {
      // every column of this warp lies right of t (the common case): a predicate-free rank-1 update of the rows >= t
#pragma unroll
      for (int q = 0; q < PR_RL; ++q) {
        const int i = lane + 32 * q;
        const int64_t r = rlo + i;
        if (i < nr && r >= t) {
          const double vr = r > t ? h.scale * xs[i] : 1.0;
#pragma unroll
          for (int c = 0; c < CPW; ++c) P[q][c] = fma(tw[c], vr, P[q][c]);
        }
      }
    } else if (j0 + CPW > t) {
      // the warp holding column t: v (or beta) into column t, the update right of it, nothing left of it
#pragma unroll
      for (int q = 0; q < PR_RL; ++q) {
        const int i = lane + 32 * q;
        const int64_t r = rlo + i;
        if (i >= nr || r < t) continue;
        const double vr = r > t ? h.scale * xs[i] : 1.0;
#pragma unroll
        for (int c = 0; c < CPW; ++c) {
          const int j = j0 + c;
          if (j > t) {
            P[q][c] = fma(tw[c], vr, P[q][c]);
          } else if (j == t) {
            P[q][c] = r > t ? vr : h.beta;
          }
        }
      }
    }
    if (g == 0) {
      // v_t^T v_p = P(t, p) + scale * sum_{r>t} x_r P(r, p) for p < t (the Gram row), saved for the T column
      for (int p = tid; p < t; p += PR_NT) Dm[t * W + p] = tot[W + p] + h.scale * tot[p];
      if (tid == 0) {
        taus[t] = h.tau;
        a.tau[t] = h.tau;
      }
    }
    PR_TRACE(6);
    // next column -> the other xs buffer (its previous readers finished before this column's grid barrier)
    if (t + 1 < a.kk && warp == (t + 1) / CPW) {
      double* xn = xsb + (par ^ 1) * 32 * PR_RL;
      const int cn = (t + 1) % CPW;
#pragma unroll
      for (int q = 0; q < PR_RL; ++q) {
        double v = 0.0;
#pragma unroll
        for (int c = 0; c < CPW; ++c)
          if (c == cn) v = P[q][c];
        xn[lane + 32 * q] = v;
      }
    }
    __syncthreads();   // xs of column t+1 visible; all reads of tot / xs of column t done
  }
  if (g == 0 && a.kk > 0) {
    t_column(Ts, Dm, taus, a.kk - 1, W, tid);
    __syncthreads();
  }
  // ---- write back R/V, explicit Y, T
#pragma unroll
  for (int q = 0; q < PR_RL; ++q) {
    const int i = lane + 32 * q;
    if (i >= nr) continue;
    const int64_t r = rlo + i;
#pragma unroll
    for (int c = 0; c < CPW; ++c) {
      const int j = j0 + c;
      if (j < a.w) a.P[r + (int64_t)j * a.ldp] = P[q][c];
      if (j < a.kk) a.Y[r + (int64_t)j * a.ldy] = r > j ? P[q][c] : (r == j ? 1.0 : 0.0);
    }
  }
  if (g == 0) {
    for (int idx = tid; idx < W * W; idx += PR_NT) {
      const int q2 = idx % W, c = idx / W;
      a.T[q2 + (int64_t)c * a.ldt] = (c < a.kk) ? Ts[q2 + c * W] : 0.0;
    }
  }
  cl.sync();   // no CTA leaves while a cluster peer may still read its shared memory
}

// Transposed butterfly: NVv per-lane partial sums -> lane holds the warp total of value index qb in f (lanes with
// (lane & (32 / NVv - 1)) == 0 own a distinct index; NVv a power of two <= 32).
template <int NVv>
__device__ __forceinline__ double warp_butterfly(double (&acc)[NVv], int lane, int& qb) {
  qb = 0;
#pragma unroll
  for (int o = 16, K = NVv; K > 1; o >>= 1, K >>= 1) {
    const bool up = (lane & o) != 0;
#pragma unroll
    for (int i = 0; i < K / 2; ++i) {
      const double send = up ? acc[i] : acc[i + K / 2];
      const double keep = up ? acc[i + K / 2] : acc[i];
      acc[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
    }
    if (up) qb += K / 2;
  }
  constexpr int LV = NVv >= 32 ? 5 : (NVv == 16 ? 4 : (NVv == 8 ? 3 : (NVv == 4 ? 2 : (NVv == 2 ? 1 : 0))));
  double f = acc[0];
#pragma unroll
  for (int o = 16 >> LV; o >= 1; o >>= 1) f += __shfl_xor_sync(0xffffffffu, f, o);
  return f;
}

// ---- two reflectors per grid barrier (look-ahead by one column) ----------------------------------------------
// One reduction serves the column pair (p, q = p + 1): besides the Gram row of column p (G1[j] = sum_{r>p} a_p a_j)
// and row p (Rp[j] = a_j(p)) it carries the Gram row of column q over rows > q (G2[j] = sum_{r>q} a_q a_j) and row q
// (Rq[j]); sums of a_p a_j over rows > q are G1[j] - Rq[p] Rq[j].  Reflector p is formed as in panel_reg_kernel: w_j = Rp[j] + s G1[j], a'_j = a_j - tau v_p w_j, i.e.
// a'_j(r) = a_j(r) - c_j a_p(r) below row p with c_j = tau s w_j.  Column q after it, and every product reflector q
// needs, follow from the same sums (exact algebra, sums over r > q):
//   sigma' = sum a'_q^2          = G2[q] - 2 c_q G2[p] + c_q^2 (G1[p] - Rq[p]^2),   alpha' = Rq[q] - c_q Rq[p],
//   sum a'_q a'_j                = G2[j] - c_j G2[p] - c_q (G1[j] - Rq[p] Rq[j]) + c_q c_j (G1[p] - Rq[p]^2),
//   w'_j = a'_j(q) + s' sum a'_q a'_j,  a'_j(q) = Rq[j] - c_j Rq[p],
// and v_q^T v_s (the T factor) likewise.  sigma' is a difference: when it falls below 1/16 of the magnitude of its
// terms, G1[p] and Rq[p]^2 counted separately (column q nearly parallel to column p, or a_p(q) dominating column p
// below row p: cancellation could cost more than 4 bits of the norm, and with it the orthogonality of H_q) the step
// takes reflector p alone and the next reduction restarts at q.  Every CTA sums
// the same partials in the same order, so all CTAs take the same branch.  Halves the grid barriers of the panel.
template <int CPW>
__global__ void __launch_bounds__(PR_NT, 1) panel_reg2_kernel(const __grid_constant__ PanelRegArgs a) {
  constexpr int W = 8 * CPW;
  constexpr int RS = 4 * W;   // [G1 | G2 | Rp | Rq]
  constexpr int NV = 2 * CPW;
  static_assert(RS % (8 * PR_CL) == 0, "the DSMEM reduction loop must be warp-uniform");
  constexpr int XS = 32 * PR_RL;
  extern __shared__ __align__(16) double sm[];
  double* xsb = sm;                     // [parity][column p, column q][rows of this CTA]
  double* mypart = xsb + 4 * XS;        // 2 x RS (by parity)
  double* tot = mypart + 2 * RS;        // RS
  double* Ts = tot + RS;                // W x W    (CTA 0)
  double* Dm = Ts + W * W;              // W x W    (CTA 0): v_t^T v_p, p < t
  double* taus = Dm + W * W;            // W        (CTA 0)
  cg::cluster_group cl = cg::this_cluster();
  const int g = blockIdx.x, G = gridDim.x, NC = G / PR_CL;
  const int crank = (int)cl.block_rank(), cid = g / PR_CL;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int64_t rlo = (int64_t)g * a.rows;
  const int nr = (int)((rlo + a.rows <= a.m) ? a.rows : (a.m > rlo ? a.m - rlo : 0));
  const int j0 = warp * CPW;

  double P[PR_RL][CPW];
#pragma unroll
  for (int q = 0; q < PR_RL; ++q) {
    const int i = lane + 32 * q;
#pragma unroll
    for (int c = 0; c < CPW; ++c)
      P[q][c] = (i < nr && j0 + c < a.w) ? a.P[(rlo + i) + (int64_t)(j0 + c) * a.ldp] : 0.0;
  }
  // columns 0 and 1 -> parity-0 buffers
#pragma unroll
  for (int cc = 0; cc < 2; ++cc)
    if (cc < a.w && warp == cc / CPW) {
#pragma unroll
      for (int q = 0; q < PR_RL; ++q) {
        double v = 0.0;
#pragma unroll
        for (int c = 0; c < CPW; ++c)
          if (c == cc % CPW) v = P[q][c];
        xsb[cc * XS + lane + 32 * q] = v;
      }
    }
  unsigned epoch = 0;
  int par = 0;
  int tp0 = -1, tp1 = -1;   // reflectors of the previous step whose T columns are still to be built (CTA 0)
  __syncthreads();

  for (int t = 0; t < a.kk;) {
    const bool pair = t + 1 < a.kk;
    const double* x1 = xsb + (2 * par) * XS;
    const double* x2 = x1 + XS;
    // ---- 1. Gram slots of this warp's columns: G1 over rows > t, G2 over rows > t + 1; rows t and t + 1
    double acc[NV];
#pragma unroll
    for (int c = 0; c < NV; ++c) acc[c] = 0.0;
    int qt = -1, qt2 = -1;
#pragma unroll
    for (int q = 0; q < PR_RL; ++q) {
      const int i = lane + 32 * q;
      const int64_t r = rlo + i;
      const bool ok = i < nr;
      const double x = (ok && r > t) ? x1[i] : 0.0;
      const double y = (ok && pair && r > t + 1) ? x2[i] : 0.0;
      if (ok && r == t) qt = q;
      if (ok && r == t + 1) qt2 = q;
#pragma unroll
      for (int c = 0; c < CPW; ++c) {
        acc[c] = fma(x, P[q][c], acc[c]);
        acc[CPW + c] = fma(y, P[q][c], acc[CPW + c]);
      }
    }
    double* mp = mypart + par * RS;
    {
      int qb;
      const double f = warp_butterfly<NV>(acc, lane, qb);
      constexpr int LV = NV >= 16 ? 4 : (NV == 8 ? 3 : (NV == 4 ? 2 : 1));
      if ((lane & ((32 >> LV) - 1)) == 0) mp[qb < CPW ? j0 + qb : W + j0 + qb - CPW] = f;
    }
    // rows t and t + 1 of this warp's columns (owner lane) or zero
#pragma unroll
    for (int rr = 0; rr < 2; ++rr) {
      const int qo = rr ? qt2 : qt;
      const unsigned own = __ballot_sync(0xffffffffu, qo >= 0);
      double* dst = mp + (2 + rr) * W + j0;
      if (own) {
        const int src = __ffs(own) - 1;
#pragma unroll
        for (int c = 0; c < CPW; ++c) {
          double vv = 0.0;
#pragma unroll
          for (int q = 0; q < PR_RL; ++q)
            if (q == qo) vv = P[q][c];
          vv = __shfl_sync(0xffffffffu, vv, src);
          if (lane == 0) dst[c] = vv;
        }
      } else if (lane < CPW) {
        dst[lane] = 0.0;
      }
    }
    // ---- 2. cluster reduction through DSMEM (fixed order over the cluster's CTAs)
    cl.sync();
    for (int k = tid / PR_CL; PR_CL * k < RS; k += PR_NT / PR_CL) {
      const int c = tid % PR_CL;
      const int sl = crank + PR_CL * k;
      double v = 0.0;
      if (sl < RS) {
        const double* rp = cl.map_shared_rank(mypart + par * RS, c);
        v = rp[sl];
      }
#pragma unroll
      for (int o = 1; o < PR_CL; o <<= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
      if (c == 0 && sl < RS) __stcg(a.gpart + ((size_t)par * NC + cid) * RS + sl, v);
    }
    // ---- 3. one grid barrier; CTA 0 builds the previous step's T columns meanwhile (warps 2-3, named barrier)
    __syncthreads();
    epoch += 1;
    if (tid == 0) asm volatile("red.release.gpu.global.add.u32 [%0], 1;\n" ::"l"(a.bar + 32 * (g % PR_NBAR)) : "memory");
    if (g == 0 && tid >= 64 && tid < 128 && tp0 >= 0) {
      const int u = tid - 64;
      for (int pass = 0; pass < 2; ++pass) {
        const int c = pass ? tp1 : tp0;
        if (c < 0) break;
        for (int q2 = u; q2 < W; q2 += 64) {
          double v = 0.0;
          if (q2 < c) {
            double sacc = 0.0;
            for (int p = q2; p < c; ++p) sacc += Ts[q2 + p * W] * Dm[c * W + p];
            v = -taus[c] * sacc;
          } else if (q2 == c) {
            v = taus[c];
          }
          Ts[q2 + c * W] = v;
        }
        asm volatile("bar.sync 1, 64;\n" ::: "memory");
      }
    }
    if (tid < PR_NBAR) {
      const unsigned target = epoch * (unsigned)((G - tid + PR_NBAR - 1) / PR_NBAR);
      const unsigned* cnt = a.bar + 32 * tid;
      while (ld_relaxed_u32(cnt) < target) {
      }
      (void)ld_acquire_u32(cnt);
    }
    __syncthreads();
    // ---- 4. totals over the NC cluster partials, fixed order
    for (int sl = tid; sl < RS; sl += PR_NT) {
      double vals[PR_MAXNC];
#pragma unroll
      for (int q = 0; q < PR_MAXNC; ++q) vals[q] = q < NC ? __ldcg(a.gpart + ((size_t)par * NC + q) * RS + sl) : 0.0;
      double v = vals[0];
#pragma unroll
      for (int q = 1; q < PR_MAXNC; ++q)
        if (q < NC) v += vals[q];
      tot[sl] = v;
    }
    __syncthreads();
    // ---- 5. reflector p (and q), update, T inputs
    const double* G1 = tot;
    const double* G2 = tot + W;
    const double* Rp = tot + 2 * W;
    const double* Rq = tot + 3 * W;
    const House h = make_house(Rp[t], G1[t]);
    bool two = false;
    House h2{0.0, 0.0, 0.0};
    double cq = 0.0, rqp = 0.0, g1pq = 0.0;
    if (pair) {
      const double wq = Rp[t + 1] + h.scale * G1[t + 1];
      cq = h.tau * h.scale * wq;
      rqp = Rq[t];
      g1pq = G1[t] - rqp * rqp;
      const double t1 = G2[t + 1], t2 = 2.0 * cq * G2[t], t3 = cq * cq * g1pq;
      const double sig2 = t1 - t2 + t3;
      two = sig2 >= 0.0625 * (fabs(t1) + fabs(t2) + cq * cq * (G1[t] + rqp * rqp));
      if (two) h2 = make_house(Rq[t + 1] - cq * rqp, sig2);
    }
    double cj[CPW], tw[CPW], dj[CPW], tw2[CPW];
#pragma unroll
    for (int c = 0; c < CPW; ++c) {
      const int j = j0 + c;
      const double wj = Rp[j] + h.scale * G1[j];
      cj[c] = h.tau * h.scale * wj;
      tw[c] = -h.tau * wj;
      dj[c] = 0.0;
      tw2[c] = 0.0;
      if (two) {
        const double ajq = Rq[j] - cj[c] * rqp;
        const double sj = G2[j] - cj[c] * G2[t] - cq * (G1[j] - rqp * Rq[j]) + cq * cj[c] * g1pq;
        const double w2 = ajq + h2.scale * sj;
        dj[c] = h2.tau * h2.scale * w2;
        tw2[c] = -h2.tau * w2;
      }
    }
    if (!two) {
      // reflector t alone (as panel_reg_kernel)
      if (j0 > t) {
#pragma unroll
        for (int q = 0; q < PR_RL; ++q) {
          const int i = lane + 32 * q;
          const int64_t r = rlo + i;
          if (i < nr && r >= t) {
            const double vr = r > t ? h.scale * x1[i] : 1.0;
#pragma unroll
            for (int c = 0; c < CPW; ++c) P[q][c] = fma(tw[c], vr, P[q][c]);
          }
        }
      } else if (j0 + CPW > t) {
#pragma unroll
        for (int q = 0; q < PR_RL; ++q) {
          const int i = lane + 32 * q;
          const int64_t r = rlo + i;
          if (i >= nr || r < t) continue;
          const double vr = r > t ? h.scale * x1[i] : 1.0;
#pragma unroll
          for (int c = 0; c < CPW; ++c) {
            const int j = j0 + c;
            if (j > t) P[q][c] = fma(tw[c], vr, P[q][c]);
            else if (j == t) P[q][c] = r > t ? vr : h.beta;
          }
        }
      }
    } else {
      const int q1 = t + 1;
      if (j0 > q1) {
        // every column right of q: a'' = a - c_j a_p - d_j a'_q below q; row q: a - c_j a_p(q) - tau' w'_j;
        // row p: a - tau w_j
#pragma unroll
        for (int q = 0; q < PR_RL; ++q) {
          const int i = lane + 32 * q;
          const int64_t r = rlo + i;
          if (i < nr && r >= t) {
            const double xp = x1[i];
            const double aq = x2[i] - cq * xp;
            if (r > q1) {
#pragma unroll
              for (int c = 0; c < CPW; ++c) P[q][c] = fma(-dj[c], aq, fma(-cj[c], xp, P[q][c]));
            } else if (r == q1) {
#pragma unroll
              for (int c = 0; c < CPW; ++c) P[q][c] = fma(-cj[c], xp, P[q][c]) + tw2[c];
            } else {
#pragma unroll
              for (int c = 0; c < CPW; ++c) P[q][c] += tw[c];
            }
          }
        }
      } else if (j0 + CPW > t) {
#pragma unroll
        for (int q = 0; q < PR_RL; ++q) {
          const int i = lane + 32 * q;
          const int64_t r = rlo + i;
          if (i >= nr || r < t) continue;
          const double xp = x1[i];
          const double aq = x2[i] - cq * xp;
#pragma unroll
          for (int c = 0; c < CPW; ++c) {
            const int j = j0 + c;
            if (j > q1) {
              if (r > q1) P[q][c] = fma(-dj[c], aq, fma(-cj[c], xp, P[q][c]));
              else if (r == q1) P[q][c] = fma(-cj[c], xp, P[q][c]) + tw2[c];
              else P[q][c] += tw[c];
            } else if (j == q1) {
              if (r > q1) P[q][c] = h2.scale * aq;
              else if (r == q1) P[q][c] = h2.beta;
              else P[q][c] += tw[c];
            } else if (j == t) {
              P[q][c] = r > t ? h.scale * xp : h.beta;
            }
          }
        }
      }
    }
    if (g == 0) {
      // v_t^T v_s (s < t) as panel_reg_kernel; v_q^T v_s (s < q) from the pair's sums
      for (int sp = tid; sp < t; sp += PR_NT) {
        Dm[t * W + sp] = Rp[sp] + h.scale * G1[sp];
        if (two) Dm[(t + 1) * W + sp] = Rq[sp] + h2.scale * (G2[sp] - cq * (G1[sp] - rqp * Rq[sp]));
      }
      if (tid == 0) {
        taus[t] = h.tau;
        a.tau[t] = h.tau;
        if (two) {
          Dm[(t + 1) * W + t] = h.scale * rqp + h2.scale * h.scale * (G2[t] - cq * g1pq);
          taus[t + 1] = h2.tau;
          a.tau[t + 1] = h2.tau;
        }
      }
    }
    tp0 = t;
    tp1 = two ? t + 1 : -1;
    const int tn = t + (two ? 2 : 1);
    // next pair of columns -> the other parity's buffers (their previous readers finished before this barrier)
#pragma unroll
    for (int cc = 0; cc < 2; ++cc) {
      const int col = tn + cc;
      if (col < a.w && warp == col / CPW) {
        double* xn = xsb + (2 * (par ^ 1) + cc) * XS;
        const int cn = col % CPW;
#pragma unroll
        for (int q = 0; q < PR_RL; ++q) {
          double v = 0.0;
#pragma unroll
          for (int c = 0; c < CPW; ++c)
            if (c == cn) v = P[q][c];
          xn[lane + 32 * q] = v;
        }
      }
    }
    t = tn;
    par ^= 1;
    __syncthreads();
  }
  if (g == 0) {
    // T columns of the last step
    for (int pass = 0; pass < 2; ++pass) {
      const int c = pass ? tp1 : tp0;
      if (c >= 0) t_column(Ts, Dm, taus, c, W, tid);
      __syncthreads();
    }
  }
#pragma unroll
  for (int q = 0; q < PR_RL; ++q) {
    const int i = lane + 32 * q;
    if (i >= nr) continue;
    const int64_t r = rlo + i;
#pragma unroll
    for (int c = 0; c < CPW; ++c) {
      const int j = j0 + c;
      if (j < a.w) a.P[r + (int64_t)j * a.ldp] = P[q][c];
      if (j < a.kk) a.Y[r + (int64_t)j * a.ldy] = r > j ? P[q][c] : (r == j ? 1.0 : 0.0);
    }
  }
  if (g == 0) {
    for (int idx = tid; idx < W * W; idx += PR_NT) {
      const int q2 = idx % W, c = idx / W;
      a.T[q2 + (int64_t)c * a.ldt] = (c < a.kk) ? Ts[q2 + c * W] : 0.0;
    }
  }
  cl.sync();
}

size_t panel_reg_gpart_bytes(int w) { return sizeof(double) * 2 * PR_MAXNC * 4 * (size_t)w; }

// TRID_PANEL_PAIR=0 selects the one-reflector-per-barrier kernel (A/B); default: two per barrier
static bool panel_pair() {
  static const bool on = !(getenv("TRID_PANEL_PAIR") && getenv("TRID_PANEL_PAIR")[0] == '0');
  return on;
}
static size_t panel_reg_smem(int w) {
  if (panel_pair()) return sizeof(double) * (size_t)(4 * 32 * PR_RL + 3 * 4 * w + 2 * w * w + w);
  return sizeof(double) * (size_t)(2 * 32 * PR_RL + 2 * 2 * w + 2 * w + 2 * w * w + w + 2 * w);
}
static const void* panel_reg_fn(int w) {
  if (panel_pair())
    return w == 16 ? (const void*)panel_reg2_kernel<2>
                   : (w == 32 ? (const void*)panel_reg2_kernel<4> : (const void*)panel_reg2_kernel<8>);
  return w == 16 ? (const void*)panel_reg_kernel<2>
                 : (w == 32 ? (const void*)panel_reg_kernel<4> : (const void*)panel_reg_kernel<8>);
}
// Co-resident 4-CTA clusters of the kernel for width w on the current device (cached per device and width;
// a racing first query stores the same value twice).  0 if the query fails (the caller then takes the general
// panel kernel).
static int panel_reg_max_clusters(int w) {
  static std::atomic<int> cache[kMaxDevices][3];
  const int wi = w == 16 ? 0 : (w == 32 ? 1 : 2);
  const int d = cur_device();
  int nc = cache[d][wi].load(std::memory_order_relaxed);
  if (nc != 0) return nc < 0 ? 0 : nc;
  const size_t smem = panel_reg_smem(w);
  const void* fn = panel_reg_fn(w);
  nc = -1;
  if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) == cudaSuccess) {
    cudaLaunchConfig_t q = {};
    q.gridDim = dim3(PR_CL * PR_MAXNC);
    q.blockDim = dim3(PR_NT);
    q.dynamicSmemBytes = smem;
    cudaLaunchAttribute qa[1];
    qa[0].id = cudaLaunchAttributeClusterDimension;
    qa[0].val.clusterDim.x = PR_CL;
    qa[0].val.clusterDim.y = 1;
    qa[0].val.clusterDim.z = 1;
    q.attrs = qa;
    q.numAttrs = 1;
    int v = 0;
    if (cudaOccupancyMaxActiveClusters(&v, fn, &q) == cudaSuccess && v >= 1) nc = v > PR_MAXNC ? PR_MAXNC : v;
  }
  (void)cudaGetLastError();
  cache[d][wi].store(nc, std::memory_order_relaxed);
  return nc < 0 ? 0 : nc;
}

bool panel_reg_supported(int64_t m, int w) {
  // every CTA holds <= 32 * PR_RL rows in registers, and the grid is limited to co-resident clusters (33 of 4
  // on an idle B200: m <= 33792); otherwise (fewer SMs, MPS limits, taller panels) the general kernel runs
  if (!(w == 16 || w == 32 || w == 64) || m < 1) return false;
  const int nc = panel_reg_max_clusters(w);
  return nc >= 1 && m <= (int64_t)PR_CL * nc * 32 * PR_RL;
}

cudaError_t panel_qr_reg(int64_t m, int w, double* P, int64_t ldp, double* tau, double* T, int64_t ldt, double* Y,
                         int64_t ldy, double* gpart, unsigned* bar, cudaStream_t st) {
  PanelRegArgs a;
  a.m = m; a.w = w; a.kk = (int)(m < w ? m : w);
  a.P = P; a.ldp = ldp; a.tau = tau; a.T = T; a.ldt = ldt; a.Y = Y; a.ldy = ldy; a.gpart = gpart; a.bar = bar;
  {
    // trace area: past the cluster partials inside the panel workspace (panel_red_bytes reserves it)
    static const char* tr = getenv("TRID_PANEL_TRACE");
    a.trace = (tr && atoll(tr) == m) ? (long long*)(gpart + 2 * (size_t)kNumSMsB200 * 2 * w + 2 * 2 * (size_t)w)
                                     : nullptr;
  }
  const size_t smem = panel_reg_smem(w);
  const int maxc = panel_reg_max_clusters(w);
  if (maxc < 1) return cudaErrorInvalidConfiguration;   // caller checks panel_reg_supported
  // as few rows per CTA as possible within the co-resident clusters (target 64 rows per CTA; env
  // TRID_PANEL_ROWS=r for A/B: the grid barrier's cost grows with G, the per-column work with the rows)
  static const int prow = [] {
    const char* e = getenv("TRID_PANEL_ROWS");
    const int v = e ? atoi(e) : 64;
    return v >= 16 && v <= 32 * PR_RL ? v : 64;
  }();
  int64_t G = (m + prow - 1) / prow;
  G = (G + PR_CL - 1) / PR_CL * PR_CL;
  if (G > (int64_t)PR_CL * maxc) G = (int64_t)PR_CL * maxc;
  if (G < PR_CL) G = PR_CL;
  a.rows = (int)((m + G - 1) / G);
  if (a.rows > 32 * PR_RL) return cudaErrorInvalidConfiguration;   // caller checks panel_reg_supported
  cudaError_t e = cudaMemsetAsync(bar, 0, sizeof(unsigned) * 32 * PR_NBAR, st);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)G);
  cfg.blockDim = dim3(PR_NT);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = PR_CL;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeCooperative;
  attr[1].val.cooperative = 1;
  cfg.attrs = attr;
  // The cooperative attribute guarantees co-residency for the grid barrier.  Nsight Compute aborts the
  // application on a cooperative cluster launch; under it (and with TRID_PANEL_NOCOOP=1) the grid is launched
  // without the attribute: it fits in one wave (G <= 4 x co-resident clusters) and the profiler serialises
  // kernels, so every CTA is resident anyway.  A refused cooperative launch is retried the same way.
  cfg.numAttrs = profiler_attached() ? 1 : 2;
  count_launches(1);
  auto launch = [&]() -> cudaError_t {
    if (panel_pair()) {
      switch (w) {
        case 16: return cudaLaunchKernelEx(&cfg, panel_reg2_kernel<2>, a);
        case 32: return cudaLaunchKernelEx(&cfg, panel_reg2_kernel<4>, a);
        default: return cudaLaunchKernelEx(&cfg, panel_reg2_kernel<8>, a);
      }
    }
    switch (w) {
      case 16: return cudaLaunchKernelEx(&cfg, panel_reg_kernel<2>, a);
      case 32: return cudaLaunchKernelEx(&cfg, panel_reg_kernel<4>, a);
      default: return cudaLaunchKernelEx(&cfg, panel_reg_kernel<8>, a);
    }
  };
  e = launch();
  if (e != cudaSuccess && cfg.numAttrs == 2) {
    (void)cudaGetLastError();
    cfg.numAttrs = 1;
    e = launch();
  }
  return e;
}

}  // namespace trid
