// panel_qr.cu — tall-skinny Householder panel QR for DBBR (Alg. 1 line 5) plus the
// compact-WY factor T (dlarft forward-columnwise) and the explicit Y = V.
//
// B200 design: one cooperative persistent grid of G <= 148 CTAs; CTA g owns a contiguous block of
// panel rows, staged in shared memory when it fits (<= ~220 KB).  Column t needs ONE grid-wide
// reduction: every CTA contributes the Gram row  sum_{r>t} x_r P(r,j)  (x = column t below row t,
// unscaled) for all j and the owner of row t contributes P(t, :).  From those totals every CTA
// derives, identically and deterministically, beta/tau/scale of the reflector (R1), the update
// vector w_j = v^T P(:,j) = P(t,j) + scale * sum x_r P(r,j) (j > t) and the T-factor inner products
// v_t^T v_q (q < t), then applies the rank-1 update to its own rows.  Totals are summed in a fixed
// CTA order, so every CTA (and every run) sees bitwise-identical values.
#include "backtrans.cuh"
#include "common.cuh"
#include "gemm.cuh"
#include "panel.cuh"
#include "prof.cuh"

#include <stdlib.h>

namespace trid {

constexpr int PQ_NT = 256;

struct PanelArgs {
  int64_t m;
  int w, kk;
  double* P;
  int64_t ldp;
  double* tau;
  double* T;
  int64_t ldt;
  double* Y;
  int64_t ldy;
  double* red;
  double* tot;
  unsigned* bar;
  int rows;      // rows per CTA
  int smem_ld;   // > 0: rows staged in shared memory with this leading dimension
  int t_smem;    // 1: CTA 0 keeps T in shared memory (w x w) and writes it out at the end
  long long* trace;   // debug (TRID_PANEL_TRACE): %globaltimer per column phase, CTAs 0 and G-1
};
__device__ __forceinline__ long long pq_gtimer() {
  long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#define PQ_TRACE(k)                                                                               \
  do {                                                                                            \
    if (a.trace && tid == 0 && (g == 0 || g == G - 1) && t < 256)                                 \
      a.trace[((g == 0 ? 0 : 1) * 256 + t) * 8 + (k)] = pq_gtimer();                              \
  } while (0)

__global__ void __launch_bounds__(PQ_NT, 1) panel_qr_kernel(PanelArgs a) {
  extern __shared__ __align__(16) double sm[];
  const int g = blockIdx.x, G = gridDim.x, tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31;
  constexpr int NW = PQ_NT / 32;
  const int w = a.w, RS = 2 * w;
  const int64_t rlo = (int64_t)g * a.rows;
  const int nr = (int)((rlo + a.rows <= a.m) ? a.rows : (a.m > rlo ? a.m - rlo : 0));

  double* L;
  int64_t ldl;
  double* scr;
  if (a.smem_ld > 0) {
    L = sm;
    ldl = a.smem_ld;
    scr = sm + (size_t)a.smem_ld * w;
    for (int idx = tid; idx < nr * w; idx += PQ_NT) {
      const int i = idx % nr, j = idx / nr;
      L[(size_t)j * ldl + i] = a.P[(rlo + i) + (int64_t)j * a.ldp];
    }
  } else {
    L = a.P + rlo;
    ldl = a.ldp;
    scr = sm;
  }
  double* tot = scr;            // RS totals
  double* wv = tot + RS;        // w: update vector (j > t) / v_t^T v_q (q < t)
  double* tmp = wv + w;         // H*RS <= PQ_NT partial totals
  double* hs = tmp + PQ_NT;     // beta, tau, scale
  double* Ts = hs + 8;          // w x w (only if t_smem; CTA 0)
  double* Tw = a.t_smem ? Ts : a.T;
  const int64_t ldT = a.t_smem ? w : a.ldt;
  __syncthreads();

  unsigned epoch = 0;
  for (int t = 0; t < a.kk; ++t) {
    PQ_TRACE(0);
    double* red = a.red + (size_t)(t & 1) * G * RS;
    // ---- partial Gram row: slot j = sum_{r > t, r owned} P(r,t) P(r,j);  slot w+j = P(t,j) (owner)
    const int i0 = (int)((t + 1 - rlo) > 0 ? (t + 1 - rlo) : 0);
    const double* xc = L + (size_t)t * ldl;
    for (int j = warp; j < w; j += NW) {
      const double* pc = L + (size_t)j * ldl;
      double s = 0.0;
      for (int i = i0 + lane; i < nr; i += 32) s += xc[i] * pc[i];
      s = warp_sum(s);
      if (lane == 0) red[(size_t)g * RS + j] = s;
    }
    const bool owner = (t >= rlo) && (t < rlo + nr);
    for (int j = tid; j < w; j += PQ_NT) red[(size_t)g * RS + w + j] = owner ? L[(size_t)j * ldl + (t - rlo)] : 0.0;
    PQ_TRACE(1);
    grid_barrier(a.bar, (unsigned)G, epoch);
    PQ_TRACE(2);
    // ---- distributed reduction: CTA g sums slots s = g, g+G, ... over all CTAs in a fixed order
    {
      const double* src = a.red + (size_t)(t & 1) * G * RS;
      double* dst = a.tot + (size_t)(t & 1) * RS;
      for (int s = g; s < RS; s += G) {
        double x = 0.0;
        for (int gg = tid; gg < G; gg += PQ_NT) x += __ldcg(src + (size_t)gg * RS + s);
        x = warp_sum(x);
        if (lane == 0) tmp[warp] = x;
        __syncthreads();
        if (tid == 0) {
          double acc = 0.0;
          for (int q = 0; q < NW; ++q) acc += tmp[q];
          __stcg(dst + s, acc);
        }
        __syncthreads();
      }
    }
    PQ_TRACE(3);
    grid_barrier(a.bar, (unsigned)G, epoch);
    PQ_TRACE(4);
    for (int s = tid; s < RS; s += PQ_NT) tot[s] = __ldcg(a.tot + (size_t)(t & 1) * RS + s);
    __syncthreads();
    PQ_TRACE(5);
    // ---- reflector (R1), update vector, T inner products
    const House h = make_house(tot[w + t], tot[t]);
    for (int j = tid; j < w; j += PQ_NT) {
      if (j != t) wv[j] = tot[w + j] + h.scale * tot[j];
    }
    if (tid == 0) { hs[0] = h.beta; hs[1] = h.tau; hs[2] = h.scale; }
    __syncthreads();
    // ---- apply to owned rows:  v_r = scale * x_r (r > t), v_t = 1;  P(r,j) -= tau * w_j * v_r (j > t)
    for (int i = tid; i < nr; i += PQ_NT) {
      const int64_t r = rlo + i;
      if (r > t) {
        const double v = h.scale * L[(size_t)t * ldl + i];
        L[(size_t)t * ldl + i] = v;
        const double tv = h.tau * v;
        for (int j = t + 1; j < w; ++j) L[(size_t)j * ldl + i] -= tv * wv[j];
      } else if (r == t) {
        L[(size_t)t * ldl + i] = h.beta;
        for (int j = t + 1; j < w; ++j) L[(size_t)j * ldl + i] -= h.tau * wv[j];
      }
    }
    PQ_TRACE(6);
    // ---- T(:, t) (CTA 0): T(t,t) = tau; T(0:t,t) = -tau T(0:t,0:t) (V^T v_t); zeros below
    if (g == 0) {
      for (int q = tid; q < w; q += PQ_NT) {
        double v = 0.0;
        if (q < t) {
          double s = 0.0;
          for (int p = q; p < t; ++p) s += Tw[q + (int64_t)p * ldT] * wv[p];
          v = -h.tau * s;
        } else if (q == t) {
          v = h.tau;
        }
        Tw[q + (int64_t)t * ldT] = v;
      }
      if (tid == 0) a.tau[t] = h.tau;
    }
    __syncthreads();
    PQ_TRACE(7);
  }
  // zero the unused columns of T (kk < w); write T out if it lived in shared memory
  if (g == 0) {
    for (int idx = tid; idx < (w - a.kk) * w; idx += PQ_NT) {
      const int q = idx % w, c = a.kk + idx / w;
      Tw[q + (int64_t)c * ldT] = 0.0;
    }
    if (a.t_smem) {
      __syncthreads();
      for (int idx = tid; idx < w * w; idx += PQ_NT) a.T[(idx % w) + (int64_t)(idx / w) * a.ldt] = Ts[idx];
    }
  }
  // ---- write back (R above, V below) and explicit Y = V (unit diagonal, zeros above)
  if (a.smem_ld > 0) {
    for (int idx = tid; idx < nr * w; idx += PQ_NT) {
      const int i = idx % nr, j = idx / nr;
      a.P[(rlo + i) + (int64_t)j * a.ldp] = L[(size_t)j * ldl + i];
    }
  }
  for (int idx = tid; idx < nr * a.kk; idx += PQ_NT) {
    const int i = idx % nr, c = idx / nr;
    const int64_t r = rlo + i;
    const double v = r > c ? L[(size_t)c * ldl + i] : (r == c ? 1.0 : 0.0);
    a.Y[r + (int64_t)c * a.ldy] = v;
  }
}

static int panel_grid(int64_t m) {
  int64_t G = (m + 63) / 64;
  if (G > num_sms()) G = num_sms();   // 1 CTA/SM (launch bounds, shared memory): co-resident for the grid barrier
  if (G < 1) G = 1;
  return (int)G;
}

constexpr int PB_IB = 64;   // inner block of the nb-blocked panel (the register kernel's widest panel)
static size_t panel_base_bytes(int w) {
  return sizeof(double) * (2 * (size_t)kNumSMsB200 * 2 * (size_t)w + 2 * 2 * (size_t)w) + sizeof(long long) * 2 * 256 * 8;
}
// blocked-path scratch (w > 64): T_k (ib x ib), X and X2 (ib x w), the Gram G (w x w), split-K partials (16 w^2)
static size_t panel_blocked_elems(int w) {
  return (size_t)PB_IB * PB_IB + 2 * (size_t)PB_IB * w + (size_t)w * w + 16 * (size_t)w * w;
}
size_t panel_red_bytes(int w) {
  size_t base = (panel_base_bytes(w) + 255) / 256 * 256;
  if (w > PB_IB) base += sizeof(double) * panel_blocked_elems(w);
  return base;
}

// nb-blocked panel QR for w > 64 (north_star: "Householder panel QR on nb-wide panels"): the panel is
// factored in sub-panels of ib = 64 columns by the register kernel; after each, its compact-WY block (I - Y_k T_k
// Y_k^T) is applied from the left (transposed) to the remaining columns with three DMMA contractions
// (X = Y_k^T C, X2 = T_k^T X, C -= Y_k X2); finally T of the whole panel from the Gram Y^T Y (dlarft).  The
// reflectors are those of the unblocked column-by-column QR (blocked Householder QR), up to rounding.
static cudaError_t panel_qr_blocked(int64_t m, int w, double* P, int64_t ldp, double* tau, double* T, double* Y,
                                    int64_t ldy, double* red, unsigned* bar, cudaStream_t st) {
  const int ib = PB_IB;
  const int kk = (int)(m < w ? m : w);
  double* scr = (double*)((char*)red + (panel_base_bytes(w) + 255) / 256 * 256);
  double* Tk = scr;
  double* X = Tk + (size_t)ib * ib;
  double* X2 = X + (size_t)ib * w;
  double* G = X2 + (size_t)ib * w;
  double* part = G + (size_t)w * w;
  const int64_t part_elems = 16 * (int64_t)w * w;
  cudaError_t e = cudaMemset2DAsync(Y, sizeof(double) * ldy, 0, sizeof(double) * m, kk, st);
  if (e != cudaSuccess) return e;
  for (int k = 0; k < kk; k += ib) {
    // sub-panel columns [k, k + bw) (bw in {16, 32, 64}: w % 16 == 0), min(m - k, bw) reflectors
    const int bw = (w - k) < ib ? (w - k) : ib;
    const int64_t mk = m - k;
    const int bk = (int)(mk < bw ? mk : bw);
    if ((e = panel_qr_reg(mk, bw, P + k + (int64_t)k * ldp, ldp, tau + k, Tk, ib, Y + k + (int64_t)k * ldy, ldy, red,
                          bar, st)) != cudaSuccess)
      return e;
    const int nc = w - k - bw;
    if (nc <= 0) continue;
    double* C = P + k + (int64_t)(k + bw) * ldp;
    const double* Yk = Y + k + (int64_t)k * ldy;
    if ((e = gemm_ws_mm(OP_T, OP_N, bk, nc, mk, 1.0, Yk, ldy, C, ldp, 0.0, X, ib, part, part_elems, st)) != cudaSuccess)
      return e;
    if ((e = gemm_ws_mm(OP_T, OP_N, bk, nc, bk, 1.0, Tk, ib, X, ib, 0.0, X2, ib, part, part_elems, st)) != cudaSuccess)
      return e;
    if ((e = gemm_ws_mm(OP_N, OP_N, mk, nc, bk, -1.0, Yk, ldy, X2, ib, 1.0, C, ldp, part, part_elems, st)) !=
        cudaSuccess)
      return e;
  }
  // T of the whole panel: G = Y^T Y, then the dlarft recurrence (one CTA)
  if ((e = gemm_ws_mm(OP_T, OP_N, kk, kk, m, 1.0, Y, ldy, Y, ldy, 0.0, G, w, part, part_elems, st)) != cudaSuccess)
    return e;
  if ((e = cudaMemsetAsync(T, 0, sizeof(double) * (size_t)w * w, st)) != cudaSuccess) return e;
  return tfactor_from_gram(w, kk, G, tau, T, st);
}

cudaError_t panel_qr(int64_t m, int w, double* P, int64_t ldp, double* tau, double* T, int64_t ldt, double* Y,
                     int64_t ldy, double* red, unsigned* bar, cudaStream_t st) {
  if (m <= 0 || w <= 0) return cudaSuccess;
  static const bool force_general = getenv("TRID_PANEL_SMEM") != nullptr;   // A/B: the general kernel for every w
  if (panel_reg_supported(m, w) && !force_general) return panel_qr_reg(m, w, P, ldp, tau, T, ldt, Y, ldy, red, bar, st);
  if (w > PB_IB && w % 16 == 0 && ldt == w && panel_reg_supported(m, PB_IB) && !force_general)
    return panel_qr_blocked(m, w, P, ldp, tau, T, Y, ldy, red, bar, st);
  const int G = panel_grid(m);
  PanelArgs a;
  a.m = m; a.w = w; a.kk = (int)(m < w ? m : w);
  a.P = P; a.ldp = ldp; a.tau = tau; a.T = T; a.ldt = ldt; a.Y = Y; a.ldy = ldy; a.red = red; a.tot = red + 2 * (size_t)kNumSMsB200 * 2 * w; a.bar = bar;
  a.rows = (int)((m + G - 1) / G);
  {
    static const char* tr = getenv("TRID_PANEL_TRACE");   // "m": trace the panel with this many rows
    a.trace = (tr && atoll(tr) == m) ? (long long*)(red + 2 * (size_t)kNumSMsB200 * 2 * w + 2 * 2 * (size_t)w) : nullptr;
  }
  const size_t scr = sizeof(double) * (size_t)(2 * w + w + PQ_NT + 8);
  const size_t tsz = sizeof(double) * (size_t)w * w;
  const size_t full = sizeof(double) * (size_t)a.rows * w + scr;
  const size_t kMaxSmem = 227 * 1024;
  size_t smem;
  if (full <= kMaxSmem) {
    a.smem_ld = a.rows;
    smem = full;
  } else {
    a.smem_ld = 0;
    smem = scr;
  }
  a.t_smem = smem + tsz <= kMaxSmem ? 1 : 0;
  if (a.t_smem) smem += tsz;
  static DeviceOnce attr;
  cudaError_t e0 = attr([&] {
    return cudaFuncSetAttribute(panel_qr_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kMaxSmem);
  });
  if (e0 != cudaSuccess) return e0;
  cudaError_t e = cudaMemsetAsync(bar, 0, sizeof(unsigned), st);
  if (e != cudaSuccess) return e;
  void* args[] = {&a};
  count_launches(1);
  if (profiler_attached()) {   // see panel_reg.cu: G <= SM count at 1 CTA/SM, one wave
    panel_qr_kernel<<<G, PQ_NT, smem, st>>>(a);
    return cudaGetLastError();
  }
  return cudaLaunchCooperativeKernel((const void*)panel_qr_kernel, dim3(G), dim3(PQ_NT), args, smem, st);
}

}  // namespace trid
