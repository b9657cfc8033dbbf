// bulge.cu — stage 2: bulge chasing from band b to tridiagonal on one GPU (sec. 2.4 Fig. 3, Alg. 2
// P:278-303, sec. 5.2; readings R7-R9 in DESIGN.md).
//
// B200 design:
//   * band_pack (Fig. 10): the lower band is copied into a compact column-major array with
//     ldab = 2b doubles per column (room for the bulge, r - c <= 2b-1); at n = 32768, b = 64 this is
//     33.5 MB and stays L2-resident (126 MB L2).  A step's working set (columns R_m, rows R_m u R_m+1)
//     is then ONE contiguous span of L*ldab doubles.
//   * bc_kernel: persistent CTAs claim sweeps from an atomic ticket (forward progress without relying
//     on CTA rasterisation order).  Step m of sweep s waits until sweep s-1 has completed step m+1
//     (lag 2, R9) via ld.acquire.gpu on a per-sweep progress counter, and publishes its own progress
//     with st.release.gpu after its stores (the paper's volatile spin flag, made a
//     well-defined release/acquire pair).  For b <= 64 the step's window is staged into shared memory
//     (dense symmetric D = B_d and the b x b block O = B_od below it); larger b works on the L2-resident
//     compact band directly.  All reductions are in fixed order: the result is bitwise independent of
//     scheduling.
#include "common.cuh"
#include "panel.cuh"
#include "prof.cuh"
#include "driver.cuh"

#include <stdlib.h>
#include <type_traits>

namespace trid {

constexpr int BC_FLAG_STRIDE = 32;   // workspace room per counter (ints); bc_v6 uses 8 (one sector) unless TRID_BC_FS

struct BcArgs {
  int64_t n;
  int b, ldab;
  int vs;  // V2 stride per step (the caller's b; >= b)
  double* band;
  double* V2;
  double* tau2;
  int* prog;        // prog[s] = m+1: column 0 of step (s, m) published
  int* prog_full;   // prog_full[s] = m+1: all columns of step (s, m) stored
  unsigned* ticket;
  int fs;           // flag stride in ints (bc_v6: one 32-byte sector per sweep counter; other kernels: 1)
  int opt;          // bc_v6 hand-off options (TRID_BC_OPT bitmask, A/B; default 8|16): 1 STORE0 spins on test_wait,
                    // 2 column 0 stored by its 2B threads (STORE0 only releases), 4 LOAD polls with acquire loads,
                    // 8 per-warp step hand-off to STORE1 (no 4th CTA barrier), 16 full windows: the z barrier
                    // is per column group's O-row warps (B = 64)
  long long* trace;     // debug (TRID_BC_TRACE=s): %globaltimer per step phase for sweeps s and s+1
  int64_t trace_sweep;
  int serial;           // debug (TRID_BC_SERIAL=1): sweep s starts after sweep s-1 stored all its steps
};

__device__ __forceinline__ long long gtimer() {
  long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#define BC_TRACE(k)                                                                             \
  do {                                                                                          \
    if (a.trace && tid == 0 && (s == a.trace_sweep || s == a.trace_sweep + 1) && m < 1024) {   \
      a.trace[((s - a.trace_sweep) * 1024 + m) * 16 + (k)] = gtimer();                          \
      if ((k) == 2 || (k) == 3) a.trace[((s - a.trace_sweep) * 1024 + m) * 16 + 8 + (k)] = clock64(); \
      if ((k) >= 12) a.trace[((s - a.trace_sweep) * 1024 + m) * 16 + (k)] = clock64();         \
    }                                                                                           \
  } while (0)

__host__ __device__ inline int64_t bc_steps(int64_t n, int b, int64_t s) {
  if (b < 2 || s < 0 || s > n - 3) return 0;
  return (n - 3 - s) / b + 1;
}
// F(x) = sum_{u=0}^{x} (floor(u/b) + 1), F(-1) = 0
__host__ __device__ inline int64_t bc_F(int64_t x, int b) {
  if (x < 0) return 0;
  const int64_t q = x / b, r = x - q * b;
  return (int64_t)b * q * (q - 1) / 2 + q * (r + 1) + x + 1;
}
// S(s) = number of steps of sweeps 0..s-1 (V2/tau2 offset of sweep s, reading R7)
__host__ __device__ inline int64_t bc_offset(int64_t n, int b, int64_t s) {
  if (b < 2) return 0;
  return bc_F(n - 3, b) - bc_F(n - 3 - s, b);
}

int bc_ldab(int64_t n, int b) {
  (void)n;
  return b >= 2 ? 2 * b : 2;
}
int64_t bc_total_steps(int64_t n, int b) { return n >= 3 ? bc_offset(n, b, n - 2) : 0; }

// element (c+o, c) of the input band lives at X[o + c*cs] (full column-major A: X = A, cs = lda+1;
// LAPACK lower band storage AB: cs = ldab)
__global__ void band_pack_kernel(int64_t n, int b, int ldab, const double* X, int64_t cs, double* band) {
  const int64_t total = n * ldab;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total; idx += (int64_t)gridDim.x * blockDim.x) {
    const int64_t c = idx / ldab, o = idx - c * ldab;
    band[idx] = (o <= b && c + o < n) ? X[o + c * cs] : 0.0;
  }
}

__global__ void band_extract_kernel(int64_t n, int ldab, const double* band, double* d, double* e) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    d[i] = band[i * ldab];
    if (i + 1 < n) e[i] = band[i * ldab + 1];
  }
}

// debug trace (TRID_BC_TRACE=s): %globaltimer per step phase for sweeps s and s+1, slot k of 16
#define BCW_TRACE(S, M, K)                                                                          \
  do {                                                                                              \
    if (a.trace && ((S) == a.trace_sweep || (S) == a.trace_sweep + 1) && (M) < 1024)                \
      a.trace[(((S)-a.trace_sweep) * 1024 + (M)) * 16 + (K)] = gtimer();                            \
  } while (0)

// ---- v6: warp-specialized chase with a short column-0 path (default for b <= 64) ------------------------
// NTH compute threads (named barrier 1) + a LOAD warp + two STORE warps; no compute warp ever waits on global
// memory.  The step window M = [D; O] ((L+L2) x L) is held in registers, one row slice per thread (a warp covers
// 32 consecutive rows of one column group, so every compact-window access is bank-conflict free).
//   LOAD  (lane 0): claims sweeps (atomic ticket), and for every step fills a window buffer by bulk copies
//         completing on mbarriers (expect_tx): columns 0..L-2 once the predecessor sweep's prog_full reached
//         m+1, the last column once its prog reached min(m+2, nprev) (R9, lag 2), plus column s at a sweep's
//         step 0.  It runs one step ahead (prefetch) and only waits on the predecessor sweep and on the
//         buffer's empty barrier.
//   STORE0/STORE1 (lane 0 each): publish column 0 (prog) and columns 1..L-1 (prog_full), then free the buffer.
//         They never wait on another CTA, so publication cannot be held up by this CTA's own prefetch.
// Step/sweep ids travel with the buffer (info[buf]); s < 0 terminates all roles.  The design is organised
// around the chain that bounds the chase (Delta per sweep = step period + link, link = predecessor's
// column 0 -> our column 0):
//   * the last window column (sweep s-1's freshly published column 0) lands on its own mbarrier (lastb);
//     it contributes to one row of D v (the diagonal D(L-1,L-1)) and to every row of O v, so the body
//     matvec (columns 0..L-2) and its cross-group reduction run while it is in flight;
//   * column 0 of the step is then produced by 2B threads (one per window row) with ONE named barrier:
//     p = tau D v / y = O v are completed with one FMA, p^T v and |x(1:)|^2 (x = the right-updated O(:,0))
//     are warp-summed together, the reflector of x is formed once (its beta/tau/scale go to shared memory
//     for the rest of the step), and the new D(:,0), beta e1 are written to a column-0 staging buffer the
//     STORE warp publishes (prog) while the full two-sided update, the z pass and the left application of
//     the step continue on all compute threads;
//   * the rest of the step takes two barriers: the rank-2 update of D and the right update of O in registers,
//     z = vn^T O by transposed warp butterflies from registers, then the left update of O;
//   * full windows (L = L2 = b = B) are compiled separately (constant strides, warp-uniform D/O split) and
//     store columns 1..L-1 straight from registers to the band; STORE1 then only releases prog_full after the
//     CTA barrier (ragged windows and the CL variant bulk-store the shared window);
//   * the per-sweep counters sit one 32-byte sector apart (a.fs) and are polled without back-off (one lane
//     per CTA).
// All sums run in a fixed order (the last-column term is added after the body, z is summed by fixed
// butterflies): bitwise reproducible and independent of scheduling (tests: serialised-vs-parallel, R9).
__device__ __forceinline__ void wait_geq_spin(const int* p, int need) {
  while (ld_relaxed_s32(p) < need) {
  }
  (void)ld_acquire_s32(p);
}

__device__ __forceinline__ void mbar_spin(uint64_t* bar, unsigned parity) {
  unsigned done = 0;
  do {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  } while (!done);
}
__device__ __forceinline__ void wait_geq_opt(const int* p, int need, bool acq_loop) {
  if (acq_loop) {
    while (ld_acquire_s32(p) < need) {
    }
  } else {
    while (ld_relaxed_s32(p) < need) {
    }
    (void)ld_acquire_s32(p);
  }
}
// 32-bit shared-window accesses for the full-window path (immediate offsets, no generic address arithmetic)
__device__ __forceinline__ double lds_f64(uint32_t addr) {
  double v;
  asm volatile("ld.shared.f64 %0, [%1];\n" : "=d"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ void sts_f64(uint32_t addr, double v) {
  asm volatile("st.shared.f64 [%0], %1;\n" ::"r"(addr), "d"(v) : "memory");
}
__device__ __forceinline__ bool bc_step_full(int64_t n, int b, int B, int64_t s, int64_t m) {
  if (b != B || s < 0 || s > n - 3 || m < 0) return false;
  const int64_t r0 = s + 1 + m * b;
  return r0 + 2 * (int64_t)B - 1 <= n - 1;   // L == B and L2 == B
}
__device__ __forceinline__ unsigned cl_rank() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;\n" : "=r"(r));
  return r;
}
__device__ __forceinline__ unsigned cl_size() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_nctarank;\n" : "=r"(r));
  return r;
}
__device__ __forceinline__ unsigned cl_mapa(const void* p, unsigned rank) {
  unsigned r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;\n" : "=r"(r) : "r"(smem_u32(p)), "r"(rank));
  return r;
}
__device__ __forceinline__ void cl_st_release(unsigned raddr, int v) {
  asm volatile("st.release.cluster.shared::cluster.s32 [%0], %1;\n" ::"r"(raddr), "r"(v) : "memory");
}
__device__ __forceinline__ void cl_wait_geq(const int* p, int need) {
  int v;
  do {
    asm volatile("ld.acquire.cluster.shared::cta.s32 %0, [%1];\n" : "=r"(v) : "r"(smem_u32(p)) : "memory");
  } while (v < need);
}
// shared (this CTA) -> shared (peer CTA) bulk copy completing on the peer's mbarrier
__device__ __forceinline__ void bulk_s2s_cl(unsigned rdst, const void* src, unsigned bytes, unsigned rbar) {
  asm volatile("cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
                   rdst),
               "r"(smem_u32(src)), "r"(bytes), "r"(rbar)
               : "memory");
}
__device__ __forceinline__ void cl_sync_all() {
  asm volatile("barrier.cluster.arrive.release;\nbarrier.cluster.wait.acquire;\n" ::: "memory");
}

// CL (clusters of C CTAs, DSMEM forwarding): CTA rank q of cluster c runs sweeps (c + i*NC)*C + q, i = 0, 1, ...
// (static order; the persistent grid is sized to co-resident clusters).  Inside a cluster, sweep s+1 (rank q+1)
// receives sweep s's data for every full-window step straight from rank q's shared memory: the step's columns
// 1..L-1 (its window body) and column 0 of the next step (its last column) are bulk-copied CTA-to-CTA onto the
// consumer's own mbarriers, after the consumer announced (armed, a monotone step count in the producer's shared
// memory) that the target buffer is free and expecting them; the consumer acknowledges arrival (recv) so the
// producer can recycle its buffer.  The global band and the prog/prog_full counters are still written for every
// step (final result, cross-cluster consumers, ragged steps), but the in-cluster link no longer pays the release /
// poll / L2 round trips.
template <int B, int NTH, bool CL>
__device__ __forceinline__ void bc_v6_body(const BcArgs& a) {
  constexpr int TPR = NTH / (2 * B);
  constexpr int CPT = B / TPR;
  constexpr int RW = (2 * B) / 32;   // warps of the column-0 path (column group 0)
  constexpr int NW = NTH / 32;
  constexpr int CPW = B / NW;
  static_assert(CPW == 4 || CPW == 8, "z-pass butterfly assumes 4 or 8 columns per warp");
  extern __shared__ __align__(16) double sm[];
  const int b = a.b, ldab = a.ldab, tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int lda1 = ldab - 1;
  const int ldab_rt = ldab, lda1_rt = lda1;
  const int64_t n = a.n;
  const int wsz = B * ldab;
  double* colb = sm + 2 * wsz;               // 2 x ldab: column s of a sweep's step 0, per buffer
  double* c0s = colb + 2 * ldab;             // 2 x ldab: column-0 staging, per buffer
  double* vb = c0s + 2 * ldab;               // 2 x B   (v / vn)
  double* pyv = vb + 2 * B;                  // 2B
  double* zv = pyv + 2 * B;                  // B
  double* red = zv + B;                      // 2*RW warp partials, x0, beta/tau/scale (16)
  double* part = red + 16;                   // TPR x 2B
  double* xs = part + TPR * 2 * B;           // 2B: x = right-updated O(:, 0) by window row
  double* zp = xs + 2 * B;                   // RW x B: per-row-warp partials of z = vn^T O
  __shared__ __align__(8) uint64_t full[2], lastb[2], empty[2], col0b[2], colsb[2], c0done[2];
  __shared__ int64_t info_s[2];
  __shared__ int info_m[2];
  __shared__ int info_f[2];            // CL: the step's body/last column arrive from the producer CTA
  __shared__ int armed_ctr, recv_ctr;  // CL: written by the consumer CTA (monotone step counts)
  if (tid == 0) {
    armed_ctr = 0;
    recv_ctr = 0;
    for (int i = 0; i < 2; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&lastb[i], (!CL && (a.opt & 32)) ? 2 * B : 1);
      mbar_init(&empty[i], 1);
      mbar_init(&col0b[i], 2 * B);
      mbar_init(&colsb[i], (a.opt & 8) ? NW : 1);
      mbar_init(&c0done[i], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  unsigned crank = 0, csize = 1;
  if constexpr (CL) {
    crank = cl_rank();
    csize = cl_size();
    cl_sync_all();   // peers' barriers and counters are initialised before any remote access
  } else {
    __syncthreads();
  }
  const bool has_prod = CL && crank > 0;            // sweep s-1 runs on rank crank-1 of this cluster
  const bool has_cons = CL && crank + 1 < csize;    // sweep s+1 runs on rank crank+1
  if (warp == NW) {
    // ============================== LOAD warp ==============================
    if (lane != 0) return;
    uint32_t it = 0;
    for (int64_t sweep_i = 0;; ++sweep_i) {
      int64_t s;
      if constexpr (CL) s = ((int64_t)(blockIdx.x / csize) + sweep_i * (int64_t)(gridDim.x / csize)) * csize + crank;
      else s = (int64_t)atomicAdd(a.ticket, 1u);
      const bool done = s > n - 3;
      const int64_t nst = done ? 1 : bc_steps(n, b, s);
      const int64_t nprev = s > 0 ? bc_steps(n, b, s - 1) : 0;
      for (int64_t m = 0; m < nst; ++m, ++it) {
        const int bi = it & 1;
        if (it >= 2) mbar_wait(&empty[bi], ((it >> 1) - 1) & 1u);
        if (done) {
          info_s[bi] = -1;
          mbar_arrive(&full[bi]);
          return;
        }
        info_s[bi] = s;
        info_m[bi] = (int)m;
        BCW_TRACE(s, m, 7);
        const int64_t r0 = s + 1 + m * b;
        const int64_t r1 = (s + (m + 1) * b < n - 1) ? s + (m + 1) * b : n - 1;
        const int L = (int)(r1 - r0 + 1);
        double* win = sm + bi * wsz;
        const bool fwd = has_prod && bc_step_full(n, b, B, s, m);
        info_f[bi] = fwd;
        mbar_arrive_expect_tx(&full[bi], (unsigned)((L - 1 + (m == 0 ? 1 : 0)) * ldab * 8));
        const bool c0fetch = !CL && (a.opt & 32);   // the column-0 path threads fetch the last column themselves
        if (!c0fetch) mbar_arrive_expect_tx(&lastb[bi], (unsigned)(ldab * 8));
        if (fwd) {   // the producer CTA copies body (+ column s at m = 0) and the last column into this buffer
          cl_st_release(cl_mapa(&armed_ctr, crank - 1), (int)(it + 1));
          BCW_TRACE(s, m, 8);
          BCW_TRACE(s, m, 9);
          continue;
        }
        if (s > 0) {
          if (m == 0 && a.serial) wait_geq_spin(a.prog_full + (s - 1) * a.fs, (int)nprev);
          if (m == 0) wait_geq_opt(a.prog + (s - 1) * a.fs, 1, a.opt & 4);
          wait_geq_opt(a.prog_full + (s - 1) * a.fs, (int)(m + 1), a.opt & 4);
        }
        BCW_TRACE(s, m, 8);
        fence_proxy_async_global();
        if (m == 0) bulk_g2s(colb + bi * ldab, a.band + s * ldab, (unsigned)(ldab * 8), &full[bi]);
        if (L > 1) bulk_g2s(win, a.band + r0 * ldab, (unsigned)((L - 1) * ldab * 8), &full[bi]);
        if (c0fetch) continue;
        if (s > 0) wait_geq_opt(a.prog + (s - 1) * a.fs, (int)((m + 2 < nprev) ? m + 2 : nprev), a.opt & 4);
        BCW_TRACE(s, m, 9);
        fence_proxy_async_global();
        bulk_g2s(win + (L - 1) * ldab, a.band + (r0 + L - 1) * ldab, (unsigned)(ldab * 8), &lastb[bi]);
      }
    }
  }
  if (warp == NW + 1) {
    // ============================== STORE0 warp: column 0 (the chain) ==============================
    if (lane != 0) return;
    uint32_t cbase = 0, cnext = 0;   // CL: the consumer CTA's step count at the start of its current sweep
    for (uint32_t it = 0;; ++it) {
      const int bi = it & 1;
      const unsigned ph = (it >> 1) & 1u;
      if (a.opt & 1) mbar_spin(&col0b[bi], ph);
      else mbar_wait(&col0b[bi], ph);
      const int64_t s = info_s[bi];
      if (s < 0) return;
      const int m = info_m[bi];
      const int64_t r0 = s + 1 + (int64_t)m * b;
      BCW_TRACE(s, m, 3);
      if (has_cons) {
        if (m == 0) {
          cbase = cnext;
          cnext += (uint32_t)bc_steps(n, b, s + 1);
        }
        // column 0 of step m is column s+1 of the consumer's step 0 (m = 0) or the last column of its step m-1
        const int mt = m == 0 ? 0 : m - 1;
        if (bc_step_full(n, b, B, s + 1, mt)) {
          const uint32_t itc = cbase + (uint32_t)mt;
          const int bc = itc & 1;
          cl_wait_geq(&armed_ctr, (int)(itc + 1));
          const unsigned dst = m == 0 ? cl_mapa(colb + bc * ldab, crank + 1)
                                      : cl_mapa(sm + bc * wsz + (B - 1) * ldab, crank + 1);
          const unsigned bar = m == 0 ? cl_mapa(&full[bc], crank + 1) : cl_mapa(&lastb[bc], crank + 1);
          bulk_s2s_cl(dst, c0s + bi * ldab, (unsigned)(ldab * 8), bar);
        }
      }
      // CL: this step may have been fed by DSMEM before the producer's own global stores of the same columns
      // landed; never let an older global store overwrite ours (write-after-write on the band)
      if (has_prod) wait_geq_spin(a.prog_full + (s - 1) * a.fs, m + 1);
      if (CL || !(a.opt & 2)) {
        bulk_s2g(a.band + r0 * ldab, c0s + bi * ldab, (unsigned)(ldab * 8));
        bulk_commit();
        bulk_wait_all();
        fence_proxy_async_global();
      }
      BCW_TRACE(s, m, 4);
      st_release_s32(a.prog + s * a.fs, m + 1);
      BCW_TRACE(s, m, 5);
      mbar_arrive(&c0done[bi]);
    }
  }
  if (warp == NW + 2) {
    // ============================== STORE1 warp: columns 1..L-1 ==============================
    // frees the window buffer as soon as the bulk store has READ it; prog_full after the writes landed
    if (lane != 0) return;
    uint32_t cbase = 0, cnext = 0;
    for (uint32_t it = 0;; ++it) {
      const int bi = it & 1;
      const unsigned ph = (it >> 1) & 1u;
      mbar_wait(&colsb[bi], ph);
      const int64_t s = info_s[bi];
      if (s < 0) return;
      const int m = info_m[bi];
      const int64_t r0 = s + 1 + (int64_t)m * b;
      const int64_t r1 = (s + ((int64_t)m + 1) * b < n - 1) ? s + ((int64_t)m + 1) * b : n - 1;
      const int L = (int)(r1 - r0 + 1);
      double* win = sm + bi * wsz;
      int recv_need = 0;
      if (has_cons) {
        if (m == 0) {
          cbase = cnext;
          cnext += (uint32_t)bc_steps(n, b, s + 1);
        }
        // columns 1..L-1 of step m are the body of the consumer's step m
        if (bc_step_full(n, b, B, s + 1, m)) {
          const uint32_t itc = cbase + (uint32_t)m;
          const int bc = itc & 1;
          cl_wait_geq(&armed_ctr, (int)(itc + 1));
          bulk_s2s_cl(cl_mapa(sm + bc * wsz, crank + 1), win + ldab, (unsigned)((B - 1) * ldab * 8),
                      cl_mapa(&full[bc], crank + 1));
          recv_need = (int)(itc + 1);
        }
        const int mt = m == 0 ? 0 : m - 1;   // where STORE0 sent this step's column 0
        if (bc_step_full(n, b, B, s + 1, mt) && (int)(cbase + mt + 1) > recv_need) recv_need = (int)(cbase + mt + 1);
      }
      if (has_prod) {   // as in STORE0: the producer's global stores of these columns landed first
        const int np = (int)bc_steps(n, b, s - 1);
        wait_geq_spin(a.prog_full + (s - 1) * a.fs, m + 1);
        wait_geq_spin(a.prog + (s - 1) * a.fs, m + 2 < np ? m + 2 : np);
      }
      // full windows (not CL): the compute threads stored columns 1..L-1 to the band themselves; their stores are
      // ordered before prog_full by the CTA barrier + colsb arrival this warp synchronised with (release below)
      const bool direct = !CL && bc_step_full(n, b, B, s, m);
      if (L > 1 && !direct) {
        bulk_s2g(a.band + (r0 + 1) * ldab, win + ldab, (unsigned)((L - 1) * ldab * 8));
        bulk_commit();
        bulk_wait_read();
      }
      if (recv_need) cl_wait_geq(&recv_ctr, recv_need);   // the consumer holds both copies (they read this buffer)
      mbar_wait(&c0done[bi], ph);   // column 0's staging buffer was read too
      mbar_arrive(&empty[bi]);
      if (L > 1 && !direct) {
        bulk_wait_all();
        fence_proxy_async_global();
      }
      st_release_s32(a.prog_full + s * a.fs, m + 1);
      BCW_TRACE(s, m, 6);
    }
  }
  // ============================== compute warps ==============================
  const int r = (warp % RW) * 32 + lane, hg = warp / RW, j0 = hg * CPT;
  const bool c0path = tid < 2 * B;   // column group 0 = one thread per window row
  auto cbar = [] { asm volatile("bar.sync 1, %0;\n" ::"n"(NTH) : "memory"); };
  auto c0bar = [] { asm volatile("bar.sync 2, %0;\n" ::"n"(2 * B) : "memory"); };
  double tau = 0.0;
  int64_t off = 0;   // V2/tau2 offset of the current sweep (once per sweep: bc_offset divides)
  for (uint32_t it = 0;; ++it) {
    const int bi = it & 1;
    const unsigned ph = (it >> 1) & 1u;
    mbar_wait(&full[bi], ph);
    const int64_t s = info_s[bi];
    if (s < 0) {
      if (c0path) mbar_arrive(&col0b[bi]);   // wake the STORE warps so they can see the end
      if ((a.opt & 8) ? lane == 0 : tid == 0) mbar_arrive(&colsb[bi]);
      return;
    }
    const int64_t m = info_m[bi];
    if (tid == 0) BCW_TRACE(s, m, 0);
    const int64_t r0 = s + 1 + m * b;
    const int64_t r1 = (s + (m + 1) * b < n - 1) ? s + (m + 1) * b : n - 1;
    const int Lx = (int)(r1 - r0 + 1);
    const int64_t r2 = (r1 + b < n - 1) ? r1 + b : n - 1;
    const int L2x = (int)(r2 - r1);
    double* win = sm + bi * wsz;
    double* v = vb + (m & 1) * B;
    double* vn = vb + ((m & 1) ^ 1) * B;
    if (m == 0) {   // the reflector annihilating column s below its first subdiagonal (from colb)
      if (a.V2) off = bc_offset(n, b, s);
      const double* col = colb + bi * ldab + 1;
      double sig = 0.0;
      for (int i = 1 + lane; i < Lx; i += 32) sig = fma(col[i], col[i], sig);
      sig = warp_sum(sig);
      const House hh = make_house(col[0], sig);
      if (tid < B) v[tid] = tid == 0 ? 1.0 : (tid < Lx ? hh.scale * col[tid] : 0.0);
      if (tid == 0) __stcg(a.band + s * ldab + 1, hh.beta);   // e_s (the rest of column s is dead)
      tau = hh.tau;
      cbar();
    }
    // Full windows (L = L2 = B: every step but the last of a sweep) are compiled separately, so the
    // row/column predicates and the O/D split (warp-uniform for B % 32 == 0) fold at compile time.
    double tau_next = 0.0;
    auto step = [&](auto fullc) {
      constexpr bool FULL = decltype(fullc)::value;
      const int L = FULL ? B : Lx;
      const int L2 = FULL ? B : L2x;
      // a full window implies b == B, so the column stride ldab = 2B is a compile-time constant there
      const int lda1 = FULL ? 2 * B - 1 : lda1_rt;
      const int ldab = FULL ? 2 * B : ldab_rt;
      // the window through the extern __shared__ base (keeps the shared address space visible to the compiler
      // inside the lambda; in full windows the buffer stride is a constant too)
      double* const win = sm + bi * (FULL ? B * 2 * B : wsz);
    const bool active = r < L + L2;
    const bool isO = r >= L && active;
    const int lo_base = j0 * lda1 + r;
    const int hi_base = r * lda1 + j0;
    // the element (r, L-1) of rows r >= L-1 lives in the last column (in flight on lastb)
    const int jd = L - 1 - j0;
    const bool defer = r >= L - 1 && jd >= 0 && jd < CPT;
    double e[CPT];
    double acc0 = 0.0, acc1 = 0.0;
    // shared byte addresses of (r, j0) in the lower (column j0) and the mirrored (column r) layout
    const uint32_t a_lo = smem_u32(win) + 8u * (uint32_t)lo_base;
    const uint32_t a_hi = smem_u32(win) + 8u * (uint32_t)hi_base;
    const int rj = r - j0;   // element jj is in the stored lower triangle iff jj <= rj
    if constexpr (FULL) {
#pragma unroll
      for (int jj = 0; jj < CPT; ++jj) {
        const bool skip = defer && jj == CPT - 1;   // full window: only the last column can be deferred
        const uint32_t ad = jj <= rj ? a_lo + 8u * (uint32_t)(jj * lda1) : a_hi + 8u * (uint32_t)jj;
        e[jj] = skip ? 0.0 : lds_f64(ad);
      }
    } else {
#pragma unroll
      for (int jj = 0; jj < CPT; ++jj) {
        const int j = j0 + jj;
        const bool ok = j < L && !(defer && jj == jd);
        e[jj] = ok ? win[j <= r ? lo_base + jj * lda1 : hi_base + jj] : 0.0;
      }
    }
    const double2* v2 = reinterpret_cast<const double2*>(v + j0);
#pragma unroll
    for (int jj = 0; jj < CPT; jj += 2) {
      const double2 vv = v2[jj / 2];
      acc0 = fma(e[jj], vv.x, acc0);
      acc1 = fma(e[jj + 1], vv.y, acc1);
    }
    part[hg * 2 * B + r] = acc0 + acc1;
    cbar();   // (1) body partials of D v / O v
    if (tid == 0) BCW_TRACE(s, m, 10);
    if (c0path) {
      // ---------------- column-0 path: thread r = window row r ----------------
      double acc = 0.0;
#pragma unroll
      for (int q = 0; q < TPR; ++q) acc += part[q * 2 * B + r];
      double lastv = 0.0;   // element (r, L-1): the last window column, the predecessor's fresh column 0
      if (!CL && (a.opt & 32)) {
        // TRID_BC_OPT bit 32: these 2B threads (idle until the last column lands) poll the predecessor's counter and
        // load the column straight from L2 -- no LOAD-warp detection, bulk copy or mbarrier on the chain; they fill
        // the shared window column for the rest of the step and release it on lastb (2B arrivals)
        if (s > 0 && tid == 0) {
          const int64_t nprev = bc_steps(n, b, s - 1);
          wait_geq_opt(a.prog + (s - 1) * a.fs, (int)((m + 2 < nprev) ? m + 2 : nprev), a.opt & 4);
        }
        c0bar();
        const double* gl = a.band + (r0 + Lx - 1) * ldab;
        if (r < ldab) win[(Lx - 1) * ldab + r] = __ldcg(gl + r);
        if (r >= Lx - 1 && r - (Lx - 1) < ldab) lastv = __ldcg(gl + (r - (Lx - 1)));
        mbar_arrive(&lastb[bi]);
      } else {
        mbar_wait(&lastb[bi], ph);
        if (active && r >= L - 1) lastv = win[(L - 1) * lda1 + r];
      }
      if (tid == 0) BCW_TRACE(s, m, 11);
      if (CL && tid == 0 && info_f[bi]) cl_st_release(cl_mapa(&recv_ctr, crank - 1), (int)(it + 1));
      if (active && r >= L - 1) acc = fma(lastv, v[L - 1], acc);
      const double py = (r >= L) ? acc : tau * acc;   // p_r = tau (D v)_r  |  y_r = (O v)_r
      pyv[r] = py;
      const double vr = r < L ? v[r] : 0.0;
      const double raw = r < ldab ? win[r] : 0.0;        // column 0, row r0 + r
      double x = 0.0;
      if (isO) x = fma(-(tau * py), v[0], raw);         // right-updated O(r-L, 0)
      double tD = r < L ? py * vr : 0.0;
      double tO = (isO && r > L) ? x * x : 0.0;
      tD = warp_sum(tD);
      tO = warp_sum(tO);
      if (lane == 0) {
        red[warp] = tD;
        red[RW + warp] = tO;
      }
      if (r == L) red[2 * RW] = x;
      xs[r] = x;
      c0bar();
      double pv = 0.0, sg = 0.0;
#pragma unroll
      for (int w = 0; w < RW; ++w) {
        pv += red[w];
        sg += red[RW + w];
      }
      const double hp = 0.5 * tau * pv;
      double val = raw;
      if (r < L) {
        const double w0 = fma(-hp, v[0], pyv[0]);
        const double wr = fma(-hp, vr, py);
        val = fma(-wr, v[0], fma(-vr, w0, raw));
      } else if (isO) {
        val = 0.0;
        if (r == L) {
          const House h2 = make_house(red[2 * RW], sg);
          val = h2.beta;
          red[2 * RW + 1] = h2.beta;
          red[2 * RW + 2] = h2.tau;
          red[2 * RW + 3] = h2.scale;
        }
      }
      if (r < ldab) {
        c0s[bi * ldab + r] = val;
        if (!CL && (a.opt & 2)) a.band[r0 * ldab + r] = val;
      }
      fence_proxy_async_smem();
      mbar_arrive(&col0b[bi]);   // column 0 final -> STORE publishes it
      if (tid == 0) BCW_TRACE(s, m, 1);
    }
    if (defer) {
      mbar_wait(&lastb[bi], ph);
      const double el = win[(L - 1) * lda1 + r];
#pragma unroll
      for (int jj = 0; jj < CPT; ++jj)
        if (jj == jd) e[jj] = el;
    }
    cbar();   // (2) pyv, p^T v partials, x, the next reflector's scalars
    if (tid == 0) BCW_TRACE(s, m, 12);
    double hscale = 0.0;
    if (L2 > 0) {
      tau_next = red[2 * RW + 2];
      hscale = red[2 * RW + 3];
    }
    if (tau != 0.0) {
      double pv = 0.0;
#pragma unroll
      for (int w = 0; w < RW; ++w) pv += red[w];
      const double hp = 0.5 * tau * pv;
      if (isO) {
        const double ty = tau * pyv[r];
        const double2* v2u = reinterpret_cast<const double2*>(v + j0);
#pragma unroll
        for (int jj = 0; jj < CPT; jj += 2) {
          const double2 vj = v2u[jj / 2];
          e[jj] = fma(-ty, vj.x, e[jj]);
          e[jj + 1] = fma(-ty, vj.y, e[jj + 1]);
        }
      } else {
        const double vr = r < L ? v[r] : 0.0;
        const double wr = r < L ? fma(-hp, vr, pyv[r]) : 0.0;
        const double2* v2u = reinterpret_cast<const double2*>(v + j0);
        const double2* p2u = reinterpret_cast<const double2*>(pyv + j0);
#pragma unroll
        for (int jj = 0; jj < CPT; jj += 2) {
          const double2 vj = v2u[jj / 2], pj = p2u[jj / 2];
          const double wj0 = fma(-hp, vj.x, pj.x), wj1 = fma(-hp, vj.y, pj.y);
          e[jj] = fma(-wr, vj.x, fma(-vr, wj0, e[jj]));
          e[jj + 1] = fma(-wr, vj.y, fma(-vr, wj1, e[jj + 1]));
        }
      }
    }
    // D rows are final: write the lower triangle back (column 0 goes out through the staging buffer)
    // full windows (not CL): final values go straight from registers to the global band (coalesced along the
    // rows of a column); column 0 goes out through the staging buffer.  STORE1 then only releases prog_full
    // (after the CTA barrier, like a split-K semaphore), so no shared write-back and no bulk store sit between
    // this step's end and the next sweep's load of these columns.
    double* const gwin = a.band + r0 * ldab + lo_base;   // element (r, j0 + jj) at gwin[jj * lda1]
    if (FULL && !CL && !isO) {
#pragma unroll
      for (int jj = 0; jj < CPT; ++jj)
        if (jj <= rj && j0 + jj >= 1) gwin[jj * lda1] = e[jj];
    } else if (FULL && !isO) {
      // (column 0 is published from the staging buffer and never read back: a full window may write it)
#pragma unroll
      for (int jj = 0; jj < CPT; ++jj)
        if (jj <= rj) sts_f64(a_lo + 8u * (uint32_t)(jj * lda1), e[jj]);
    } else if (active && !isO) {
#pragma unroll
      for (int jj = 0; jj < CPT; ++jj) {
        const int j = j0 + jj;
        if (j >= 1 && j < L && j <= r) win[lo_base + jj * lda1] = e[jj];
      }
    }
    // next reflector vn (rows L..L+L2-1 of the window): vn_0 = 1, vn_i = scale * x_i
    const double vnr = isO ? (r == L ? 1.0 : hscale * xs[r]) : 0.0;
    if (L2 > 0 && tid < B) vn[tid] = tid < L2 ? (tid == 0 ? 1.0 : hscale * xs[L + tid]) : 0.0;
    const bool zwarp = L2 > 0 && tau_next != 0.0 && L > 1 && (warp % RW) * 32 + 31 >= L;   // warp holds O rows
    if (zwarp) {
      // z_j = sum_i vn_i O(i, j) over this warp's 32 rows for the group's CPT columns: transposed butterfly
      double c[CPT];
#pragma unroll
      for (int jj = 0; jj < CPT; ++jj) c[jj] = vnr * e[jj];
#pragma unroll
      for (int o = 16, K = CPT; K > 1; o >>= 1, K >>= 1) {
        const bool up = (lane & o) != 0;
#pragma unroll
        for (int i = 0; i < K / 2; ++i) {
          const double send = up ? c[i] : c[i + K / 2];
          const double keep = up ? c[i + K / 2] : c[i];
          c[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
        }
      }
      constexpr int SH = CPT == 16 ? 1 : (CPT == 8 ? 2 : 3);   // lanes per column after the butterfly
      double f = c[0];
#pragma unroll
      for (int o = (1 << SH) >> 1; o >= 1; o >>= 1) f += __shfl_xor_sync(0xffffffffu, f, o);
      if ((lane & ((1 << SH) - 1)) == 0) zp[(warp % RW) * B + j0 + (lane >> SH)] = f;
    } else if (lane < CPT) {
      zp[(warp % RW) * B + j0 + lane] = 0.0;
    }
    if (FULL && RW == 4 && (a.opt & 16)) {
      // (3') full windows: z_j of column group hg needs only the partials of its own two O-row warps (rows
      // L..L+L2-1), so those 64 threads meet on the group's named barrier and the D-row warps go on (TRID_BC_OPT
      // bit 16, with bit 8)
      if (isO) asm volatile("bar.sync %0, %1;\n" ::"r"(3 + hg), "n"(2 * 32) : "memory");
    } else {
      cbar();   // (3) z partials, vn
    }
    if (tid == 0) BCW_TRACE(s, m, 13);
    if (FULL && isO) {
      // full window: the O rows are the last two row-warps of the group (the others' partials are zero, and
      // 0 + x == x, so this is the generic sum below bit for bit)
      const double tv = tau_next * vnr;
      const double2* za = reinterpret_cast<const double2*>(zp + (RW - 2) * B + j0);
      const double2* zb = reinterpret_cast<const double2*>(zp + (RW - 1) * B + j0);
#pragma unroll
      for (int jj = 0; jj < CPT; jj += 2) {
        const double2 x = za[jj / 2], y = zb[jj / 2];
        const double z0 = x.x + y.x, z1 = x.y + y.y;
        const double o0 = tau_next != 0.0 ? fma(-tv, z0, e[jj]) : e[jj];
        const double o1 = tau_next != 0.0 ? fma(-tv, z1, e[jj + 1]) : e[jj + 1];
        if constexpr (!CL) {
          if (j0 + jj >= 1) gwin[jj * lda1] = o0;
          gwin[(jj + 1) * lda1] = o1;
        } else {
          if (j0 + jj >= 1) sts_f64(a_lo + 8u * (uint32_t)(jj * lda1), o0);
          sts_f64(a_lo + 8u * (uint32_t)((jj + 1) * lda1), o1);
        }
      }
    } else if (isO) {
      const double tv = tau_next * vnr;
#pragma unroll
      for (int jj = 0; jj < CPT; ++jj) {
        const int j = j0 + jj;
        if (j >= 1 && j < L) {
          double z = 0.0;
#pragma unroll
          for (int w = 0; w < RW; ++w) z += zp[w * B + j];
          win[lo_base + jj * lda1] = (L2 > 0 && tau_next != 0.0) ? fma(-tv, z, e[jj]) : e[jj];
        }
      }
    }
    // the window goes out through a bulk store only for CL or ragged windows; full windows were stored from
    // registers (a proxy fence here would also wait for those global stores)
    if (CL || !FULL) fence_proxy_async_smem();
    if (tid == 0) BCW_TRACE(s, m, 14);
    if (a.V2) {
      double* vd = a.V2 + (off + m) * a.vs;
      for (int i = tid; i < a.vs; i += NTH) vd[i] = i < L ? v[i] : 0.0;
      if (tid == 0) a.tau2[off + m] = tau;
    }
    if (a.opt & 8) {
      // per-warp hand-off (TRID_BC_OPT bit 8): each warp releases its own stores of this step to STORE1 (colsb
      // counts the NW compute warps), so warps that finished early start the next step's body matvec while the
      // O-row warps finish the left application; the next step's first CTA barrier still orders every shared
      // scratch reuse
      __syncwarp();
      if (lane == 0) mbar_arrive(&colsb[bi]);
      if (tid == 0) BCW_TRACE(s, m, 2);
    } else {
      cbar();   // (4) columns 1..L-1 final
      if (tid == 0) {
        BCW_TRACE(s, m, 2);
        mbar_arrive(&colsb[bi]);   // -> STORE1
      }
    }
    };
    if (Lx == B && L2x == B) step(std::true_type{});
    else step(std::false_type{});
    tau = tau_next;
  }
}

template <int B, int NTH, bool CL>
__global__ void __launch_bounds__(NTH + 96, 1) bc_v6_kernel(BcArgs a) {
  bc_v6_body<B, NTH, CL>(a);
  if constexpr (CL) cl_sync_all();   // no CTA leaves while a peer may still copy into / signal its shared memory
}


// ---- wide-band chase (64 < b <= 256) ----------------------------------------------------------------------------------
// The b <= 64 register-resident design does not scale: at b = 128 a step window ([D; O], 2b rows x b columns) is
// 197 KB even when only its stored part is kept, at b = 256 it is 788 KB.  Here a step's window lives in shared
// memory as a TRAPEZOID: window column j holds only its rows j .. 2b-1 (the lower triangle of D and the whole
// bulge block O), 2b - j doubles rounded up to even, packed one after the other (16-byte aligned columns, loaded and
// stored with 16-byte cp.async / st.global.cg by all threads).  For b <= 128 one CTA holds the whole trapezoid
// (197 KB at b = 128); beyond, the window is split by columns over a cluster of CS = 4 CTAs (balanced by stored size,
// <= 197 KB each) that cooperate on one sweep through DSMEM:
//   1. every CTA forms the partial matvec [D; O] v over its columns for all 2b rows (the lower part of D row-wise,
//      the mirrored upper part as a column dot, both from its own columns), writes it to shared memory;
//   2. cluster barrier; every CTA sums the CS partials in rank order (DSMEM loads): identical p = tau D v, y = O v;
//   3. rank-2 update of D and right update of O on its own columns;
//   4. the CTA owning window column 0 forms the next reflector from O(:, 0) and broadcasts it (DSMEM stores);
//      cluster barrier;
//   5. z_j = vn^T O(:, j) and the left update on its own columns; store back; cluster barrier; rank 0 publishes.
// Sweeps are claimed from the atomic ticket and pipelined at lag 2 on per-sweep counters (R9) as in bc_v6.  All sums
// run in a fixed order: bitwise reproducible, independent of scheduling (serial-vs-parallel test).
constexpr int BW_NT = 512;
struct BwPart {
  int c[5];   // window columns [c[q], c[q+1]) belong to cluster rank q
};

// offset (doubles) of window column j in the packed trapezoid, columns of 2b - j rows rounded up to even
__host__ __device__ __forceinline__ int bw_coff(int b, int j) { return 2 * b * j - j * (j - 1) / 2 + j / 2; }

// DSMEM access to the same shared variable in cluster rank `rank` (shared::cluster addresses from mapa); CS == 1:
// plain shared memory
template <int CS>
__device__ __forceinline__ double bw_ld(const double* p, unsigned rank) {
  if constexpr (CS == 1) {
    return *p;
  } else {
    double v;
    asm volatile("ld.shared::cluster.f64 %0, [%1];\n" : "=d"(v) : "r"(cl_mapa(p, rank)) : "memory");
    return v;
  }
}
template <int CS>
__device__ __forceinline__ void bw_st(double* p, unsigned rank, double v) {
  if constexpr (CS == 1) *p = v;
  else asm volatile("st.shared::cluster.f64 [%0], %1;\n" ::"r"(cl_mapa(p, rank)), "d"(v) : "memory");
}
template <int CS>
__device__ __forceinline__ void bw_csync() {
  if constexpr (CS == 1) __syncthreads();
  else cl_sync_all();
}

template <int CS>
__global__ void __launch_bounds__(BW_NT, 1) bc_wide_kernel(BcArgs a, BwPart part) {
  extern __shared__ __align__(16) double sm[];
  constexpr int NW = BW_NT / 32;
  const int b = a.b, ldab = a.ldab, tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t n = a.n;
  const unsigned q = CS > 1 ? cl_rank() : 0u;
  const int cbeg = part.c[q], cend = part.c[q + 1];
  const int H2 = 2 * b;
  // shared layout: vb[2][b] | prt[2][2b] | pf[2b] | w[b] | colv[b] | scal[16] | sweep[2] | cofs[b] (ints) | window
  double* vb = sm;
  double* prt = vb + 2 * b;   // [0, 2b): this CTA's partial matvec; [2b, 4b): the second half-row partial
  double* pf = prt + 2 * H2;
  double* wv = pf + H2;
  double* colv = wv + b;
  double* scal = colv + b;   // 0 pv, 1..3 reflector of column s (beta, tau, scale), 4..6 next reflector
  double* swp = scal + 16;   // the claimed sweep (as a double-sized slot)
  int* cofs = reinterpret_cast<int*>(swp + 2);
  double* win = sm + ((10 * b + 18 + (b + 1) / 2 + 1) & ~1);   // 16-byte aligned, past cofs
  // window element (i, j), i >= j, of my column j: win[cofs[j] + i]
  for (int j = tid; j < b; j += BW_NT) cofs[j] = (j >= cbeg && j < cend) ? bw_coff(b, j) - bw_coff(b, cbeg) - j : 0;
  __syncthreads();
  // threads per window row in the matvec (b <= 128: two, each over half of my columns)
  const int tpr = BW_NT / H2 >= 2 ? 2 : 1;
  const int jmid = cbeg + (cend - cbeg + 1) / 2;
  for (;;) {
    if (q == 0 && tid == 0) {
      const double s0 = (double)atomicAdd(a.ticket, 1u);   // exact (< 2^53)
      for (unsigned r = 0; r < CS; ++r) bw_st<CS>(swp, r, s0);
    }
    bw_csync<CS>();
    const int64_t s = (int64_t)swp[0];
    bw_csync<CS>();
    if (s > n - 3) return;
    const int64_t nst = bc_steps(n, b, s);
    const int64_t off = bc_offset(n, b, s);
    const int64_t nprev = s > 0 ? bc_steps(n, b, s - 1) : 0;
    double tau = 0.0;
    bool pref = false;   // this warp's body columns of the current step were requested during the previous one
    for (int64_t m = 0; m < nst; ++m) {
      double* v = vb + (m & 1) * b;
      double* vn = vb + ((m & 1) ^ 1) * b;
      const int64_t r0 = s + 1 + m * b;
      const int64_t r1 = (s + (m + 1) * b < n - 1) ? s + (m + 1) * b : n - 1;
      const int L = (int)(r1 - r0 + 1);
      const int64_t r2 = (r1 + b < n - 1) ? r1 + b : n - 1;
      const int L2 = (int)(r2 - r1);
      const int H = L + L2;
      const int je = cend < L ? cend : L;   // my window columns [cbeg, je)
      const double* gw = a.band + r0 * ldab;   // window column j at gw + j*ldab (rows j.. at offsets 0..)
      // ---- dependencies on sweep s-1 (R9, lag 2, refined by column ownership as in bc_v6): window columns
      // 0 .. L-2 were last written by its step m (prog_full >= m+1), the last column is column 0 of its step m+1
      // (published early, prog >= m+2).  Serial mode: all of its steps.  The body loads while the last column is
      // still being produced.
      const int need_full = (int)(a.serial ? nprev : m + 1);
      const int need_c0 = (int)((m + 2 < nprev && !a.serial) ? m + 2 : nprev);
      // ---- load my window columns, one warp per column (rows j .. H-1: offsets 0 .. H-1-j); the last one after
      // its producer published it.  A warp whose columns were prefetched at the end of the previous step (pref,
      // below) skips this; otherwise its lane 0 waits for the dependency (each warp orders its own loads).
      auto load_col_at = [&](int j, const double* gwx, int Hx) {
        const int len = Hx - j, len2 = len >> 1;
        double* dst = win + cofs[j] + j;
        const double* src = gwx + (int64_t)j * ldab;
        for (int i = lane; i < len2; i += 32)
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(smem_u32(dst + 2 * i)), "l"(src + 2 * i)
                       : "memory");
        // the odd tail element asynchronously too (round 2: a synchronous L2 load here stalled the warp once per
        // odd-length column, about half of them)
        if ((len & 1) && lane == 0)
          asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(smem_u32(dst + len - 1)), "l"(src + len - 1)
                       : "memory");
      };
      auto load_col = [&](int j) { load_col_at(j, gw, H); };
      if (!pref) {
        if (s > 0) {
          if (lane == 0) wait_geq(a.prog_full + (s - 1) * a.fs, need_full);
          __syncwarp();
        }
        for (int j = cbeg + warp; j < je && j < L - 1; j += NW) load_col(j);
      }
      pref = false;
      asm volatile("cp.async.commit_group;\n" ::: "memory");
      if (q == 0 && tid == 0) BCW_TRACE(s, m, 0);
      if (a.opt & 64) bw_csync<CS>();   // debug (TRID_BC_OPT): extra cluster barriers
      const bool own_last = je == L && L - 1 >= cbeg;   // this CTA holds the window's last column
      // ---- step 0: the reflector annihilating column s below its first subdiagonal (every CTA, same bits)
      if (m == 0) {
        for (int i = tid; i < L; i += BW_NT) colv[i] = __ldcg(a.band + s * ldab + 1 + i);
        __syncthreads();
        if (warp == 0) {
          double sg = 0.0;
          for (int i = 1 + lane; i < L; i += 32) sg = fma(colv[i], colv[i], sg);
          sg = warp_sum(sg);
          if (lane == 0) {
            const House h = make_house(colv[0], sg);
            scal[1] = h.beta;
            scal[2] = h.tau;
            scal[3] = h.scale;
          }
        }
        __syncthreads();
        for (int i = tid; i < b; i += BW_NT) v[i] = i == 0 ? 1.0 : (i < L ? scal[3] * colv[i] : 0.0);
        tau = scal[2];
      }
      asm volatile("cp.async.wait_group 0;\n" ::: "memory");   // the body columns
      __syncthreads();
      if (q == 0 && tid == 0) BCW_TRACE(s, m, 1);
      if (a.opt & 128) bw_csync<CS>();
      // ---- 1. partial matvec [D; O] v over my BODY columns (all but the window's last, which sweep s-1 may still
      //      be producing), all H rows; the last column's terms are added once it arrives
      if (tau != 0.0) {
        if constexpr (CS == 1) {
          // one CTA holds every column: thread (i, h) forms row i of [D; O] v over half h of the body columns in one
          // pass, the upper part of D from its mirror in column i (D(j, i), j > i, incl. the last column's term,
          // which column i holds), four accumulators (round 2: the former row pass + per-column warp dots took
          // 7.2 us of a 19.5 us step at b = 128)
          const int i = tid % H2, h = tid / H2;   // tpr == 2 (b <= 128, 512 threads)
          double a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0;
          if (i < H) {
            const int jend = i < L - 1 ? L : L - 1;
            const int jlo = h ? jmid : 0;
            const int jhi = h ? jend : (jmid < jend ? jmid : jend);
            const int ci = i < L ? cofs[i] : 0;
            auto el = [&](int j) { return win[j <= i ? cofs[j] + i : ci + j]; };
            int j = jlo;
            for (; j + 4 <= jhi; j += 4) {
              const double e0 = el(j), e1 = el(j + 1), e2 = el(j + 2), e3 = el(j + 3);
              a0 = fma(e0, v[j], a0);
              a1 = fma(e1, v[j + 1], a1);
              a2 = fma(e2, v[j + 2], a2);
              a3 = fma(e3, v[j + 3], a3);
            }
            for (; j < jhi; ++j) a0 = fma(el(j), v[j], a0);
          }
          if (h < 2) prt[h * H2 + i] = (a0 + a1) + (a2 + a3);
          __syncthreads();
          for (int r = tid; r < H2; r += BW_NT) prt[r] += prt[H2 + r];
          // (the barrier after the last column's load orders these sums before their last-column terms)
        } else {
          {
            const int i = tid % H2, h = tid / H2;   // row i, half h (tpr == 2) of my columns
            if (h < tpr) {
              double acc = 0.0;
              if (i < H) {
                const int jlo = tpr == 2 ? (h ? jmid : cbeg) : cbeg;
                int jhi = tpr == 2 ? (h ? je : (jmid < je ? jmid : je)) : je;
                if (jhi > i + 1) jhi = i + 1;   // lower part of D (and all of O): columns j <= i
                if (jhi > L - 1) jhi = L - 1;   // body only
                for (int j = jlo; j < jhi; ++j) acc = fma(win[cofs[j] + i], v[j], acc);
              }
              prt[h * H2 + i] = acc;
            }
          }
          __syncthreads();
          if (tpr == 2)
            for (int i = tid; i < H2; i += BW_NT) prt[i] += prt[H2 + i];
          __syncthreads();
          // mirrored upper part of D for my columns c: sum_{j > c, j < L} D(j, c) v_j (a column dot, one warp)
          for (int c = cbeg + warp; c < je; c += NW) {
            const double* col = win + cofs[c];
            double acc = 0.0;
            for (int j = c + 1 + lane; j < L; j += 32) acc = fma(col[j], v[j], acc);
            acc = warp_sum(acc);
            if (lane == 0) prt[c] += acc;
          }
        }
      }
      if (q == 0 && tid == 0) BCW_TRACE(s, m, 9);   // (body matvec done in thread 0's warp)
      // ---- the last column = column 0 of sweep s-1's step m+1: wait for its early publication, load, add its terms
      //      D(L-1, L-1) v_{L-1} and O(:, L-1) v_{L-1} (fixed order: after the body and the mirror)
      if (s > 0 && need_c0 > need_full) {
        if (tid == 0) wait_geq(a.prog + (s - 1) * a.fs, need_c0);
        __syncthreads();
      }
      if (q == 0 && tid == 0) BCW_TRACE(s, m, 2);
      if (own_last && warp == (L - 1 - cbeg) % NW) load_col(L - 1);
      asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;\n" ::: "memory");
      __syncthreads();
      if (tau != 0.0) {
        if (own_last) {
          const double vl = v[L - 1];
          const double* cl = win + cofs[L - 1];
          for (int i = L - 1 + tid; i < H; i += BW_NT) prt[i] = fma(cl[i], vl, prt[i]);
        }
        bw_csync<CS>();   // (1) partials of every CTA complete
        if (q == 0 && tid == 0) BCW_TRACE(s, m, 3);
        // ---- 2. p = tau D v, y = O v: the CS partials summed in rank order
        for (int i = tid; i < H; i += BW_NT) {
          double acc = 0.0;
#pragma unroll
          for (unsigned r = 0; r < CS; ++r) acc += bw_ld<CS>(prt + i, r);
          pf[i] = i < L ? tau * acc : acc;
        }
      }
      __syncthreads();
      // ---- p^T v (warp 0) and 3. the next reflector from x = O(:, 0) - tau y v_0 (O(:, 0) after the right update;
      //      window column 0 belongs to rank 0; warp 1 at the same time), before any column is updated
      //      (round 2: one barrier for both reductions instead of three)
      if (tau != 0.0 && warp == 0) {
        double pv = 0.0;
        for (int i = lane; i < L; i += 32) pv = fma(pf[i], v[i], pv);
        pv = warp_sum(pv);
        if (lane == 0) scal[0] = pv;
      }
      const double* c0 = win + cofs[0] + L;
      const double tv0 = tau * v[0];
      auto xo = [&](int i) { return tau != 0.0 ? fma(-pf[L + i], tv0, c0[i]) : c0[i]; };
      if (L2 > 0 && q == 0 && warp == 1) {
        double sg = 0.0;
        for (int i = 1 + lane; i < L2; i += 32) {
          const double x = xo(i);
          sg = fma(x, x, sg);
        }
        sg = warp_sum(sg);
        if (lane == 0) {
          const House h = make_house(xo(0), sg);
          for (unsigned r = 0; r < CS; ++r) {
            bw_st<CS>(scal + 4, r, h.beta);
            bw_st<CS>(scal + 5, r, h.tau);
            bw_st<CS>(scal + 6, r, h.scale);
          }
        }
      }
      __syncthreads();
      if (a.opt & 512) bw_csync<CS>();
      if (tau != 0.0) {
        const double hp = 0.5 * tau * scal[0];
        for (int i = tid; i < L; i += BW_NT) wv[i] = fma(-hp, v[i], pf[i]);
      }
      double taun = 0.0;
      if (L2 > 0) {
        if (q == 0) {
          const double hs = scal[6];
          for (int i = tid; i < b; i += BW_NT) {
            const double x = i < L2 ? (i == 0 ? 1.0 : hs * xo(i)) : 0.0;
#pragma unroll
            for (unsigned r = 0; r < CS; ++r) bw_st<CS>(vn + i, r, x);
          }
        }
        bw_csync<CS>();   // (2) w, vn and its scalars everywhere
        if (q == 0 && tid == 0) BCW_TRACE(s, m, 4);
        taun = scal[5];
      } else {
        __syncthreads();   // w
      }
      // ---- 4. one fused pass per column (one warp per column): D -= v w^T + w v^T (lower); O -= tau y v^T, then
      //      O(:, j) -= taun vn (vn^T O(:, j)) for j >= 1, O(:, 0) = beta e1.  Window column 0 (rank 0, warp 0,
      //      first) is final right after its pass: stored and published at once (prog)
      // Round 2: the step vectors are held in registers by absolute window row (lane + 32 k), and every column but
      // column 0 goes from its fused pass straight to the band (no shared write-back, no separate store pass): the
      // pass was bound by shared-memory traffic (5 accesses per element, then a 6th to store; trace: fused pass
      // 7.4 us + store 4.1 us of a 25 us step at b = 128).  Same expressions in the same order (bitwise).
      constexpr int KR = CS == 1 ? 4 : 8;   // rows per lane: L, L2 <= b <= 128 (CS = 1) or <= 256
      double vD[KR], wD[KR], pO[KR], vnO[KR];
#pragma unroll
      for (int k = 0; k < KR; ++k) {
        const int i = lane + 32 * k;
        vD[k] = i < L ? v[i] : 0.0;
        wD[k] = (tau != 0.0 && i < L) ? wv[i] : 0.0;
        pO[k] = (tau != 0.0 && i < L2) ? pf[L + i] : 0.0;
        vnO[k] = (L2 > 0 && i < L2) ? vn[i] : 0.0;
      }
      for (int j = cbeg + warp; j < je; j += NW) {
        double* col = win + cofs[j];
        if (j == 0 && L2 > 0) {
          // window column 0: final in shared memory, stored and published at once (the chain's early hand-off)
          if (tau != 0.0) {
            const double vj = v[j], wj = wv[j];
            for (int i = j + lane; i < L; i += 32) col[i] = fma(-wv[i], vj, fma(-v[i], wj, col[i]));
          }
#pragma unroll
          for (int k = 0; k < KR; ++k) {
            const int i = lane + 32 * k;
            if (i < L2) col[L + i] = i == 0 ? scal[4] : 0.0;
          }
          __syncwarp();
          double* dst0 = a.band + r0 * ldab;
          for (int i = lane; i < H; i += 32) __stcg(dst0 + i, col[i]);
          __syncwarp();   // the warp's stores of column 0 are ordered before lane 0's release
          if (lane == 0) st_release_s32(a.prog + s * a.fs, (int)(m + 1));
          if (q == 0 && tid == 0) BCW_TRACE(s, m, 8);
          continue;
        }
        double* dst = a.band + (r0 + j) * ldab - j;   // window element (i, j), i >= j, at dst[i]
        if (tau != 0.0) {
          const double vj = v[j], wj = wv[j];
#pragma unroll
          for (int k = 0; k < KR; ++k) {
            const int i = lane + 32 * k;
            if (i >= j && i < L) __stcg(dst + i, fma(-wD[k], vj, fma(-vD[k], wj, col[i])));
          }
        } else {
#pragma unroll
          for (int k = 0; k < KR; ++k) {
            const int i = lane + 32 * k;
            if (i >= j && i < L) __stcg(dst + i, col[i]);
          }
        }
        if (L2 > 0) {
          const double* oc = col + L;
          const double tvj = tau * v[j];
          double o[KR];
          double z = 0.0;
#pragma unroll
          for (int k = 0; k < KR; ++k) {
            const int i = lane + 32 * k;
            o[k] = 0.0;
            if (i < L2) {
              o[k] = tau != 0.0 ? fma(-pO[k], tvj, oc[i]) : oc[i];
              z = fma(vnO[k], o[k], z);
            }
          }
          z = warp_sum(z);
          const double tz = taun * z;
#pragma unroll
          for (int k = 0; k < KR; ++k) {
            const int i = lane + 32 * k;
            if (i < L2) __stcg(dst + L + i, taun != 0.0 ? fma(-tz, vnO[k], o[k]) : o[k]);
          }
        }
      }
      // prefetch: this warp's columns are final in the band and its shared slots dead, so if the predecessor has
      // already completed step m+1 (non-blocking check) the same columns of step m+1 are requested now and the
      // load overlaps the rest of this step (round 2: the synchronous window load was 2.8 us of a 17 us step)
      if (m + 1 < nst) {
        const int need_n = (int)(a.serial ? nprev : m + 2);
        int ready = 1;
        if (s > 0 && lane == 0) ready = ld_acquire_s32(a.prog_full + (s - 1) * a.fs) >= need_n;
        ready = __shfl_sync(0xffffffffu, ready, 0);
        if (ready) {
          const int64_t r0n = r0 + b;
          const int64_t r1n = (s + (m + 2) * b < n - 1) ? s + (m + 2) * b : n - 1;
          const int Ln = (int)(r1n - r0n + 1);
          const int64_t r2n = (r1n + b < n - 1) ? r1n + b : n - 1;
          const int Hn = Ln + (int)(r2n - r1n);
          const int jen = cend < Ln ? cend : Ln;
          const double* gwn = a.band + r0n * ldab;
          for (int j = cbeg + warp; j < jen && j < Ln - 1; j += NW) load_col_at(j, gwn, Hn);
          pref = true;
        }
      }
      if (a.opt & 256) bw_csync<CS>();
      if (q == 0 && tid == 0) BCW_TRACE(s, m, 5);
      if (q == 0 && a.V2) {
        double* vd = a.V2 + (off + m) * a.vs;
        for (int i = tid; i < a.vs; i += BW_NT) vd[i] = i < L ? v[i] : 0.0;
        if (tid == 0) a.tau2[off + m] = tau;
      }
      bw_csync<CS>();   // (3) every CTA's stores of this step issued (ordered before the release below)
      if (q == 0 && tid == 0) BCW_TRACE(s, m, 6);
      if (q == 0 && tid == 0) {
        // e_s (the rest of column s is dead): written only now, when every CTA of the cluster has read column s
        if (m == 0) __stcg(a.band + s * ldab + 1, scal[1]);
        if (L2 == 0) st_release_s32(a.prog + s * a.fs, (int)(m + 1));   // no early column-0 publication this step
        st_release_s32(a.prog_full + s * a.fs, (int)(m + 1));
        BCW_TRACE(s, m, 7);
      }
      tau = taun;
    }
  }
}

size_t bc_work_bytes(int64_t n, int b) {
  const size_t band = sizeof(double) * (size_t)n * bc_ldab(n, b);
  const size_t flags = sizeof(int) * (size_t)(2 * n + 128) * BC_FLAG_STRIDE;
  const size_t trace = sizeof(long long) * 2 * 1024 * 16;
  return ((band + 255) / 256) * 256 + ((flags + 255) / 256) * 256 + trace;
}

cudaError_t bulge_chase(int64_t n, int b, const double* A, int64_t lda, double* d, double* e, double* V2,
                        double* tau2, void* work, cudaStream_t st) {
  return bulge_chase_cs(n, b, A, lda + 1, d, e, V2, tau2, work, st);
}

cudaError_t bulge_chase_cs(int64_t n, int b, const double* X, int64_t cs, double* d, double* e, double* V2,
                           double* tau2, void* work, cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  const int beff = (int)((b < n - 1) ? b : (n - 1 > 0 ? n - 1 : 1));
  const int ldab = bc_ldab(n, beff);
  double* band = (double*)work;
  const size_t band_bytes = ((sizeof(double) * (size_t)n * ldab + 255) / 256) * 256;
  // per-sweep counters: one 32-byte sector apart (no two sweeps' counters share a sector: packed, the producers'
  // releases and the consumers' polls of neighbouring sweeps contended on the same lines); TRID_BC_FS = stride in
  // ints (A/B); the region is sized for the widest layout (BC_FLAG_STRIDE)
  const char* fse = getenv("TRID_BC_FS");
  int fsv = fse ? atoi(fse) : 8;
  if (fsv < 1 || fsv > BC_FLAG_STRIDE) fsv = 8;
  const int fs = fsv;   // round 2: the wide chase too (it used packed counters)
  int* prog = (int*)((char*)work + band_bytes);
  int* prog_full = prog + (n + 32) * fs;
  unsigned* ticket = (unsigned*)(prog_full + (n + 32) * fs);
  const size_t flags_bytes = ((sizeof(int) * (size_t)(2 * n + 128) * BC_FLAG_STRIDE + 255) / 256) * 256;
  long long* trace = (long long*)((char*)work + band_bytes + flags_bytes);
  const char* tr = getenv("TRID_BC_TRACE");
  {
    int64_t total = n * (int64_t)ldab;
    int blocks = (int)((total + 255) / 256);
    if (blocks > 32 * num_sms()) blocks = 32 * num_sms();
    band_pack_kernel<<<blocks, 256, 0, st>>>(n, beff, ldab, X, cs, band);
    count_launches(1);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) return err;
  }
  if (beff >= 2 && n >= 3) {
    cudaError_t err = cudaMemsetAsync(prog, 0, sizeof(int) * (size_t)(2 * n + 128) * fs, st);
    if (err != cudaSuccess) return err;
    BcArgs a;
    // beff = min(b, n-1) gives the same step geometry as b (for b >= n-1 every sweep is one step on
    // rows s+1..n-1); V2 keeps the caller's stride b (header contract).
    a.n = n; a.b = beff; a.ldab = ldab; a.vs = b; a.band = band; a.V2 = V2; a.tau2 = tau2; a.prog = prog;
    a.prog_full = prog_full;
    a.fs = fs;
    {
      const char* oe = getenv("TRID_BC_OPT");
      a.opt = oe ? atoi(oe) : (8 | 16);   // default: per-warp step hand-off + per-group O barrier (measured -2.7% at n = 32768)
    }
    a.ticket = ticket;
    a.trace = tr ? trace : nullptr;
    a.trace_sweep = tr ? atoll(tr) : -1;
    // TRID_BC_SERIAL=1 (debug/tests): ONE CTA, and a sweep starts only after its predecessor stored every step:
    // the sweep-major order of the oracle (O2b), run by the same kernel.  Its output must equal the pipelined
    // chase's bit for bit (R9: lag 2 reads exactly what sweep-major order reads).
    const char* se = getenv("TRID_BC_SERIAL");
    const bool serial = se && se[0] == '1';
    a.serial = serial ? 1 : 0;
    const int64_t max_grid = serial ? 1 : (n - 2);
    int occ = 1;
    if (beff <= 64) {
      // bc_v6_kernel (warp-specialized, short column-0 path, 1 CTA/SM).  TRID_BC_FORCE=7 (A/B, tests): the same
      // kernel in CTA clusters with DSMEM forwarding between consecutive sweeps (measured slower).
      const int B = beff <= 32 ? 32 : 64;
      const char* force = getenv("TRID_BC_FORCE");
      const bool cluster = force && force[0] == '7' && !serial;
      const int nth = B == 32 ? 256 : 512;
      const size_t smem = sizeof(double) * (2 * (size_t)B * ldab + 4 * (size_t)ldab + 2 * B + 2 * B + B + 16 +
                                            (size_t)(nth / (2 * B)) * 2 * B + 2 * B + (2 * B / 32) * B + 8);
      const void* fn6 = B == 32 ? (const void*)bc_v6_kernel<32, 256, false> : (const void*)bc_v6_kernel<64, 512, false>;
      const void* fn7 = B == 32 ? (const void*)bc_v6_kernel<32, 256, true> : (const void*)bc_v6_kernel<64, 512, true>;
      bool launched = false;
      if (cluster) {
        // clusters of C (env TRID_BC_CLUSTER, default 2) sized to the co-resident cluster count
        const char* ce = getenv("TRID_BC_CLUSTER");
        const int C = ce ? atoi(ce) : 2;
        cudaFuncSetAttribute(fn7, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (C > 8) cudaFuncSetAttribute(fn7, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        cudaLaunchConfig_t cfg = {};
        cfg.blockDim = dim3((unsigned)(nth + 96));
        cfg.dynamicSmemBytes = smem;
        cfg.stream = st;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = (unsigned)C;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        cfg.gridDim = dim3((unsigned)(C * 40));
        int nc = 0;
        if (C >= 2 && cudaOccupancyMaxActiveClusters(&nc, fn7, &cfg) == cudaSuccess && nc >= 1) {
          int64_t ncl = nc;
          const int64_t need = (n - 2 + C - 1) / C;   // clusters with at least one sweep
          if (ncl > need) ncl = need;
          cfg.gridDim = dim3((unsigned)(ncl * C));
          cudaError_t le = B == 32 ? cudaLaunchKernelEx(&cfg, bc_v6_kernel<32, 256, true>, a)
                                   : cudaLaunchKernelEx(&cfg, bc_v6_kernel<64, 512, true>, a);
          if (le != cudaSuccess) return le;
          launched = true;
        } else {
          (void)cudaGetLastError();
        }
      }
      if (!launched) {
        cudaFuncSetAttribute(fn6, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        int64_t grid = num_sms();
        if (grid > max_grid) grid = max_grid;
        if (B == 32) bc_v6_kernel<32, 256, false><<<(unsigned)grid, 256 + 96, smem, st>>>(a);
        else bc_v6_kernel<64, 512, false><<<(unsigned)grid, 512 + 96, smem, st>>>(a);
      }
    } else {
      // 64 < b <= 256: bc_wide_kernel, a cluster of CS CTAs per sweep
      // cluster split: one CTA per sweep for b <= 128 (the whole trapezoid fits), 4 beyond.  Measured at n = 32768,
      // b = 128 with the early column-0 hand-off: CS = 1 994 ms, CS = 2 1092-1165 ms (the cluster barriers of a
      // step cost more than the halved step work saves), profiles/r02_bc_wide_cluster_split_ab.jsonl
      int CS = beff <= 128 ? 1 : 4;
      {
        const char* ce = getenv("TRID_BC_WCS");   // debug/A-B: force the cluster split (1, 2 or 4)
        if (ce && (atoi(ce) == 1 || atoi(ce) == 2 || atoi(ce) == 4)) CS = atoi(ce);
      }
      BwPart part{};
      const int total = bw_coff(beff, beff);
      part.c[0] = 0;
      for (int q = 1; q < CS; ++q) {
        int j = part.c[q - 1];
        while (j < beff && bw_coff(beff, j) < (int)((int64_t)total * q / CS)) ++j;
        part.c[q] = j;
      }
      part.c[CS] = beff;
      int maxw = 0;
      for (int q = 0; q < CS; ++q) {
        const int w = bw_coff(beff, part.c[q + 1]) - bw_coff(beff, part.c[q]);
        if (w > maxw) maxw = w;
      }
      // vb 2b | prt 4b | pf 2b | w b | colv b | scal 16 | sweep 2 | cofs (b ints) + pad | window
      const size_t smem = sizeof(double) * ((size_t)((10 * beff + 18 + (beff + 1) / 2 + 1) & ~1) + maxw);
      if (smem > 227 * 1024) return cudaErrorInvalidConfiguration;
      const void* fn = CS == 1 ? (const void*)bc_wide_kernel<1>
                               : (CS == 2 ? (const void*)bc_wide_kernel<2> : (const void*)bc_wide_kernel<4>);
      cudaError_t e2 = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      if (e2 != cudaSuccess) return e2;
      if (CS == 1) {
        int64_t grid = num_sms();
        if (grid > max_grid) grid = max_grid;
        bc_wide_kernel<1><<<(unsigned)grid, BW_NT, smem, st>>>(a, part);
      } else {
        cudaLaunchConfig_t cfg = {};
        cfg.blockDim = dim3(BW_NT);
        cfg.dynamicSmemBytes = smem;
        cfg.stream = st;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = (unsigned)CS;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        cfg.gridDim = dim3((unsigned)(CS * 37));
        int nc = 0;
        if (cudaOccupancyMaxActiveClusters(&nc, fn, &cfg) != cudaSuccess || nc < 1) return cudaErrorInvalidConfiguration;
        int64_t ncl = nc;
        if (ncl > max_grid) ncl = max_grid;
        cfg.gridDim = dim3((unsigned)(ncl * CS));
        e2 = CS == 2 ? cudaLaunchKernelEx(&cfg, bc_wide_kernel<2>, a, part)
                     : cudaLaunchKernelEx(&cfg, bc_wide_kernel<4>, a, part);
        if (e2 != cudaSuccess) return e2;
      }
    }
    count_launches(1);
    err = cudaGetLastError();
    if (err != cudaSuccess) return err;
  }
  {
    int blocks = (int)((n + 255) / 256);
    if (blocks > 4 * num_sms()) blocks = 4 * num_sms();
    band_extract_kernel<<<blocks, 256, 0, st>>>(n, ldab, band, d, e);
    count_launches(1);
    return cudaGetLastError();
  }
}

}  // namespace trid
