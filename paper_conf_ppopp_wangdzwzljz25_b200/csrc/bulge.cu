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

namespace trid {

constexpr int BC_NT = 256;
constexpr int BC_SMEM_MAXB = 64;

struct BcArgs {
  int64_t n;
  int b, ldab;
  int vs;  // V2 stride per step (the caller's b; >= b)
  double* band;
  double* V2;
  double* tau2;
  int* prog;
  unsigned* ticket;
};

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

__global__ void band_pack_kernel(int64_t n, int b, int ldab, const double* A, int64_t lda, double* band) {
  const int64_t total = n * ldab;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total; idx += (int64_t)gridDim.x * blockDim.x) {
    const int64_t c = idx / ldab, o = idx - c * ldab;
    band[idx] = (o <= b && c + o < n) ? A[(c + o) + c * lda] : 0.0;
  }
}

__global__ void band_extract_kernel(int64_t n, int ldab, const double* band, double* d, double* e) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    d[i] = band[i * ldab];
    if (i + 1 < n) e[i] = band[i * ldab + 1];
  }
}

// ---- block-level helpers (deterministic fixed-order reductions) ---------------------------------
// out[i] = sum_j M(i, j) x[j], i < R, j < C, via accessor get(i, j).  scratch >= BC_NT doubles.
template <class Get>
__device__ __forceinline__ void block_matvec(Get get, int R, int C, const double* x, double* out, double* scratch) {
  const int tid = threadIdx.x;
  const int q = R > 0 ? BC_NT / R : 1;
  if (R > 0 && tid < q * R) {
    const int i = tid % R, c = tid / R;
    double s = 0.0;
    for (int j = c; j < C; j += q) s += get(i, j) * x[j];
    scratch[c * R + i] = s;
  }
  __syncthreads();
  if (tid < R) {
    double s = 0.0;
    for (int c = 0; c < q; ++c) s += scratch[c * R + tid];
    out[tid] = s;
  }
  __syncthreads();
}

// Sum of x[lo..hi) computed by warp 0 in a fixed order; result broadcast through *res.
__device__ __forceinline__ void warp0_sumsq_tail(const double* x, int lo, int hi, double* res) {
  if (threadIdx.x < 32) {
    double s = 0.0;
    for (int i = lo + (int)threadIdx.x; i < hi; i += 32) s += x[i] * x[i];
    s = warp_sum(s);
    if (threadIdx.x == 0) *res = s;
  }
}
__device__ __forceinline__ void warp0_dot(const double* x, const double* y, int nn, double* res) {
  if (threadIdx.x < 32) {
    double s = 0.0;
    for (int i = threadIdx.x; i < nn; i += 32) s += x[i] * y[i];
    s = warp_sum(s);
    if (threadIdx.x == 0) *res = s;
  }
}

// Window accessors.  SMEM: dense symmetric D (LD = b+1) and dense O in shared memory.
// Global: directly on the compact band, D lower-only (symmetric reads mirror), O below it.
template <bool SM>
struct Win {
  double* Dm;   // SM: dense L x L (ld LD);  global: band + r0*ldab
  double* Om;   // SM: dense L2 x L (ld LD)
  int LD;       // SM: leading dimension; global: ldab
  int L;
  __device__ __forceinline__ double D(int i, int j) const {
    if (SM) return Dm[j * LD + i];
    return i >= j ? __ldcg(Dm + (int64_t)j * LD + (i - j)) : __ldcg(Dm + (int64_t)i * LD + (j - i));
  }
  __device__ __forceinline__ void Dsub(int i, int j, double v) const {  // i >= j (and mirror in SM)
    if (SM) {
      Dm[j * LD + i] -= v;
      if (i != j) Dm[i * LD + j] -= v;
    } else {
      double* p = Dm + (int64_t)j * LD + (i - j);
      __stcg(p, __ldcg(p) - v);
    }
  }
  __device__ __forceinline__ double* Optr(int i, int j) const {
    if (SM) return Om + j * LD + i;
    return Dm + (int64_t)j * LD + (L + i - j);
  }
  __device__ __forceinline__ double O(int i, int j) const { return SM ? *Optr(i, j) : __ldcg(Optr(i, j)); }
  __device__ __forceinline__ void Oset(int i, int j, double v) const {
    if (SM) *Optr(i, j) = v; else __stcg(Optr(i, j), v);
  }
};

template <bool SM>
__global__ void __launch_bounds__(BC_NT) bc_kernel(BcArgs a) {
  extern __shared__ __align__(16) double sm[];
  const int b = a.b, tid = threadIdx.x;
  const int64_t n = a.n;
  const int LD = b + 1;
  double* Dm = sm;
  double* Om = SM ? sm + LD * b : sm;
  double* vec = SM ? Om + LD * b : sm;
  double* v = vec;            // b   current reflector
  double* vn = v + b;         // b   next reflector
  double* p = vn + b;         // b   D v / O v / v^T O
  double* wv = p + b;         // b
  double* scratch = wv + b;   // BC_NT
  double* sc = scratch + BC_NT;  // scalars: [0] sum, [1] tau, [2] tau_next, [3] beta
  __shared__ int64_t s_sweep;

  for (;;) {
    if (tid == 0) s_sweep = (int64_t)atomicAdd(a.ticket, 1u);
    __syncthreads();
    const int64_t s = s_sweep;
    __syncthreads();
    if (s > n - 3) return;
    const int64_t nst = bc_steps(n, b, s);
    const int64_t off = bc_offset(n, b, s);
    const int64_t nprev = s > 0 ? bc_steps(n, b, s - 1) : 0;
    for (int64_t m = 0; m < nst; ++m) {
      const int64_t r0 = s + 1 + m * b;
      const int64_t r1 = (s + (m + 1) * b < n - 1) ? s + (m + 1) * b : n - 1;
      const int L = (int)(r1 - r0 + 1);
      const int64_t r2 = (r1 + b < n - 1) ? r1 + b : n - 1;
      const int L2 = (int)(r2 - r1);
      // ---- lag-2 dependency (R9): sweep s-1 must have completed step m+1
      if (s > 0) {
        if (tid == 0) {
          const int need = (int)((m + 2 < nprev) ? m + 2 : nprev);
          while (ld_acquire_s32(a.prog + (s - 1)) < need) {
          }
        }
        __syncthreads();
      }
      // ---- step 0: reflector from column s (rows s+1 .. s+L), compact column s offsets 1..L
      if (m == 0) {
        double* col = a.band + s * a.ldab;
        for (int i = tid; i < L; i += BC_NT) v[i] = __ldcg(col + 1 + i);
        __syncthreads();
        warp0_sumsq_tail(v, 1, L, sc);
        __syncthreads();
        const House h = make_house(v[0], sc[0]);
        __syncthreads();
        for (int i = tid; i < L; i += BC_NT) {
          const double x = v[i];
          v[i] = i == 0 ? 1.0 : h.scale * x;
          __stcg(col + 1 + i, i == 0 ? h.beta : 0.0);
        }
        if (tid == 0) sc[1] = h.tau;
        __syncthreads();
      }
      const double tau = sc[1];
      Win<SM> W;
      W.L = L;
      if (SM) {
        W.Dm = Dm; W.Om = Om; W.LD = LD;
        const double* src = a.band + r0 * a.ldab;
        const int span = L * a.ldab;
        for (int idx = tid; idx < span; idx += BC_NT) {
          const int j = idx / a.ldab, o = idx - j * a.ldab;
          const double x = __ldcg(src + idx);
          if (j + o < L) {
            Dm[j * LD + (j + o)] = x;
            Dm[(j + o) * LD + j] = x;
          } else if (j + o - L < L2) {
            Om[j * LD + (j + o - L)] = x;
          }
        }
      } else {
        W.Dm = a.band + r0 * a.ldab; W.Om = nullptr; W.LD = a.ldab;
      }
      __syncthreads();
      if (tau != 0.0) {
        // ---- two-sided on B_d:  p = tau D v;  wv = p - 1/2 tau (p^T v) v;  D -= v wv^T + wv v^T
        block_matvec([&](int i, int j) { return W.D(i, j); }, L, L, v, p, scratch);
        for (int i = tid; i < L; i += BC_NT) p[i] *= tau;
        __syncthreads();
        warp0_dot(p, v, L, sc);   // pv = p^T v with p = tau D v
        __syncthreads();
        const double pv = sc[0];
        for (int i = tid; i < L; i += BC_NT) wv[i] = p[i] - 0.5 * tau * pv * v[i];
        __syncthreads();
        for (int idx = tid; idx < L * L; idx += BC_NT) {
          const int i = idx % L, j = idx / L;
          if (i >= j) W.Dsub(i, j, v[i] * wv[j] + wv[i] * v[j]);
        }
        __syncthreads();
        // ---- right-apply to B_od (creates the bulge):  O -= tau (O v) v^T
        if (L2 > 0) {
          block_matvec([&](int i, int j) { return W.O(i, j); }, L2, L, v, p, scratch);
          for (int idx = tid; idx < L2 * L; idx += BC_NT) {
            const int i = idx % L2, j = idx / L2;
            W.Oset(i, j, W.O(i, j) - tau * p[i] * v[j]);
          }
          __syncthreads();
        }
      }
      // ---- next reflector from the bulge's first column, left-apply to O(:, 1:)
      if (L2 > 0) {
        for (int i = tid; i < L2; i += BC_NT) vn[i] = W.O(i, 0);
        __syncthreads();
        warp0_sumsq_tail(vn, 1, L2, sc);
        __syncthreads();
        const House h = make_house(vn[0], sc[0]);
        __syncthreads();
        for (int i = tid; i < L2; i += BC_NT) {
          vn[i] = i == 0 ? 1.0 : h.scale * vn[i];
          W.Oset(i, 0, i == 0 ? h.beta : 0.0);
        }
        if (tid == 0) sc[2] = h.tau;
        __syncthreads();
        if (h.tau != 0.0 && L > 1) {
          // z_j = vn^T O(:, j), j = 1..L-1 (stored in p[j])
          const int C = L - 1;
          const int q = BC_NT / C;
          if (tid < q * C) {
            const int j = 1 + tid % C, c = tid / C;
            double acc = 0.0;
            for (int i = c; i < L2; i += q) acc += vn[i] * W.O(i, j);
            scratch[c * C + (j - 1)] = acc;
          }
          __syncthreads();
          if (tid < C) {
            double acc = 0.0;
            for (int c = 0; c < q; ++c) acc += scratch[c * C + tid];
            p[tid + 1] = acc;
          }
          __syncthreads();
          for (int idx = tid; idx < L2 * C; idx += BC_NT) {
            const int i = idx % L2, j = 1 + idx / L2;
            W.Oset(i, j, W.O(i, j) - h.tau * vn[i] * p[j]);
          }
        }
        __syncthreads();
      }
      // ---- write back the window, the reflector of this step, then publish progress
      if (SM) {
        double* dst = a.band + r0 * a.ldab;
        const int span = L * a.ldab;
        for (int idx = tid; idx < span; idx += BC_NT) {
          const int j = idx / a.ldab, o = idx - j * a.ldab;
          if (j + o < L) __stcg(dst + idx, Dm[j * LD + (j + o)]);
          else if (j + o - L < L2) __stcg(dst + idx, Om[j * LD + (j + o - L)]);
        }
      }
      if (a.V2) {
        double* vd = a.V2 + (off + m) * a.vs;
        for (int i = tid; i < a.vs; i += BC_NT) vd[i] = i < L ? v[i] : 0.0;
        if (tid == 0) a.tau2[off + m] = tau;
      }
      __syncthreads();
      if (tid == 0) {
        __threadfence();
        st_release_s32(a.prog + s, (int)(m + 1));
      }
      // hand the next reflector to step m+1
      for (int i = tid; i < L2; i += BC_NT) v[i] = vn[i];
      if (tid == 0) sc[1] = sc[2];
      __syncthreads();
    }
  }
}

size_t bc_work_bytes(int64_t n, int b) {
  const size_t band = sizeof(double) * (size_t)n * bc_ldab(n, b);
  const size_t flags = sizeof(int) * (size_t)(n + 64);
  return ((band + 255) / 256) * 256 + ((flags + 255) / 256) * 256;
}

cudaError_t bulge_chase(int64_t n, int b, const double* A, int64_t lda, double* d, double* e, double* V2,
                        double* tau2, void* work, cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  const int beff = (int)((b < n - 1) ? b : (n - 1 > 0 ? n - 1 : 1));
  const int ldab = bc_ldab(n, beff);
  double* band = (double*)work;
  const size_t band_bytes = ((sizeof(double) * (size_t)n * ldab + 255) / 256) * 256;
  int* prog = (int*)((char*)work + band_bytes);
  unsigned* ticket = (unsigned*)(prog + n + 32);
  {
    int64_t total = n * (int64_t)ldab;
    int blocks = (int)((total + 255) / 256);
    if (blocks > 8 * kNumSMsB200 * 4) blocks = 8 * kNumSMsB200 * 4;
    band_pack_kernel<<<blocks, 256, 0, st>>>(n, beff, ldab, A, lda, band);
    count_launches(1);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) return err;
  }
  if (beff >= 2 && n >= 3) {
    cudaError_t err = cudaMemsetAsync(prog, 0, sizeof(int) * (size_t)(n + 64), st);
    if (err != cudaSuccess) return err;
    BcArgs a;
    // beff = min(b, n-1) gives the same step geometry as b (for b >= n-1 every sweep is one step on
    // rows s+1..n-1); V2 keeps the caller's stride b (header contract).
    a.n = n; a.b = beff; a.ldab = ldab; a.vs = b; a.band = band; a.V2 = V2; a.tau2 = tau2; a.prog = prog;
    a.ticket = ticket;
    const size_t vec = sizeof(double) * (size_t)(4 * beff + BC_NT + 8);
    const bool use_sm = beff <= BC_SMEM_MAXB;
    const size_t smem = use_sm ? vec + sizeof(double) * 2 * (size_t)(beff + 1) * beff : vec;
    int occ = 1;
    if (use_sm) {
      cudaFuncSetAttribute(bc_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, bc_kernel<true>, BC_NT, smem);
    } else {
      cudaFuncSetAttribute(bc_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, bc_kernel<false>, BC_NT, smem);
    }
    if (occ < 1) occ = 1;
    int64_t grid = (int64_t)kNumSMsB200 * occ;
    if (grid > n - 2) grid = n - 2;
    if (use_sm) bc_kernel<true><<<(unsigned)grid, BC_NT, smem, st>>>(a);
    else bc_kernel<false><<<(unsigned)grid, BC_NT, smem, st>>>(a);
    count_launches(1);
    err = cudaGetLastError();
    if (err != cudaSuccess) return err;
  }
  {
    int blocks = (int)((n + 255) / 256);
    if (blocks > 4 * kNumSMsB200) blocks = 4 * kNumSMsB200;
    band_extract_kernel<<<blocks, 256, 0, st>>>(n, ldab, band, d, e);
    count_launches(1);
    return cudaGetLastError();
  }
}

}  // namespace trid
