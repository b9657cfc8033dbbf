// eig.cu — eigenvalues of the symmetric tridiagonal T = tridiag(e, d, e) on the GPU by Sturm-sequence
// bisection (the eigenvalues-only EVD of P:446-448 without MAGMA; the gate G3 of
// north_star uses the same definition).
//
// Method (plain definition, as LAPACK dstebz/dlaebz): the number of eigenvalues of T below x equals the
// number of negative pivots q_i of the LDL^T factorisation of T - x I,
//     q_0 = d_0 - x,   q_i = d_i - x - e_{i-1}^2 / q_{i-1},
// with |q| < pivmin replaced by -pivmin (pivmin = DBL_MIN * max(1, max e^2)).  Eigenvalue k (ascending) is the
// limit of bisection on [gl, gu] (Gershgorin bounds widened by 2 eps |.| + 2 pivmin) keeping count(lo) <= k <
// count(hi), stopped when hi - lo <= 2 eps max(|lo|, |hi|) + pivmin.
//
// B200 design: the count is a sequential recurrence with one IEEE division per element, so one bisection step is
// a long latency-bound chain.  A group of G = 2^P lanes per eigenvalue (G chosen so n G fills ~2048 threads per SM,
// at most a warp) runs an EXACT multisection: in one pass it counts at the 2^P - 1 nodes of the depth-P bisection
// subtree below the current interval (each node value built by the same halvings the serial loop performs), then
// walks P levels with the serial loop's tests -- the serial bisection, P steps per dependent recurrence.  Every
// thread of a CTA walks the same d_i / e_i^2 in lockstep out of a shared-memory tile.  The bounds come from one
// small reduction kernel (min/max are exact, so the order does not matter).  Every operation is the plain
// expression above in the same order with IEEE division (no FMA can contract it): the results equal a serial
// implementation of the same definition bit for bit (TRID_STEBZ_P=0 runs the one-thread-per-eigenvalue loop).
#include "common.cuh"
#include "eig.cuh"
#include "prof.cuh"

#include <float.h>
#include <stdlib.h>

namespace trid {

constexpr int EIG_NT = 128;    // threads (eigenvalues) per CTA of the bisection kernel
constexpr int EIG_TILE = 1024; // d / e^2 elements staged per shared-memory tile

// bounds[0] = gl, bounds[1] = gu, bounds[2] = pivmin (widened as in the header comment); one CTA.
__global__ void __launch_bounds__(1024) sturm_bounds_kernel(int64_t n, const double* d, const double* e,
                                                            double* bounds) {
  __shared__ double s_lo[32], s_hi[32], s_e2[32];
  double lo = d[0], hi = d[0], em = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += blockDim.x) {
    const double r = (i > 0 ? fabs(e[i - 1]) : 0.0) + (i + 1 < n ? fabs(e[i]) : 0.0);
    lo = fmin(lo, d[i] - r);
    hi = fmax(hi, d[i] + r);
    if (i + 1 < n) em = fmax(em, e[i] * e[i]);
  }
  for (int o = 16; o > 0; o >>= 1) {
    lo = fmin(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = fmax(hi, __shfl_xor_sync(0xffffffffu, hi, o));
    em = fmax(em, __shfl_xor_sync(0xffffffffu, em, o));
  }
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) {
    s_lo[w] = lo;
    s_hi[w] = hi;
    s_e2[w] = em;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    const int nw = (blockDim.x + 31) / 32;
    for (int q = 1; q < nw; ++q) {
      lo = fmin(lo, s_lo[q]);
      hi = fmax(hi, s_hi[q]);
      em = fmax(em, s_e2[q]);
    }
    lo = fmin(lo, s_lo[0]);
    hi = fmax(hi, s_hi[0]);
    em = fmax(em, s_e2[0]);
    const double pivmin = DBL_MIN * (em > 1.0 ? em : 1.0);
    const double scale = fabs(lo) > fabs(hi) ? fabs(lo) : fabs(hi);
    bounds[0] = lo - (2.0 * DBL_EPSILON * scale + 2.0 * pivmin + 1e-300);
    bounds[1] = hi + (2.0 * DBL_EPSILON * scale + 2.0 * pivmin + 1e-300);
    bounds[2] = pivmin;
  }
}

// e2[i] = e[i]^2 (exact product, computed once instead of once per bisection step)
__global__ void square_kernel(int64_t n1, const double* e, double* e2) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n1; i += (int64_t)gridDim.x * blockDim.x)
    e2[i] = e[i] * e[i];
}

// One thread per eigenvalue index k = blockIdx.x * EIG_NT + threadIdx.x.  All threads of the CTA run the same
// number of bisection steps (a thread whose interval converged keeps its result and idles through the count),
// so the CTA walks the shared tiles together.
__global__ void __launch_bounds__(EIG_NT) sturm_bisect_kernel(int64_t n, const double* __restrict__ d,
                                                              const double* __restrict__ e2,
                                                              const double* __restrict__ bounds, double* w) {
  __shared__ double sd[EIG_TILE], se[EIG_TILE];
  __shared__ int s_active;
  const int64_t k = (int64_t)blockIdx.x * EIG_NT + threadIdx.x;
  const double pivmin = bounds[2];
  double lo = bounds[0], hi = bounds[1];
  bool active = k < n;
  for (int it = 0; it < 256; ++it) {
    double mid = 0.0;
    if (active) {
      const double tol = 2.0 * DBL_EPSILON * (fabs(lo) > fabs(hi) ? fabs(lo) : fabs(hi)) + pivmin;
      if (hi - lo <= tol) {
        active = false;
      } else {
        mid = 0.5 * (lo + hi);
        if (mid <= lo || mid >= hi) active = false;
      }
    }
    if (threadIdx.x == 0) s_active = 0;
    __syncthreads();
    if (active) s_active = 1;
    __syncthreads();
    if (!s_active) break;
    // Sturm count of T - mid I
    int64_t cnt = 0;
    double q = 1.0;
    for (int64_t t0 = 0; t0 < n; t0 += EIG_TILE) {
      const int len = (int)((n - t0) < EIG_TILE ? (n - t0) : EIG_TILE);
      __syncthreads();
      for (int i = threadIdx.x; i < len; i += EIG_NT) {
        sd[i] = d[t0 + i];
        se[i] = (t0 + i > 0) ? e2[t0 + i - 1] : 0.0;
      }
      __syncthreads();
      if (active) {
        int i = 0;
        if (t0 == 0) {
          q = sd[0] - mid;
          if (fabs(q) < pivmin) q = -pivmin;
          if (q < 0) ++cnt;
          i = 1;
        }
        for (; i < len; ++i) {
          q = sd[i] - mid - se[i] / q;
          if (fabs(q) < pivmin) q = -pivmin;
          if (q < 0) ++cnt;
        }
      }
    }
    if (active) {
      if (cnt > k) hi = mid;
      else lo = mid;
    }
  }
  if (k < n) w[k] = 0.5 * (lo + hi);
}

// Exact multisection: a group of G = 2^P lanes per eigenvalue evaluates, in one pass, the Sturm counts at all
// 2^P - 1 midpoints of the depth-P bisection subtree below the current interval (lane l >= 1 = heap node l; each node
// value is obtained by the same halvings 0.5 (lo + hi) the serial bisection performs along that path), then every
// lane walks the P levels with the serial loop's termination tests, taking each level's count from the node's lane.
// The walk visits exactly the serial bisection's midpoints, so the result is the serial result bit for bit, in
// ceil(steps / P) dependent recurrences instead of `steps` (the count is a latency-bound chain of divisions).
template <int P>
__global__ void __launch_bounds__(EIG_NT) sturm_msect_kernel(int64_t n, const double* __restrict__ d,
                                                            const double* __restrict__ e2,
                                                            const double* __restrict__ bounds, double* w) {
  constexpr int G = 1 << P;
  __shared__ double sd[EIG_TILE], se[EIG_TILE];
  __shared__ int s_active;
  const int lane = threadIdx.x & 31, gl = threadIdx.x & (G - 1);
  const int gbase = lane & ~(G - 1);
  const int64_t k = ((int64_t)blockIdx.x * EIG_NT + threadIdx.x) / G;
  const double pivmin = bounds[2];
  double lo = bounds[0], hi = bounds[1];
  bool active = k < n;
  int it = 0;   // serial bisection steps taken (the serial loop stops after 256)
  for (;;) {
    if (threadIdx.x == 0) s_active = 0;
    __syncthreads();
    if (active) s_active = 1;
    __syncthreads();
    if (!s_active) break;
    // this lane's node of the subtree
    double mid = 0.0;
    const bool node = active && gl >= 1;
    if (node) {
      double nl = lo, nh = hi;
      const int depth = 31 - __clz(gl);
      for (int dd = depth - 1; dd >= 0; --dd) {
        const double m2 = 0.5 * (nl + nh);
        if ((gl >> dd) & 1) nl = m2;
        else nh = m2;
      }
      mid = 0.5 * (nl + nh);
    }
    // Sturm count of T - mid I
    int64_t cnt = 0;
    double q = 1.0;
    for (int64_t t0 = 0; t0 < n; t0 += EIG_TILE) {
      const int len = (int)((n - t0) < EIG_TILE ? (n - t0) : EIG_TILE);
      __syncthreads();
      for (int i = threadIdx.x; i < len; i += EIG_NT) {
        sd[i] = d[t0 + i];
        se[i] = (t0 + i > 0) ? e2[t0 + i - 1] : 0.0;
      }
      __syncthreads();
      if (node) {
        int i = 0;
        if (t0 == 0) {
          q = sd[0] - mid;
          if (fabs(q) < pivmin) q = -pivmin;
          if (q < 0) ++cnt;
          i = 1;
        }
        for (; i < len; ++i) {
          q = sd[i] - mid - se[i] / q;
          if (fabs(q) < pivmin) q = -pivmin;
          if (q < 0) ++cnt;
        }
      }
    }
    // walk the P levels exactly as the serial loop (every lane of the warp takes part in the shuffles)
    int nd = 1;
    for (int dd = 0; dd < P; ++dd) {
      bool go = active && it < 256;
      double m = 0.0;
      if (go) {
        const double tol = 2.0 * DBL_EPSILON * (fabs(lo) > fabs(hi) ? fabs(lo) : fabs(hi)) + pivmin;
        if (hi - lo <= tol) {
          go = false;
        } else {
          m = 0.5 * (lo + hi);
          if (m <= lo || m >= hi) go = false;
        }
      }
      const long long c = __shfl_sync(0xffffffffu, (long long)cnt, gbase + (nd < G ? nd : 0));
      if (go) {
        ++it;
        if (c > k) {
          hi = m;
          nd = 2 * nd;
        } else {
          lo = m;
          nd = 2 * nd + 1;
        }
      } else {
        active = false;
      }
    }
    if (it >= 256) active = false;
  }
  if (gl == 0 && k < n) w[k] = 0.5 * (lo + hi);
}

size_t stebz_work_bytes(int64_t n) {
  return ((sizeof(double) * (size_t)(n > 1 ? n - 1 : 1) + 255) / 256) * 256 + 256;
}

cudaError_t stebz(int64_t n, const double* d, const double* e, double* w, void* work, cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  double* e2 = (double*)work;
  double* bounds = (double*)((char*)work + ((sizeof(double) * (size_t)(n > 1 ? n - 1 : 1) + 255) / 256) * 256);
  if (n > 1) {
    int blocks = (int)((n - 1 + 255) / 256);
    if (blocks > 4 * num_sms()) blocks = 4 * num_sms();
    square_kernel<<<blocks, 256, 0, st>>>(n - 1, e, e2);
    count_launches(1);
  }
  sturm_bounds_kernel<<<1, 1024, 0, st>>>(n, d, e, bounds);
  count_launches(1);
  // lanes per eigenvalue: fill ~2048 threads per SM (latency-bound chains), at most a warp; below 16 lanes the
  // extra counts cost as much as the shorter chain saves (measured at n = 32768: 195 ms with 8 lanes, 192 ms with
  // one thread per eigenvalue; n = 8192: 29 ms with 32 lanes vs 46 ms)
  const int64_t g = (int64_t)num_sms() * 2048 / (n > 0 ? n : 1);
  int P = 0;
  if (g >= 16)
    while (P < 5 && ((int64_t)1 << (P + 1)) <= g) ++P;
  static const char* me = getenv("TRID_STEBZ_P");   // A/B: force the multisection depth (0 = plain bisection)
  if (me) P = atoi(me) < 0 ? 0 : (atoi(me) > 5 ? 5 : atoi(me));
  if (P == 0) {
    const int64_t grid = (n + EIG_NT - 1) / EIG_NT;
    sturm_bisect_kernel<<<(unsigned)grid, EIG_NT, 0, st>>>(n, d, e2, bounds, w);
  } else {
    const int64_t grid = ((n << P) + EIG_NT - 1) / EIG_NT;
    switch (P) {
      case 1: sturm_msect_kernel<1><<<(unsigned)grid, EIG_NT, 0, st>>>(n, d, e2, bounds, w); break;
      case 2: sturm_msect_kernel<2><<<(unsigned)grid, EIG_NT, 0, st>>>(n, d, e2, bounds, w); break;
      case 3: sturm_msect_kernel<3><<<(unsigned)grid, EIG_NT, 0, st>>>(n, d, e2, bounds, w); break;
      case 4: sturm_msect_kernel<4><<<(unsigned)grid, EIG_NT, 0, st>>>(n, d, e2, bounds, w); break;
      default: sturm_msect_kernel<5><<<(unsigned)grid, EIG_NT, 0, st>>>(n, d, e2, bounds, w); break;
    }
  }
  count_launches(1);
  return cudaGetLastError();
}

}  // namespace trid
