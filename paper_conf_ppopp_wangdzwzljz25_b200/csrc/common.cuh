// common.cuh — device helpers shared by the libtrid kernels (sm_100a only).
// FP64 tensor-core math on Blackwell: tcgen05 has no f64 kind, so FP64 contractions use the warp-level
// DMMA path (mma.sync ... f64, SASS DMMA.8x8x4).  Measured on this pool's B200: 37.0 TFLOP/s for DMMA
// and 36.7 for DFMA at 1965 MHz (profiles/r01_fp64_microbench.jsonl).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <stdlib.h>

#include <atomic>

#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ != 1000)
#error "libtrid is written for sm_100a only"
#endif

namespace trid {

constexpr int kNumSMsB200 = 148;   // B200 SM count: upper bound for grid-sized workspaces (partials, barriers)

// ---- host: per-device cached attributes (thread-safe: libtrid is driven from several host threads by the
// local multi-GPU ranks).  A racing first call may query twice; both store the same value.
constexpr int kMaxDevices = 64;
inline int cur_device() {
  int d = 0;
  if (cudaGetDevice(&d) != cudaSuccess || d < 0 || d >= kMaxDevices) d = 0;
  return d;
}
// SMs of the current device, capped at kNumSMsB200 (workspaces are sized for at most that many CTAs).
inline int num_sms() {
  static std::atomic<int> cache[kMaxDevices];
  const int d = cur_device();
  int v = cache[d].load(std::memory_order_relaxed);
  if (v == 0) {
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d) != cudaSuccess || v < 1) v = kNumSMsB200;
    if (v > kNumSMsB200) v = kNumSMsB200;
    cache[d].store(v, std::memory_order_relaxed);
  }
  return v;
}
// True when a CUDA profiler/injection tool (Nsight Compute) is attached: such tools may refuse cooperative
// cluster launches, so the grid-barrier kernels then launch without the cooperative attribute (their grids are
// sized to co-resident clusters and the profiler serialises kernels, so every CTA is resident anyway).
inline bool profiler_attached() {
  static const bool on = getenv("NV_NSIGHT_INJECTION_TRANSPORT_TYPE") != nullptr ||
                         getenv("NV_NSIGHT_INJECTION_PORT_BASE") != nullptr || getenv("TRID_PANEL_NOCOOP") != nullptr;
  return on;
}
// Idempotent per-device setup (e.g. cudaFuncSetAttribute): runs f() until it succeeds once on this device.
struct DeviceOnce {
  std::atomic<unsigned long long> done{0};
  template <class F>
  cudaError_t operator()(F&& f) {
    const unsigned long long bit = 1ull << cur_device();
    if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
    const cudaError_t e = f();
    if (e == cudaSuccess) done.fetch_or(bit, std::memory_order_acq_rel);
    return e;
  }
};

// D(16x8) += A(16x8) * B(8x8), fp64.  Fragment layout (verified on B200, tools/microbench_fp64.cu):
//   g = lane>>2, t = lane&3;  a[i] = A[g + 8*(i&1)][t + 4*(i>>1)];  b[i] = B[t + 4*i][g];
//   c[0] = C[g][2t], c[1] = C[g][2t+1], c[2] = C[g+8][2t], c[3] = C[g+8][2t+1].
__device__ __forceinline__ void dmma_16x8x8(double (&c)[4], const double (&a)[4], const double (&b)[2]) {
  asm volatile(
      "mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};\n"
      : "+d"(c[0]), "+d"(c[1]), "+d"(c[2]), "+d"(c[3])
      : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(b[0]), "d"(b[1]));
}

// D(16x8) += A(16x4) * B(4x8), fp64: a0 = A[g][t], a1 = A[g+8][t]; b0 = B[t][g]; c as above.
__device__ __forceinline__ void dmma_16x8x4(double (&c)[4], double a0, double a1, double b0) {
  asm volatile(
      "mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};\n"
      : "+d"(c[0]), "+d"(c[1]), "+d"(c[2]), "+d"(c[3])
      : "d"(a0), "d"(a1), "d"(b0));
}

// 8-byte async copy global -> shared; pred == false zero-fills without reading global memory.
__device__ __forceinline__ void cp_async8(double* smem, const double* gmem, bool pred) {
  unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  int sz = pred ? 8 : 0;
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(s), "l"(gmem), "r"(sz) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }

__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];\n" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int ld_acquire_s32(const int* p) {
  int v;
  asm volatile("ld.acquire.gpu.global.s32 %0, [%1];\n" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned ld_relaxed_u32(const unsigned* p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];\n" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int ld_relaxed_s32(const int* p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];\n" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;\n" ::: "memory"); }
// Spin until *p >= need.  Polls with relaxed loads (an acquire load invalidates the SM's L1 on every
// poll) and finishes with one acquire re-read (cheaper than fence.acq_rel, which adds a GPU MEMBAR).
__device__ __forceinline__ void wait_geq(const int* p, int need) {
  while (ld_relaxed_s32(p) < need) __nanosleep(32);
  (void)ld_acquire_s32(p);   // the counter is monotone: this re-read succeeds and orders what follows
}
__device__ __forceinline__ void st_release_s32(int* p, int v) {
  asm volatile("st.release.gpu.global.s32 [%0], %1;\n" ::"l"(p), "r"(v) : "memory");
}

// Grid-wide barrier for a cooperatively launched grid.  `counter` is zero at launch; `epoch` is a
// per-CTA register copy of how many barriers this CTA has passed.  Monotone counter: no reset race.
__device__ __forceinline__ void grid_barrier(unsigned* counter, unsigned nblocks, unsigned& epoch) {
  __syncthreads();
  epoch += 1;
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(counter, 1u);
    const unsigned target = epoch * nblocks;
    while (ld_relaxed_u32(counter) < target) {
    }
    fence_acq_rel_gpu();
  }
  __syncthreads();
}

// ---- mbarrier + bulk (TMA) copies -----------------------------------------------------------------
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned parity) {
  unsigned done = 0;
  while (!done) {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  }
}
// global -> shared bulk copy completing on an mbarrier (bytes % 16 == 0, 16-byte aligned)
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
// shared -> global bulk copy (bulk-group completion)
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, unsigned bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;\n" ::"l"(dst), "r"(smem_u32(src)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;\n" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;\n" ::: "memory"); }
// Narrow proxy fences (the unqualified fence.proxy.async is a full GPU-scope MEMBAR).
__device__ __forceinline__ void fence_proxy_async_smem() { asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;\n" ::: "memory"); }

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// LAPACK dlarfg sign convention (R1/R1'): beta = -sign(alpha)*sqrt(alpha^2+sigma) with the
// sign taken from the sign bit; sigma == 0 -> tau = 0, beta = alpha, scale = 0 (no reflection).
struct House {
  double beta, tau, scale;
};
__device__ __forceinline__ House make_house(double alpha, double sigma) {
  House h;
  if (sigma == 0.0) {
    h.beta = alpha;
    h.tau = 0.0;
    h.scale = 0.0;
  } else {
    double nrm = sqrt(alpha * alpha + sigma);
    h.beta = signbit(alpha) ? nrm : -nrm;
    h.tau = (h.beta - alpha) / h.beta;
    h.scale = 1.0 / (alpha - h.beta);
  }
  return h;
}

}  // namespace trid

namespace trid {
void record_cuda_error(cudaError_t e, const char* what);
}
#define TRID_CUDA_TRY(x)                              \
  do {                                                \
    cudaError_t _e = (x);                             \
    if (_e != cudaSuccess) {                          \
      trid::record_cuda_error(_e, #x);                \
      return TRID_ERR_CUDA;                           \
    }                                                 \
  } while (0)
