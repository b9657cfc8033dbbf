// FP64 throughput microbenchmark for B200 (sm_100a): DMMA (mma.sync f64) shapes vs DFMA.
// Also verifies the register-fragment layouts assumed by the library's DMMA engine.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb tools/microbench_fp64.cu
// Test-side tooling only: it measures the FP64 ceiling the roofline in DESIGN.md uses.
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

constexpr int ITERS = 4096;
constexpr int CHAINS = 4;

__global__ void k_m8n8k4(double* out) {
  double a = 1.0 + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
  double c[CHAINS][2] = {};
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int q = 0; q < CHAINS; ++q)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                   : "+d"(c[q][0]), "+d"(c[q][1]) : "d"(a), "d"(b));
  }
  double s = 0; for (int q = 0; q < CHAINS; ++q) s += c[q][0] + c[q][1];
  if (s == 12345.678) out[0] = s;
}

__global__ void k_m16n8k4(double* out) {
  double a0 = 1.0 + threadIdx.x * 1e-9, a1 = a0, b = 1.0 - threadIdx.x * 1e-9;
  double c[CHAINS][4] = {};
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int q = 0; q < CHAINS; ++q)
      asm volatile("mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};\n"
                   : "+d"(c[q][0]), "+d"(c[q][1]), "+d"(c[q][2]), "+d"(c[q][3]) : "d"(a0), "d"(a1), "d"(b));
  }
  double s = 0; for (int q = 0; q < CHAINS; ++q) s += c[q][0] + c[q][1] + c[q][2] + c[q][3];
  if (s == 12345.678) out[0] = s;
}

__global__ void k_m16n8k8(double* out) {
  double a[4], b[2];
  for (int i = 0; i < 4; ++i) a[i] = 1.0 + (threadIdx.x + i) * 1e-9;
  for (int i = 0; i < 2; ++i) b[i] = 1.0 - (threadIdx.x + i) * 1e-9;
  double c[CHAINS][4] = {};
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int q = 0; q < CHAINS; ++q)
      asm volatile("mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};\n"
                   : "+d"(c[q][0]), "+d"(c[q][1]), "+d"(c[q][2]), "+d"(c[q][3])
                   : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(b[0]), "d"(b[1]));
  }
  double s = 0; for (int q = 0; q < CHAINS; ++q) s += c[q][0] + c[q][1] + c[q][2] + c[q][3];
  if (s == 12345.678) out[0] = s;
}

__global__ void k_m16n8k16(double* out) {
  double a[8], b[4];
  for (int i = 0; i < 8; ++i) a[i] = 1.0 + (threadIdx.x + i) * 1e-9;
  for (int i = 0; i < 4; ++i) b[i] = 1.0 - (threadIdx.x + i) * 1e-9;
  double c[CHAINS][4] = {};
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int q = 0; q < CHAINS; ++q)
      asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, {%12,%13,%14,%15}, {%0,%1,%2,%3};\n"
                   : "+d"(c[q][0]), "+d"(c[q][1]), "+d"(c[q][2]), "+d"(c[q][3])
                   : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(a[4]), "d"(a[5]), "d"(a[6]), "d"(a[7]),
                     "d"(b[0]), "d"(b[1]), "d"(b[2]), "d"(b[3]));
  }
  double s = 0; for (int q = 0; q < CHAINS; ++q) s += c[q][0] + c[q][1] + c[q][2] + c[q][3];
  if (s == 12345.678) out[0] = s;
}

__global__ void k_dfma(double* out) {
  double x[8];
  for (int i = 0; i < 8; ++i) x[i] = 1.0 + (threadIdx.x + i) * 1e-12;
  const double m = 0.999999999, ad = 1e-7;
  for (int it = 0; it < ITERS * 4; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] = fma(x[i], m, ad);
  }
  double s = 0; for (int i = 0; i < 8; ++i) s += x[i];
  if (s == 12345.678) out[0] = s;
}

// ---- fragment-layout verification: D = A*B (A 16xK row-major, B Kx8), one warp -------------
__global__ void k_layout16(const double* A, const double* B, double* D, int K) {
  int lane = threadIdx.x, g = lane >> 2, t = lane & 3;
  double c[4] = {0, 0, 0, 0};
  if (K == 4) {
    double a0 = A[g * 4 + t], a1 = A[(g + 8) * 4 + t], b0 = B[t * 8 + g];
    asm volatile("mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};\n"
                 : "+d"(c[0]), "+d"(c[1]), "+d"(c[2]), "+d"(c[3]) : "d"(a0), "d"(a1), "d"(b0));
  } else if (K == 8) {
    double a[4], b[2];
    for (int i = 0; i < 4; ++i) a[i] = A[(g + 8 * (i & 1)) * 8 + t + 4 * (i >> 1)];
    for (int i = 0; i < 2; ++i) b[i] = B[(t + 4 * i) * 8 + g];
    asm volatile("mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};\n"
                 : "+d"(c[0]), "+d"(c[1]), "+d"(c[2]), "+d"(c[3])
                 : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(b[0]), "d"(b[1]));
  } else {
    double a[8], b[4];
    for (int i = 0; i < 8; ++i) a[i] = A[(g + 8 * (i & 1)) * 16 + t + 4 * (i >> 1)];
    for (int i = 0; i < 4; ++i) b[i] = B[(t + 4 * i) * 8 + g];
    asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, {%12,%13,%14,%15}, {%0,%1,%2,%3};\n"
                 : "+d"(c[0]), "+d"(c[1]), "+d"(c[2]), "+d"(c[3])
                 : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(a[4]), "d"(a[5]), "d"(a[6]), "d"(a[7]),
                   "d"(b[0]), "d"(b[1]), "d"(b[2]), "d"(b[3]));
  }
  D[g * 8 + 2 * t] = c[0]; D[g * 8 + 2 * t + 1] = c[1];
  D[(g + 8) * 8 + 2 * t] = c[2]; D[(g + 8) * 8 + 2 * t + 1] = c[3];
}

static double check_layout(int K) {
  double hA[16 * 16], hB[16 * 8], hD[16 * 8];
  for (int i = 0; i < 16 * K; ++i) hA[i] = (double)((i * 7919) % 97) - 48.0;
  for (int i = 0; i < K * 8; ++i) hB[i] = (double)((i * 104729) % 89) - 44.0;
  double *dA, *dB, *dD;
  CK(cudaMalloc(&dA, sizeof hA)); CK(cudaMalloc(&dB, sizeof hB)); CK(cudaMalloc(&dD, sizeof hD));
  CK(cudaMemcpy(dA, hA, sizeof hA, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, hB, sizeof hB, cudaMemcpyHostToDevice));
  k_layout16<<<1, 32>>>(dA, dB, dD, K);
  CK(cudaMemcpy(hD, dD, sizeof hD, cudaMemcpyDeviceToHost));
  double err = 0;
  for (int i = 0; i < 16; ++i)
    for (int j = 0; j < 8; ++j) {
      double s = 0;
      for (int k = 0; k < K; ++k) s += hA[i * K + k] * hB[k * 8 + j];
      err = fmax(err, fabs(s - hD[i * 8 + j]));
    }
  cudaFree(dA); cudaFree(dB); cudaFree(dD);
  return err;
}

template <typename F>
static void run(const char* name, F kern, double flop_per_thread_iter, int blocks, int threads) {
  double* out; CK(cudaMalloc(&out, 8));
  kern<<<blocks, threads>>>(out); CK(cudaDeviceSynchronize());
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  const int reps = 5;
  for (int r = 0; r < reps; ++r) kern<<<blocks, threads>>>(out);
  cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  double flops = flop_per_thread_iter * (double)blocks * threads * reps;
  printf("{\"kernel\": \"%s\", \"blocks\": %d, \"threads\": %d, \"tflops\": %.3f}\n", name, blocks, threads,
         flops / (ms * 1e-3) / 1e12);
  cudaFree(out);
}

int main() {
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  printf("{\"device\": \"%s\", \"sms\": %d, \"cc\": \"%d.%d\"}\n", p.name, p.multiProcessorCount, p.major, p.minor);
  printf("{\"layout_err_k4\": %g, \"layout_err_k8\": %g, \"layout_err_k16\": %g}\n", check_layout(4), check_layout(8),
         check_layout(16));
  int sms = p.multiProcessorCount;
  // per warp per mma: 2*M*N*K flops; per thread = /32
  for (int wpb : {4, 8, 16}) {
    int thr = 32 * wpb;
    for (int bps : {1, 2}) {
      run("dmma_m8n8k4", k_m8n8k4, 2.0 * 8 * 8 * 4 / 32 * CHAINS * ITERS, sms * bps, thr);
      run("dmma_m16n8k4", k_m16n8k4, 2.0 * 16 * 8 * 4 / 32 * CHAINS * ITERS, sms * bps, thr);
      run("dmma_m16n8k8", k_m16n8k8, 2.0 * 16 * 8 * 8 / 32 * CHAINS * ITERS, sms * bps, thr);
      run("dmma_m16n8k16", k_m16n8k16, 2.0 * 16 * 8 * 16 / 32 * CHAINS * ITERS, sms * bps, thr);
      run("dfma", k_dfma, 2.0 * 8 * ITERS * 4, sms * bps, thr);
    }
  }
  return 0;
}
