// Latency microbenchmark on B200: dependent-chain cycles per op for DFMA/DADD/DMUL/FFMA, LDS.64,
// SHFL (double), __syncthreads at 256 threads, and DMMA m16n8k8.  Test-side tooling.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/lat tools/microbench_latency.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int N = 1024;

__global__ void lat_kernel(double* out, long long* cyc, double seed) {
  __shared__ double sm[1024];
  const int tid = threadIdx.x;
  for (int i = tid; i < 1024; i += blockDim.x) sm[i] = (i + 1) * 1e-3;
  __syncthreads();
  double x = seed + tid, y = 1.0000001, z = 1e-9;
  float xf = (float)seed;
  long long t0, t1;
  // DFMA chain
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) x = fma(x, y, z);
  t1 = clock64();
  if (tid == 0) cyc[0] = t1 - t0;
  // DADD chain
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) x = x + z;
  t1 = clock64();
  if (tid == 0) cyc[1] = t1 - t0;
  // DMUL chain
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) x = x * y;
  t1 = clock64();
  if (tid == 0) cyc[2] = t1 - t0;
  // FFMA chain
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) xf = fmaf(xf, 1.0000001f, 1e-9f);
  t1 = clock64();
  if (tid == 0) cyc[3] = t1 - t0;
  // LDS.64 pointer chase
  int idx = tid & 7;
  t0 = clock64();
  for (int i = 0; i < N; ++i) idx = ((int)sm[idx] + idx) & 511;
  t1 = clock64();
  if (tid == 0) cyc[4] = t1 - t0;
  // SHFL double chain
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) x = __shfl_xor_sync(0xffffffffu, x, 1);
  t1 = clock64();
  if (tid == 0) cyc[5] = t1 - t0;
  // syncthreads
  t0 = clock64();
  for (int i = 0; i < N; ++i) __syncthreads();
  t1 = clock64();
  if (tid == 0) cyc[6] = t1 - t0;
  // DMMA chain
  double c[4] = {0, 0, 0, 0}, a[4] = {x, x, x, x}, b[2] = {y, y};
  t0 = clock64();
  for (int i = 0; i < N; ++i)
    asm volatile("mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};\n"
                 : "+d"(c[0]), "+d"(c[1]), "+d"(c[2]), "+d"(c[3]) : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(b[0]), "d"(b[1]));
  t1 = clock64();
  if (tid == 0) cyc[7] = t1 - t0;
  // DFMA throughput with 8 independent chains in one warp
  double w[8];
  for (int k = 0; k < 8; ++k) w[k] = x + k;
  t0 = clock64();
  for (int i = 0; i < N; ++i)
#pragma unroll
    for (int k = 0; k < 8; ++k) w[k] = fma(w[k], y, z);
  t1 = clock64();
  if (tid == 0) cyc[8] = t1 - t0;
  double s = 0;
  for (int k = 0; k < 8; ++k) s += w[k];
  out[tid] = x + xf + idx + c[0] + c[1] + c[2] + c[3] + s;
}

int main() {
  double* out;
  long long* cyc;
  cudaMalloc(&out, 1024 * 8);
  cudaMalloc(&cyc, 16 * 8);
  const char* names[] = {"dfma", "dadd", "dmul", "ffma", "lds64_chase", "shfl_f64", "syncthreads_256", "dmma_m16n8k8",
                         "dfma_8chains_per_iter"};
  for (int threads : {32, 256}) {
    lat_kernel<<<1, threads>>>(out, cyc, 1.0);
    cudaDeviceSynchronize();
    long long h[16];
    cudaMemcpy(h, cyc, sizeof h, cudaMemcpyDeviceToHost);
    for (int i = 0; i < 9; ++i)
      printf("{\"threads\": %d, \"op\": \"%s\", \"cycles_per_op\": %.2f}\n", threads, names[i], (double)h[i] / N);
  }
  return 0;
}
