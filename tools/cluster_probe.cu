// Probe: max co-resident clusters for a 256-thread, 1-CTA/SM kernel (test-side tool).
#include <cstdio>
#include <cuda_runtime.h>
__global__ void __launch_bounds__(256, 1) k(double* p) { if (p) p[threadIdx.x] = 0; }
int main() {
  for (int cs : {2, 4, 8, 16}) {
    for (int smem : {8 * 1024, 100 * 1024, 200 * 1024}) {
      cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      if (cs == 16) cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
      cudaLaunchConfig_t q = {};
      q.gridDim = dim3(cs * 64); q.blockDim = dim3(256); q.dynamicSmemBytes = smem;
      cudaLaunchAttribute a[1]; a[0].id = cudaLaunchAttributeClusterDimension;
      a[0].val.clusterDim.x = cs; a[0].val.clusterDim.y = 1; a[0].val.clusterDim.z = 1;
      q.attrs = a; q.numAttrs = 1;
      int nc = -1; cudaError_t e = cudaOccupancyMaxActiveClusters(&nc, k, &q);
      printf("{\"cluster\": %d, \"smem_kb\": %d, \"max_active_clusters\": %d, \"ctas\": %d, \"err\": \"%s\"}\n", cs, smem / 1024, nc, nc * cs, cudaGetErrorName(e));
    }
  }
}
