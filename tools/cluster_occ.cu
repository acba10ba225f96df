// How many thread-block clusters of a given size can be co-resident on this GPU (one CTA per SM:
// ~211 KB of shared memory), and the measured time of an empty cluster kernel grid.
// usage: tools/cluster_occ
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k(int* o) {
  extern __shared__ int s[];
  s[threadIdx.x] = threadIdx.x;
  __syncthreads();
  if (s[0] == 12345) o[0] = 1;
}
int main() {
  int* o;
  cudaMalloc(&o, 4);
  const int smem = 211 * 1024;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  for (int cl = 1; cl <= 16; cl *= 2) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(cl * 64);
    cfg.blockDim = dim3(320);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute a[1];
    a[0].id = cudaLaunchAttributeClusterDimension;
    a[0].val.clusterDim.x = cl;
    a[0].val.clusterDim.y = 1;
    a[0].val.clusterDim.z = 1;
    cfg.attrs = a;
    cfg.numAttrs = 1;
    int n = -1;
    cudaError_t e = cudaOccupancyMaxActiveClusters(&n, (void*)k, &cfg);
    printf("cluster %2d: max active clusters %d (%d CTAs) %s\n", cl, n, n * cl, cudaGetErrorString(e));
  }
  return 0;
}
