// TMA im2col throughput on the IMC conv1 operand stream (B200): the exact producer walk of
// tc_gemm_kernel (persistent tiles of 128 output pixels, 3x3 taps of a 57x57x64 NHWC bf16
// tensor after space-to-depth, 128-byte rows) with no MMA and no epilogue, for a tensor that
// fits L2 (N small) and one that streams from HBM (N=1024).  Isolates the TMA/L2 side of the
// conv1 stall.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/tma_bench2 tools/tma_bench2.cu
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t done;
  do {
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(done) : "r"(bar), "r"(parity) : "memory");
  } while (!done);
}

template <int STAGES>
__global__ void __launch_bounds__(32, 1) walk_kernel(const __grid_constant__ CUtensorMap tm, int tiles, int OW, int OH,
                                                    int taps_x, int taps_y, unsigned long long* cycles, int* bytes_out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bars[STAGES];
  if (threadIdx.x != 0) return;
  for (int s = 0; s < STAGES; ++s)
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[s])) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  unsigned long long t0 = clock64();
  int it = 0;
  const int per_img = OW * OH;
  for (int t = blockIdx.x; t < tiles; t += gridDim.x) {
    const int m0 = t * 128, img = m0 / per_img, rem = m0 - img * per_img, oy = rem / OW, ox = rem - oy * OW;
    for (int ky = 0; ky < taps_y; ++ky)
      for (int kx = 0; kx < taps_x; ++kx, ++it) {
        const int s = it % STAGES;
        const uint32_t bar = smem_u32(&bars[s]);
        if (it >= STAGES) mbar_wait(bar, ((it / STAGES) - 1) & 1);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(16384) : "memory");
        asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes"
                     " [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};"
                     ::"r"(smem_u32(smem + s * 16384)), "l"((uint64_t)&tm), "r"(bar), "r"(0), "r"(ox), "r"(oy), "r"(img),
                     "h"((uint16_t)kx), "h"((uint16_t)ky) : "memory");
      }
  }
  for (int j = it - STAGES; j < it; ++j)
    if (j >= 0) mbar_wait(smem_u32(&bars[j % STAGES]), (j / STAGES) & 1);
  cycles[blockIdx.x] = clock64() - t0;
  bytes_out[blockIdx.x] = it;
}

__global__ void fill_kernel(uint32_t* p, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    p[i] = (uint32_t)(i * 2654435761u) & 0x3f7f3f7fu;  // non-zero bf16 pairs
}


// Same walk with the tc_gemm handshake: producer waits EMPTY[s], a consumer thread (another
// warp) waits FULL[s] and arrives on EMPTY[s].  spin=1: consumer/producer poll with test_wait.
template <int STAGES>
__global__ void __launch_bounds__(352, 1) walk2_kernel(const __grid_constant__ CUtensorMap tm, int tiles, int OW, int OH,
                                                     int taps, int spin, unsigned long long* cycles) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t full[STAGES], empty[STAGES];
  __shared__ int g_done;
  if (threadIdx.x == 0) g_done = 0;
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[s])) : "memory");
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&empty[s])) : "memory");
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int per_img = OW * OH;
  unsigned long long t0 = clock64();
  if (threadIdx.x == 0) {
    int it = 0;
    for (int t = blockIdx.x; t < tiles; t += gridDim.x) {
      const int m0 = t * 128, img = m0 / per_img, rem = m0 - img * per_img, oy = rem / OW, ox = rem - oy * OW;
      for (int k = 0; k < taps * taps; ++k, ++it) {
        const int kx = k % taps, ky = k / taps;
        const int s = it % STAGES;
        const uint32_t bar = smem_u32(&full[s]);
        mbar_wait(smem_u32(&empty[s]), ((it / STAGES) & 1) ^ 1);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(16384) : "memory");
        asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes"
                     " [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};"
                     ::"r"(smem_u32(smem + s * 16384)), "l"((uint64_t)&tm), "r"(bar), "r"(0), "r"(ox), "r"(oy), "r"(img),
                     "h"((uint16_t)kx), "h"((uint16_t)ky) : "memory");
      }
    }
  } else if (threadIdx.x >= 64 && spin) {
    // idle warps polling a barrier that completes only at the end (the epilogue's tfull wait)
    __shared__ uint64_t never;
    if (threadIdx.x == 64) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&never)) : "memory");
    if (spin == 2 && (threadIdx.x & 31)) return;
    uint32_t done = 0;
    while (!done && !*(volatile int*)&g_done) {
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(done) : "r"(smem_u32(&never)), "r"(0) : "memory");
    }
  } else if (threadIdx.x == 32) {
    int it = 0;
    for (int t = blockIdx.x; t < tiles; t += gridDim.x)
      for (int k = 0; k < taps * taps; ++k, ++it) {
        const int s = it % STAGES;
        mbar_wait(smem_u32(&full[s]), (it / STAGES) & 1);
        asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[s])) : "memory");
      }
    cycles[blockIdx.x] = clock64() - t0;
    *(volatile int*)&g_done = 1;
  }
}

typedef CUresult (*EncIm2col)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                              const int*, const int*, cuuint32_t, cuuint32_t, const cuuint32_t*, CUtensorMapInterleave,
                              CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  void* pi = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &pi, cudaEnableDefault, &q));
  EncIm2col enci = (EncIm2col)pi;
  const int H = 57, W = 57, C = 64, K = 3, OH = H - K + 1, OW = W - K + 1;
  const size_t maxN = 1024;
  void* buf;
  CK(cudaMalloc(&buf, maxN * H * W * C * 2));
  CK(cudaMemset(buf, 0, maxN * H * W * C * 2));
  unsigned long long* cyc;
  int* cnt;
  CK(cudaMalloc(&cyc, 148 * 8));
  CK(cudaMalloc(&cnt, 148 * 4));
  const int smem = 12 * 16384 + 1024;
  CK(cudaFuncSetAttribute(walk_kernel<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  CK(cudaFuncSetAttribute(walk_kernel<12>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  CK(cudaFuncSetAttribute(walk_kernel<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  const int Ns[4] = {16, 128, 1024, 1024};
  for (int ni = 0; ni < 4; ++ni) {
    const int N = Ns[ni];
    if (ni == 3) {  // same walk over non-zero data
      fill_kernel<<<1024, 256>>>((uint32_t*)buf, maxN * H * W * C / 2);
      CK(cudaDeviceSynchronize());
      printf("-- non-zero data --\n");
    }
    cuuint64_t d[4] = {(cuuint64_t)C, (cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)N};
    cuuint64_t s[3] = {(cuuint64_t)C * 2, (cuuint64_t)C * 2 * W, (cuuint64_t)C * 2 * W * H};
    cuuint32_t e[4] = {1, 1, 1, 1};
    int lo[2] = {0, 0}, hi[2] = {-(K - 1), -(K - 1)};
    CUtensorMap tm;
    CUresult r = enci(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, buf, d, s, lo, hi, C, 128, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) { printf("encode failed %d\n", (int)r); return 1; }
    const int tiles = (N * OH * OW + 127) / 128;
    if (N == 1024) {
      CK(cudaFuncSetAttribute(walk2_kernel<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
      for (int rep = 0; rep < 8; ++rep) {
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0); cudaEventCreate(&e1);
        cudaEventRecord(e0);
        const int spin = rep / 2;
        if (spin < 2) {
          walk2_kernel<8><<<148, spin ? 352 : 64, smem>>>(tm, tiles, OW, OH, K, spin, cyc);
        } else {  // the library's launch: cudaLaunchKernelEx with a cluster dimension
          cudaLaunchConfig_t cfg = {};
          cfg.gridDim = dim3(148);
          cfg.blockDim = dim3(352);
          cfg.dynamicSmemBytes = smem;
          cudaLaunchAttribute attr[1];
          attr[0].id = cudaLaunchAttributeClusterDimension;
          attr[0].val.clusterDim.x = spin == 2 ? 1 : 2;
          attr[0].val.clusterDim.y = 1;
          attr[0].val.clusterDim.z = 1;
          cfg.attrs = attr;
          cfg.numAttrs = 1;
          CK(cudaLaunchKernelEx(&cfg, walk2_kernel<8>, tm, tiles, OW, OH, K, 1, cyc));
        }
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (rep & 1) printf("N=%4d handshake walk (producer/consumer) stages=8 variant=%d (0 plain, 1 +spinning warps, 2 cluster-launch dim1, 3 dim2): %8.1f us\n", N, spin, ms * 1e3);
      }
    }
    for (int stg = 0; stg < 3; ++stg)
      for (int rep = 0; rep < 2; ++rep) {
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0); cudaEventCreate(&e1);
        cudaEventRecord(e0);
        if (stg == 0) walk_kernel<4><<<148, 32, smem>>>(tm, tiles, OW, OH, K, K, cyc, cnt);
        if (stg == 1) walk_kernel<8><<<148, 32, smem>>>(tm, tiles, OW, OH, K, K, cyc, cnt);
        if (stg == 2) walk_kernel<12><<<148, 32, smem>>>(tm, tiles, OW, OH, K, K, cyc, cnt);
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        const double bytes = (double)tiles * K * K * 16384;
        if (rep == 1)
          printf("N=%4d (%6.1f MB input) stages=%2d: %8.1f us  %6.2f TB/s  %6.1f B/cyc/SM @1.9GHz\n", N,
                 N * H * W * C * 2 / 1e6, stg == 0 ? 4 : stg == 1 ? 8 : 12, ms * 1e3, bytes / (ms * 1e-3) / 1e12,
                 bytes / (ms * 1e-3) / 148 / 1.9e9);
      }
  }
  return 0;
}
