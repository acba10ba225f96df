// TMA throughput microbenchmark (B200): bytes/cycle/SM delivered into shared memory by one
// producer thread per CTA for different tensor-map box shapes / modes.  Used to choose the
// conv A-operand strategy.  Build: nvcc -gencode arch=compute_100a,code=sm_100a
//   -O3 -o tools/tma_bench tools/tma_bench.cu
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <string.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t done;
  do {
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(done) : "r"(bar), "r"(parity) : "memory");
  } while (!done);
}

// mode 0: 2D tiled {c0=k, c1=row}; 1: 4D tiled {c, x, y, n}; 2: 4D im2col {c, w, h, n} + offsets
template <int STAGES>
__global__ void __launch_bounds__(32, 2) tma_kernel(const __grid_constant__ CUtensorMap tm, int mode, int iters,
                                                   int bytes, int xdim, int ydim, int ndim, int step_pixels,
                                                   unsigned long long* cycles) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bars[STAGES];
  if (threadIdx.x != 0) return;
  for (int s = 0; s < STAGES; ++s)
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[s])) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  unsigned long long t0 = clock64();
  int pix = blockIdx.x * 977;
  for (int it = 0; it < iters; ++it) {
    const int s = it % STAGES;
    const uint32_t bar = smem_u32(&bars[s]);
    if (it >= STAGES) mbar_wait(bar, ((it / STAGES) - 1) & 1);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
    const uint32_t dst = smem_u32(smem + s * 16384);
    // cheap address walk (no integer division on the issuing thread)
    int x = (it * 37) & (xdim - 1), y = (it * 13) & (ydim - 1), n = (it * 7) & 31;
    pix = x;
    if (mode == 0) {
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                   ::"r"(dst), "l"((uint64_t)&tm), "r"(bar), "r"((it * 64) & 2047), "r"((it * 131) & 2047) : "memory");
    } else if (mode == 1) {
      asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];"
                   ::"r"(dst), "l"((uint64_t)&tm), "r"(bar), "r"(0), "r"(x), "r"(y), "r"(n) : "memory");
    } else {
      const uint16_t ox = it % 3, oy = (it / 3) % 3;
      asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes"
                   " [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};"
                   ::"r"(dst), "l"((uint64_t)&tm), "r"(bar), "r"(0), "r"(x - 1), "r"(y - 1), "r"(n), "h"(ox), "h"(oy) : "memory");
    }
  }
  for (int it = iters - STAGES; it < iters; ++it) mbar_wait(smem_u32(&bars[it % STAGES]), (it / STAGES) & 1);
  cycles[blockIdx.x] = clock64() - t0;
}

typedef CUresult (*EncTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
typedef CUresult (*EncIm2col)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                              const int*, const int*, cuuint32_t, cuuint32_t, const cuuint32_t*, CUtensorMapInterleave,
                              CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static CUtensorMapSwizzle swz(int rowb) {
  return rowb >= 128 ? CU_TENSOR_MAP_SWIZZLE_128B : rowb == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
}

int main() {
  void *pt = nullptr, *pi = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &pt, cudaEnableDefault, &q));
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &pi, cudaEnableDefault, &q));
  EncTiled enc = (EncTiled)pt;
  EncIm2col enci = (EncIm2col)pi;
  const size_t bytes = (size_t)1 << 30;
  void* buf;
  CK(cudaMalloc(&buf, bytes));
  CK(cudaMemset(buf, 0, bytes));
  unsigned long long* cyc;
  CK(cudaMalloc(&cyc, 296 * sizeof(unsigned long long)));
  int smem = 6 * 16384 + 1024;
  CK(cudaFuncSetAttribute(tma_kernel<6>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  int clk_khz;
  cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);

  struct Case { const char* name; int mode; int C; int bx, by, bn; int xdim, ydim, ndim; int rowb; };
  Case cases[] = {
      {"2D tiled {64,128} rows 4KB apart (dense A)", 0, 0, 0, 0, 0, 2048, 4096, 0, 128},
      {"4D tiled C64 {64,32,1,4} (32-px runs)", 1, 64, 32, 1, 4, 64, 64, 40, 128},
      {"4D tiled C64 {64,128,1,1} (128-px run)", 1, 64, 128, 1, 1, 256, 16, 40, 128},
      {"4D tiled C64 {64,16,8,1}", 1, 64, 16, 8, 1, 64, 64, 40, 128},
      {"4D tiled C64 {64,1,1,128} (128 images)", 1, 64, 1, 1, 128, 16, 16, 160, 128},
      {"4D tiled C32 {32,64,2,1} (64B rows)", 1, 32, 64, 2, 1, 64, 64, 80, 64},
      {"4D tiled C16 {16,128,1,1} (32B rows)", 1, 16, 128, 1, 1, 128, 64, 80, 32},
      {"im2col C64 128px (128B rows)", 2, 64, 0, 0, 0, 64, 64, 40, 128},
      {"im2col C32 128px (64B rows)", 2, 32, 0, 0, 0, 64, 64, 80, 64},
      {"im2col C16 128px (32B rows)", 2, 16, 0, 0, 0, 64, 64, 160, 32},
  };
  for (const Case& c : cases) {
    CUtensorMap tm;
    CUresult r;
    int box_bytes;
    if (c.mode == 0) {
      cuuint64_t d[2] = {2048, 4096}, s[1] = {2048 * 2};
      cuuint32_t b[2] = {64, 128}, e[2] = {1, 1};
      r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, d, s, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
              CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      box_bytes = 16384;
    } else {
      cuuint64_t d[4] = {(cuuint64_t)c.C, (cuuint64_t)c.xdim, (cuuint64_t)c.ydim, (cuuint64_t)c.ndim};
      cuuint64_t s[3] = {(cuuint64_t)c.C * 2, (cuuint64_t)c.C * 2 * c.xdim, (cuuint64_t)c.C * 2 * c.xdim * c.ydim};
      cuuint32_t e[4] = {1, 1, 1, 1};
      if (c.mode == 1) {
        cuuint32_t b[4] = {(cuuint32_t)c.C, (cuuint32_t)c.bx, (cuuint32_t)c.by, (cuuint32_t)c.bn};
        r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, buf, d, s, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE, swz(c.rowb),
                CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      } else {
        int lo[2] = {-1, -1}, hi[2] = {-1, -1};
        r = enci(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, buf, d, s, lo, hi, (cuuint32_t)c.C, 128, e,
                 CU_TENSOR_MAP_INTERLEAVE_NONE, swz(c.rowb), CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                 CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      }
      box_bytes = 128 * c.C * 2;
    }
    if (r != CUDA_SUCCESS) { printf("%-46s encode failed %d\n", c.name, (int)r); continue; }
    const int iters = 4000;
    for (int rep = 0; rep < 4; ++rep) {
      const int ctas = rep < 2 ? 148 : 296;
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0); cudaEventCreate(&e1);
      cudaEventRecord(e0);
      tma_kernel<6><<<ctas, 32, smem>>>(tm, c.mode, iters, box_bytes, c.xdim, c.ydim, c.ndim > 0 ? c.ndim : 16, 128, cyc);
      cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      if (rep == 1 || rep == 3)
        printf("%-46s %s %6d B/box  %7.2f TB/s chip  %6.1f B/cyc/SM @1.9GHz\n", c.name, ctas == 148 ? "1cta/SM" : "2cta/SM",
               box_bytes, (double)box_bytes * iters * ctas / (ms * 1e-3) / 1e12,
               (double)box_bytes * iters * ctas / (ms * 1e-3) / 148 / 1.9e9);
    }
  }
  return 0;
}
