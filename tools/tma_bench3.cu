// TMA streaming microbenchmark (B200), for the slab convolution's operand streams
// (DESIGN.md sec 5): bytes/cycle/SM delivered into shared memory by one issuing thread per CTA
// (one CTA per SM) for a ring of S stages of 2D SWIZZLE_128B boxes {64 bf16, rows}, when
//   shared:   every CTA streams the same 1 MB region in the same order (a weight operand B),
//   stagger:  the same region, each CTA starting at a different offset,
//   distinct: each CTA streams its own region (an activation slab; total 148 MB, DRAM + L2).
// Also the latency of one box with nothing else in flight, and (second table) what sets the
// ~310-cycle per-box cost: tensor-map prefetch, issuing threads per SM, box shape, plain bulk copy.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/tma_bench3 tools/tma_bench3.cu -lcuda
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

// rows_total: rows of the region each CTA walks; region_rows_base: first row of this CTA's walk
__global__ void __launch_bounds__(128, 1) stream_kernel(const __grid_constant__ CUtensorMap tm, int stages, int box_rows,
                                                      int iters, int region_rows, int mode, unsigned long long* cycles,
                                                      int variant = 0, const uint8_t* gsrc = nullptr) {
  // variant bit0: prefetch.tensormap; bit1: two issuing warps (each its own ring half);
  // bit2: 3D box {64, box_rows/2, 2} view; bit3: plain cp.async.bulk (no tensor map)
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem_base = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bars_all[8 * 32];
  // bit4: the issuing threads are lanes 0..nw-1 of warp 0 (not lane 0 of warps 0..nw-1);
  // bits 5-6: nw = 4 / 8 issuing threads
  const int nw = (variant & 64) ? 8 : (variant & 32) ? 4 : (variant & 2) ? 2 : 1;
  const int w = (variant & 16) ? threadIdx.x : threadIdx.x / 32;
  if ((variant & 16) ? threadIdx.x >= nw : (threadIdx.x % 32 != 0 || w >= nw)) return;
  uint64_t* bars = bars_all + 32 * w;
  uint8_t* smem = smem_base + w * stages * box_rows * 128;
  if (variant & 1) asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tm) : "memory");
  for (int s = 0; s < stages; ++s)
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[s])) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  const int box_bytes = box_rows * 128;
  const int nbox = region_rows / box_rows;
  int b = mode == 1 ? (int)(blockIdx.x * 7) % nbox : 0;
  const int base = mode == 2 ? (int)blockIdx.x * region_rows : 0;
  b = (b + w * nbox / nw) % nbox;
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    const int s = it % stages;
    const uint32_t bar = smem_u32(&bars[s]);
    if (it >= stages) mbar_wait(bar, ((it / stages) - 1) & 1);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(box_bytes) : "memory");
    const uint32_t dst = smem_u32(smem + s * box_bytes);
    if (variant & 8)
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   ::"r"(dst), "l"(gsrc + (size_t)(base + b * box_rows) * 128), "r"(box_bytes), "r"(bar) : "memory");
    else if (variant & 4)
      asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];"
                   ::"r"(dst), "l"((uint64_t)&tm), "r"(bar), "r"(0), "r"(0), "r"((base + b * box_rows) / (box_rows / 2)) : "memory");
    else
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                   ::"r"(dst), "l"((uint64_t)&tm), "r"(bar), "r"(0), "r"(base + b * box_rows) : "memory");
    if (++b == nbox) b = 0;
  }
  for (int it = iters - stages; it < iters; ++it) mbar_wait(smem_u32(&bars[it % stages]), (it / stages) & 1);
  if (w == 0) cycles[blockIdx.x] = clock64() - t0;
}

typedef CUresult (*EncTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  void* pt = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &pt, cudaEnableDefault, &q));
  EncTiled enc = (EncTiled)pt;
  const size_t rows_all = 148 * 8192;  // 148 regions of 1 MB (8192 rows of 128 B)
  void* buf;
  CK(cudaMalloc(&buf, rows_all * 128));
  CK(cudaMemset(buf, 0, rows_all * 128));
  unsigned long long* cyc;
  CK(cudaMalloc(&cyc, 148 * sizeof(unsigned long long)));
  CK(cudaFuncSetAttribute(stream_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024));
  const char* mname[3] = {"shared", "stagger", "distinct"};
  for (int box_rows : {64, 128, 256}) {
    CUtensorMap tm;
    cuuint64_t d[2] = {64, rows_all}, s[1] = {128};
    cuuint32_t bx[2] = {64, (cuuint32_t)box_rows}, e[2] = {1, 1};
    if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, d, s, bx, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      printf("encode failed\n");
      return 1;
    }
    const int box_bytes = box_rows * 128;
    for (int mode = 0; mode < 3; ++mode)
      for (int stages : {1, 2, 4, 8, 12, 16, 24}) {
        if (stages * box_bytes > 200 * 1024) continue;
        const int iters = stages == 1 ? 400 : 3000;
        unsigned long long h[148];
        double avg = 0;
        for (int rep = 0; rep < 2; ++rep) {
          stream_kernel<<<148, 32, stages * box_bytes + 1024>>>(tm, stages, box_rows, iters, 8192, mode, cyc);
          CK(cudaDeviceSynchronize());
        }
        CK(cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost));
        for (int i = 0; i < 148; ++i) avg += h[i];
        avg /= 148;
        printf("box %3d rows (%5d B) %-8s stages %2d (%6d B in flight): %6.1f B/cyc/SM  %7.0f cyc/box\n", box_rows,
               box_bytes, mname[mode], stages, stages * box_bytes, (double)box_bytes * iters / avg, avg / iters);
      }
  }
  // second table: what sets the per-box cost (shared region, 8 stages per issuing warp)
  const char* vname[10] = {"plain", "prefetch", "2 warps", "2 warps+prefetch", "3D {64,r/2,2}", "bulk copy",
                           "2 lanes of 1 warp", "4 warps", "4 lanes of 1 warp", "8 lanes of 1 warp"};
  const int vbits[10] = {0, 1, 2, 3, 4, 8, 2 | 16, 32, 32 | 16, 64 | 16};
  for (int box_rows : {32, 64, 128}) {
    CUtensorMap tm2, tm3;
    cuuint64_t d[2] = {64, rows_all}, s2[1] = {128};
    cuuint32_t bx[2] = {64, (cuuint32_t)box_rows}, e[2] = {1, 1};
    enc(&tm2, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, d, s2, bx, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    cuuint64_t d3[3] = {64, (cuuint64_t)box_rows / 2, rows_all / (box_rows / 2)}, s3[2] = {128, (cuuint64_t)box_rows / 2 * 128};
    cuuint32_t b3[3] = {64, (cuuint32_t)box_rows / 2, 2}, e3[3] = {1, 1, 1};
    enc(&tm3, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, buf, d3, s3, b3, e3, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    for (int vi = 0; vi < 10; ++vi) {
      const int v = vbits[vi], stages = (v & 64) ? 4 : 8, iters = 3000;
      const int nw = (v & 64) ? 8 : (v & 32) ? 4 : (v & 2) ? 2 : 1;
      if (nw * stages * box_rows * 128 > 200 * 1024) continue;
      unsigned long long h[148];
      for (int rep = 0; rep < 2; ++rep) {
        stream_kernel<<<148, 128, nw * stages * box_rows * 128 + 1024>>>((v & 4) ? tm3 : tm2, stages, box_rows, iters, 8192, 0,
                                                                        cyc, v, (const uint8_t*)buf);
        CK(cudaDeviceSynchronize());
      }
      CK(cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost));
      double avg = 0;
      for (int i = 0; i < 148; ++i) avg += h[i];
      avg /= 148;
      printf("box %3d rows shared, 8 stages/warp, %-18s: %6.1f B/cyc/SM  %5.0f cyc/box/warp\n", box_rows, vname[vi],
             (double)box_rows * 128 * iters * nw / avg, avg / iters);
    }
  }
  return 0;
}
