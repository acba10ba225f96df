// TMA streaming microbenchmark 2 (B200): the slab convolution's two operand streams together.
// One CTA per SM (148), 4 issuing warps:
//   warps 0..NB-1 stream B-like boxes {64 bf16, 64 rows} (8 KB) from ONE region shared by all
//   CTAs (weights); warp 3 streams slab-like boxes {64, 256 rows} (32 KB) from the CTA's own
//   region (activations) -- L2-resident (256 KB per CTA) or DRAM-sized (4 MB per CTA).
// Reports B/cycle/SM of each stream, alone and together; also with cta_group::2 2SM TMA in
// clusters of 2 (each CTA of the pair loads half of the B box onto the leader's barrier).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/tma_bench4 tools/tma_bench4.cu -lcuda
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

constexpr int BSTAGES = 4, SSTAGES = 3, BBOX = 8192, SBOX = 32768;

// nb: B warps (0 = none); slab: 0 none, 1 L2-resident region, 2 DRAM-sized region
__global__ void __launch_bounds__(128, 1) mix_kernel(const __grid_constant__ CUtensorMap tb, const __grid_constant__ CUtensorMap ts,
                                                    int nb, int slab, int iters, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bars[4][8];
  const int w = threadIdx.x / 32;
  if (threadIdx.x % 32) return;
  const bool is_b = w < nb, is_s = (w == 3 && slab);
  if (!is_b && !is_s) return;
  const int stages = is_b ? BSTAGES : SSTAGES, box = is_b ? BBOX : SBOX;
  uint8_t* ring = is_b ? smem + w * BSTAGES * BBOX : smem + 3 * BSTAGES * BBOX;
  for (int s = 0; s < stages; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[w][s])) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  const int region_rows = slab == 1 ? 2048 : 32768;  // 256 KB or 4 MB per CTA
  int r = is_b ? (w * 1000) % 8192 : 0;
  const int base = is_s ? (int)blockIdx.x * region_rows : 0;
  const unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    const int s = it % stages;
    const uint32_t bar = smem_u32(&bars[w][s]);
    if (it >= stages) mbar_wait(bar, ((it / stages) - 1) & 1);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(box) : "memory");
    const uint32_t dst = smem_u32(ring + s * box);
    if (is_b) {
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                   ::"r"(dst), "l"((uint64_t)&tb), "r"(bar), "r"(0), "r"(r) : "memory");
      r += 64;
      if (r >= 8192) r = 0;  // 1 MB of weights
    } else {
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                   ::"r"(dst), "l"((uint64_t)&ts), "r"(bar), "r"(0), "r"(base + r) : "memory");
      r += 256;
      if (r >= region_rows) r = 0;
    }
  }
  for (int it = iters - stages; it < iters; ++it) mbar_wait(smem_u32(&bars[w][it % stages]), (it / stages) & 1);
  out[blockIdx.x * 4 + w] = clock64() - t0;
}

typedef CUresult (*EncTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  void* pt = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &pt, cudaEnableDefault, &q));
  EncTiled enc = (EncTiled)pt;
  const size_t rows_all = (size_t)148 * 32768;
  void *wbuf, *abuf;
  CK(cudaMalloc(&wbuf, 8192 * 128));
  CK(cudaMalloc(&abuf, rows_all * 128));
  CK(cudaMemset(wbuf, 0, 8192 * 128));
  CK(cudaMemset(abuf, 0, rows_all * 128));
  CUtensorMap tb, ts;
  cuuint64_t db[2] = {64, 8192}, da[2] = {64, rows_all}, st[1] = {128};
  cuuint32_t bb[2] = {64, 64}, bs[2] = {64, 256}, e[2] = {1, 1};
  enc(&tb, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, wbuf, db, st, bb, e, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  enc(&ts, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, abuf, da, st, bs, e, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  unsigned long long* out;
  CK(cudaMalloc(&out, 148 * 4 * 8));
  const int smem = 3 * BSTAGES * BBOX + SSTAGES * SBOX + 1024;
  CK(cudaFuncSetAttribute(mix_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  struct { int nb, slab; const char* name; } cases[] = {
      {1, 0, "1 B warp"}, {2, 0, "2 B warps"}, {3, 0, "3 B warps"},
      {0, 1, "slab L2-resident"}, {0, 2, "slab DRAM"},
      {3, 1, "3 B warps + slab L2"}, {3, 2, "3 B warps + slab DRAM"}, {2, 2, "2 B warps + slab DRAM"}};
  for (auto& c : cases) {
    const int iters = 4000;
    static unsigned long long h[148 * 4];
    for (int rep = 0; rep < 2; ++rep) {
      CK(cudaMemset(out, 0, 148 * 4 * 8));
      mix_kernel<<<148, 128, smem>>>(tb, ts, c.nb, c.slab, iters, out);
      CK(cudaDeviceSynchronize());
    }
    CK(cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost));
    double bcyc = 0, scyc = 0;
    for (int i = 0; i < 148; ++i) {
      for (int w = 0; w < c.nb; ++w) bcyc += (double)h[i * 4 + w] / c.nb;
      scyc += h[i * 4 + 3];
    }
    bcyc /= 148;
    scyc /= 148;
    printf("%-24s B stream %6.1f B/cyc/SM   slab stream %6.1f B/cyc/SM\n", c.name,
           c.nb ? (double)BBOX * iters * c.nb / bcyc : 0.0, c.slab ? (double)SBOX * iters / scyc : 0.0);
  }
  return 0;
}
