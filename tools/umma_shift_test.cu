// Row-shifted UMMA A operand test (B200): does a K-major SWIZZLE_128B shared-memory matrix
// descriptor whose start address is s rows (s*128 B) past a 1024-B aligned tile read rows
// s..s+127 correctly, and what must the descriptor's "matrix base offset" field (bits 49-51)
// hold?  The slab convolution reads every filter tap as such a shift.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/umma_shift_test tools/umma_shift_test.cu
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

constexpr int ROWS = 256, KD = 64, N = 64, M = 128;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t base_off) {
  return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) | ((uint64_t)1 << 46) |
         ((uint64_t)(base_off & 7) << 49) | ((uint64_t)2 << 61);
}
__host__ __device__ inline float aval(int r, int k) { return (float)((r * 7 + k * 3) % 9 - 4); }
__host__ __device__ inline float bval(int n, int k) { return (float)((n * 5 + k) % 7 - 3); }

// mode 0: base offset field 0; mode 1: field = (start >> 7) & 7
__global__ void __launch_bounds__(128, 1) shift_kernel(int s, int mode, float* out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sA = smem;
  uint8_t* sB = smem + ROWS * 128;
  __shared__ uint64_t bar;
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  for (int i = threadIdx.x; i < ROWS * KD; i += blockDim.x) {
    const int r = i / KD, k = i % KD;
    *(__nv_bfloat16*)(sA + r * 128 + (((k / 8) ^ (r % 8)) * 16) + (k % 8) * 2) = __float2bfloat16(aval(r, k));
  }
  for (int i = threadIdx.x; i < N * KD; i += blockDim.x) {
    const int r = i / KD, k = i % KD;
    *(__nv_bfloat16*)(sB + r * 128 + (((k / 8) ^ (r % 8)) * 16) + (k % 8) * 2) = __float2bfloat16(bval(r, k));
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" ::"r"(smem_u32(&tslot)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tslot;
  if (threadIdx.x == 0) {
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
    const uint32_t a0 = smem_u32(sA) + s * 128;
    const uint64_t ad = sdesc(a0, mode ? (a0 >> 7) : 0), bd = sdesc(smem_u32(sB), 0);
    for (int k = 0; k < KD / 16; ++k)
      asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
                   ::"r"(tmem), "l"(ad + 2 * k), "l"(bd + 2 * k), "r"(idesc), "r"(k) : "memory");
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)) : "memory");
  }
  uint32_t done;
  do {
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(done) : "r"(smem_u32(&bar)) : "memory");
  } while (!done);
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const int row = warp * 32 + lane;
  for (int c = 0; c < N; ++c) {
    uint32_t v;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];" : "=r"(v) : "r"(tmem + ((uint32_t)(warp * 32) << 16) + c));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    out[row * N + c] = __uint_as_float(v);
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" ::"r"(tmem) : "memory");
}

int main() {
  float* d;
  cudaMalloc(&d, M * N * 4);
  const int smem = ROWS * 128 + N * 128 + 1024;
  cudaFuncSetAttribute(shift_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  static float h[M * N];
  for (int mode = 0; mode < 2; ++mode)
    for (int s = 0; s <= 13; ++s) {
      shift_kernel<<<1, 128, smem>>>(s, mode, d);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
      cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
      double maxerr = 0;
      for (int m = 0; m < M; ++m)
        for (int n = 0; n < N; ++n) {
          double ref = 0;
          for (int k = 0; k < KD; ++k) ref += aval(s + m, k) * bval(n, k);
          const double err = fabs(ref - h[m * N + n]);
          if (err > maxerr) maxerr = err;
        }
      printf("mode %d (base offset %s) shift %2d rows: max err %g %s\n", mode, mode ? "=(addr>>7)&7" : "=0", s, maxerr,
             maxerr == 0 ? "OK" : "WRONG");
    }
  return 0;
}
