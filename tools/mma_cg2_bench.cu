// tcgen05.mma.cta_group::2 throughput (B200): cycles per kind::f16 MMA (K=16, M=256 across a
// CTA pair, both operands K-major SWIZZLE_128B in each CTA's shared memory) for a range of N,
// with the A descriptor shifted by 0 or 1 rows, and with a tcgen05.commit after every 4 MMAs
// (one pipeline stage) or only at the end.  Drives the slab convolution's tile width choice
// (DESIGN.md sec 5).  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
//   -o tools/mma_cg2_bench tools/mma_cg2_bench.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) | ((uint64_t)1 << 46) |
         ((uint64_t)2 << 61);
}
__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1)
    mma2_kernel(int N, int iters, int shift, int commit_every, int cmode, unsigned long long* out) {
  // cmode 0: multicast commit to one barrier; 1: multicast to a ring of 8 barriers;
  //       2: leader-only (non-multicast) commit to a ring of 8
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar, sbars[8];
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x / 32;
  const uint32_t rank = cluster_rank();
  for (int i = threadIdx.x; i < 65536 / 4; i += blockDim.x) ((uint32_t*)smem)[i] = 0x3c003c00u;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    for (int j = 0; j < 8; ++j) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&sbars[j])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(smem_u32(&tslot)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  cluster_sync();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tslot;
  if (rank == 0 && threadIdx.x == 0) {
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
    const uint64_t ad = sdesc(smem_u32(smem) + shift * 128), bd = sdesc(smem_u32(smem + 36864));
    unsigned long long t0 = clock64();
    // groups of commit_every MMAs (4 K-steps of one stage cycling), then a commit: no integer
    // division in the issue loop (an earlier version measured its own modulo arithmetic)
    const int ce = commit_every ? commit_every : 4;
    for (int i = 0; i < iters; i += ce) {
      for (int k = 0; k < ce; ++k) {
        const uint64_t a = ad + 2 * (k & 3), b = bd + 2 * (k & 3);
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}"
                     ::"r"(tmem), "l"(a), "l"(b), "r"(idesc), "r"(i + k) : "memory");
      }
      if (commit_every) {
        const uint32_t sb = smem_u32(&sbars[cmode == 0 ? 0 : (i / ce) & 7]);
        if (cmode == 2)
          asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sb) : "memory");
        else
          asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                       ::"r"(sb), "h"((uint16_t)3) : "memory");
      }
    }
    asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                 ::"r"(smem_u32(&bar)), "h"((uint16_t)3) : "memory");
    uint32_t done;
    do {
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(done) : "r"(smem_u32(&bar)) : "memory");
    } while (!done);
    out[blockIdx.x / 2] = clock64() - t0;
  }
  if (rank == 1 && threadIdx.x == 0) {  // wait for the leader's final commit before tearing down
    uint32_t done;
    do {
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(done) : "r"(smem_u32(&bar)) : "memory");
    } while (!done);
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  cluster_sync();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 256;" ::"r"(tmem) : "memory");
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 74 * 8);
  const int smem = 65536 + 8192 + 1024;
  cudaFuncSetAttribute(mma2_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  for (int N : {96, 128, 256})
    for (int shift : {0})
      for (int cfg = 0; cfg < 6; ++cfg) {
        const int ce = cfg == 0 ? 0 : cfg == 4 ? 8 : cfg == 5 ? 16 : 4, cmode = cfg == 2 ? 1 : cfg == 3 ? 2 : (cfg >= 4 ? 1 : 0);
        const int iters = 20000;
        for (int rep = 0; rep < 2; ++rep) mma2_kernel<<<148, 128, smem>>>(N, iters, shift, ce, cmode, d);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("N=%d: %s\n", N, cudaGetErrorString(e)); return 1; }
        unsigned long long h[74];
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < 74; ++i) avg += h[i];
        avg /= 74;
        printf("cta_group::2 M=256 N=%3d commit every %2d MMAs (%s): %7.1f cycles/MMA (ideal 128*N/256 = %5.1f)\n", N, ce,
               cmode == 0 ? "multicast, one barrier" : cmode == 1 ? "multicast, ring of 8" : "leader only, ring of 8",
               avg / iters, 128 * N / 256.0);
      }
  return 0;
}
