// tcgen05.mma throughput when the operands stream through distinct shared-memory stages
// (as in a real pipeline), optionally with concurrent TMA-like smem writes by other warps.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/mma_bench2 tools/mma_bench2.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) | ((uint64_t)1 << 46) |
         ((uint64_t)2 << 61);
}

template <int N>
__global__ void __launch_bounds__(256, 1) kern(int nstages, int iters, int writers, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar;
  __shared__ uint32_t tslot;
  __shared__ volatile int stop;
  const int warp = threadIdx.x / 32;
  const int stage_bytes = 16384 + N * 128;
  for (int i = threadIdx.x; i < nstages * stage_bytes / 4; i += blockDim.x) ((uint32_t*)smem)[i] = 0x3c003c00u;
  if (threadIdx.x == 0) {
    stop = 0;
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(smem_u32(&tslot)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tslot;
  if (threadIdx.x == 0) {
    const uint32_t idesc = (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const int st = (i / 4) % nstages;
      const uint32_t base = smem_u32(smem + st * stage_bytes);
      const uint64_t a = sdesc(base) + 2 * (i & 3), b = sdesc(base + 16384) + 2 * (i & 3);
      asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
                   ::"r"(tmem), "l"(a), "l"(b), "r"(idesc), "r"(i) : "memory");
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)) : "memory");
    uint32_t done;
    do {
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(done) : "r"(smem_u32(&bar)) : "memory");
    } while (!done);
    out[blockIdx.x] = clock64() - t0;
    stop = 1;
  } else if (warp >= 4 && warp < 4 + writers) {
    // smem write traffic (16-byte stores) into a region the MMAs do not read
    uint4* w = (uint4*)(smem + nstages * stage_bytes);
    const int nvec = 8192 / 16;
    int k = threadIdx.x - 128;
    while (!stop) {
      for (int j = 0; j < 64; ++j) w[(k + j * 128) % nvec] = make_uint4(j, j, j, j);
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tmem) : "memory");
}

template <int N>
void run(int nstages, int writers) {
  unsigned long long* d;
  cudaMalloc(&d, 148 * 8);
  const int smem = nstages * (16384 + N * 128) + 8192 + 1024;
  cudaFuncSetAttribute(kern<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int iters = 20000;
  for (int rep = 0; rep < 2; ++rep) kern<N><<<148, 256, smem>>>(nstages, iters, writers, d);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return; }
  unsigned long long h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  double avg = 0;
  for (int i = 0; i < 148; ++i) avg += h[i];
  avg /= 148;
  printf("N=%3d stages=%d smem-writer-warps=%d: %6.1f cycles/MMA (ideal %5.1f)\n", N, nstages, writers, avg / iters,
         128.0 * N / 256);
  cudaFree(d);
}

int main() {
  run<64>(1, 0); run<64>(6, 0); run<64>(6, 2);
  run<128>(1, 0); run<128>(6, 0); run<128>(6, 2); run<128>(6, 4);
  run<256>(1, 0); run<256>(4, 0); run<256>(4, 2); run<256>(4, 4);
  return 0;
}
