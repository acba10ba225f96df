// K1/K2/K3: tcgen05 tensor-core implicit GEMM for fully-connected, convolution and
// locally-connected layers with bias + activation fused in the epilogue.
//
// What it computes ("each neuron computes a weighted sum of its inputs";
// L65: "the learned weights are kernels that are convolved with the image"; L185:
// batching "increases the dimensions of the matrix multiplication"):
//     Y[pix(m), goff(z) + n] = act( bias[z][n] + sum_k A[m,k] * B[z][n][k] )
// with A gathered from the NHWC activations (implicit im2col) or read densely, B the
// packed weights [Z][N][Kpad] (K-major), fp32 accumulation in TMEM.
//
// Structure (Blackwell-native):
//   warps 0-3  epilogue: tcgen05.ld TMEM -> registers, +bias, activation, 16-bit/fp32 stores
//   warp  4    TMA producer: B tiles (3D tensor map, SWIZZLE_128B), dense A tiles (2D map)
//   warp  5    TMEM allocator + single-thread tcgen05.mma issuer (M=128, N=BN, K=16)
//   warps 6-9  (conv/LC) A gather producers: cp.async 16-byte chunks of 8 channels into the
//              SWIZZLE_128B K-major layout, proxy-fenced, mbarrier-signalled
// Ring of STAGES smem stages with full/empty mbarriers; tcgen05.commit frees a stage.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <stdint.h>

#include "kernels.h"

namespace djinn {
namespace {

constexpr int BM = 128, BK = 64;
constexpr int TMA_WARP = 4, MMA_WARP = 5, GATHER_WARP0 = 6;
constexpr int GATHER_THREADS = 128;
constexpr int LAG = 2;  // cp.async groups kept in flight per gather thread

template <int BN>
struct Cfg {
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES = (200 * 1024) / STAGE_BYTES > 8 ? 8 : (200 * 1024) / STAGE_BYTES;
  static constexpr int TMEM_COLS = BN < 32 ? 32 : BN;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 256;
};

// ---------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t done, iters = 0;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(bar), "r"(parity)
        : "memory");
    if (++iters > (1u << 26)) __trap();  // a lost arrival must fault, never hang the GPU
  } while (!done);
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0,
                                            int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
          dst),
      "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void tma_load_3d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0,
                                            int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(
          dst),
      "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}
__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}

// UMMA shared-memory descriptor, K-major, SWIZZLE_128B canonical layout: rows of 128 B,
// 8-row core groups 1024 B apart (SBO), LBO unused (1), version 1 (sm_100), layout 2.
__device__ __forceinline__ uint64_t sdesc_sw128(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}

// Instruction descriptor, kind::f16: D fp32, A/B fp16 (0) or bf16 (1), both K-major.
template <int BN, bool BF16>
__device__ __forceinline__ uint32_t idesc_f16() {
  const uint32_t ab = BF16 ? 1u : 0u;
  return (1u << 4) | (ab << 7) | (ab << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}

__device__ __forceinline__ void mma_f16(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                        uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accum)
      : "memory");
}
__device__ __forceinline__ void mma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar)
               : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ float act_fast(float v, int act) {
  switch (act) {
    case ACT_RELU: return v > 0.f ? v : 0.f;
    case ACT_SIGMOID: return 1.f / (1.f + __expf(-v));
    case ACT_TANH: return tanhf(v);
    case ACT_HARDTANH: return fminf(fmaxf(v, -1.f), 1.f);
    default: return v;
  }
}

template <bool BF16>
__device__ __forceinline__ uint32_t pack2(float a, float b) {
  if (BF16) {
    __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
    return *reinterpret_cast<uint32_t*>(&h);
  } else {
    __half2 h = __floats2half2_rn(a, b);
    return *reinterpret_cast<uint32_t*>(&h);
  }
}

// ---------------------------------------------------------------- the kernel
template <int BN, bool GATHER, bool BF16>
__global__ void __launch_bounds__(GATHER ? 320 : 192, 1)
    tc_gemm_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const GemmGeom g, const uint16_t* __restrict__ A, const float* __restrict__ bias,
                   void* __restrict__ Y) {
  using C = Cfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * C::A_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sB + C::STAGES * C::B_BYTES);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * C::STAGES + 1);
  const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + C::STAGES);
  const uint32_t tmem_full = smem_u32(bars + 2 * C::STAGES);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int m0 = blockIdx.x * BM, n0 = blockIdx.y * BN, z = blockIdx.z;
  const int num_kb = g.Kpad / BK;

  if (warp == TMA_WARP && lane == 0) {
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(full0 + 8 * s, GATHER ? 1 + GATHER_THREADS : 1);
      mbar_init(empty0 + 8 * s, 1);
    }
    mbar_init(tmem_full, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    fence_proxy_async();
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmB) : "memory");
    if (!GATHER) asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmA) : "memory");
  }
  if (warp == MMA_WARP) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"((uint32_t)C::TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == TMA_WARP) {
    if (lane == 0) {
      for (int kb = 0; kb < num_kb; ++kb) {
        const int s = kb % C::STAGES;
        const uint32_t ph = (kb / C::STAGES) & 1;
        mbar_wait(empty0 + 8 * s, ph ^ 1);
        mbar_arrive_expect_tx(full0 + 8 * s, C::B_BYTES + (GATHER ? 0 : C::A_BYTES));
        tma_load_3d(smem_u32(sB + s * C::B_BYTES), &tmB, full0 + 8 * s, kb * BK, n0, z);
        if (!GATHER) tma_load_2d(smem_u32(sA + s * C::A_BYTES), &tmA, full0 + 8 * s, kb * BK, m0);
      }
    }
    __syncwarp();
  } else if (warp == MMA_WARP) {
    if (lane == 0) {
      const uint32_t idesc = idesc_f16<BN, BF16>();
      for (int kb = 0; kb < num_kb; ++kb) {
        const int s = kb % C::STAGES;
        const uint32_t ph = (kb / C::STAGES) & 1;
        mbar_wait(full0 + 8 * s, ph);
        tc_fence_after();
        const uint64_t ad = sdesc_sw128(smem_u32(sA + s * C::A_BYTES));
        const uint64_t bd = sdesc_sw128(smem_u32(sB + s * C::B_BYTES));
#pragma unroll
        for (int k = 0; k < BK / 16; ++k)  // advance 16 elements = 32 B = 2 descriptor units
          mma_f16(tmem, ad + 2 * k, bd + 2 * k, idesc, (kb | k) != 0);
        mma_commit(empty0 + 8 * s);
      }
      mma_commit(tmem_full);
    }
    __syncwarp();
  } else if (GATHER && warp >= GATHER_WARP0) {
    // ---- implicit im2col producer: thread -> (chunk j, rows r0 + 16 i) ----
    const int gt = threadIdx.x - GATHER_WARP0 * 32;
    const int j = gt & 7, r0 = gt >> 3;
    int img[8], iy0[8], ix0[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int m = m0 + r0 + 16 * i;
      int im = m, oy, ox;
      if (g.mode == GM_CONV) {
        im = m / (g.OH * g.OW);
        const int rem = m - im * g.OH * g.OW;
        oy = rem / g.OW;
        ox = rem - oy * g.OW;
      } else {
        oy = z / g.OW;
        ox = z - oy * g.OW;
      }
      img[i] = im;
      iy0[i] = m < g.M ? oy * g.stride - g.pad : -(1 << 28);
      ix0[i] = ox * g.stride - g.pad;
    }
    const int CPT = g.Cgp >> 3;
    const int cin = (g.mode == GM_CONV) ? z * g.cin_goff : 0;
    const uint32_t swz = (uint32_t)((j ^ (r0 & 7)) << 4);
    const uint16_t* Ab = A + cin;
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % C::STAGES;
      const uint32_t ph = (kb / C::STAGES) & 1;
      mbar_wait(empty0 + 8 * s, ph ^ 1);
      const int q = kb * 8 + j;
      const bool kval = q * 8 < g.K;
      const int tap = q / CPT, c8 = q - tap * CPT;
      const int ky = tap / g.KW, kx = tap - ky * g.KW;
      const uint32_t dst = smem_u32(sA + s * C::A_BYTES) + swz;
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int r = r0 + 16 * i;
        const int iy = iy0[i] + ky, ix = ix0[i] + kx;
        const bool ok = kval && iy >= 0 && iy < g.H && ix >= 0 && ix < g.W;
        const uint16_t* src =
            ok ? Ab + (((int64_t)img[i] * g.H + iy) * g.W + ix) * g.Cp_in + c8 * 8 : A;
        cp_async16(dst + r * 128, src, ok ? 16u : 0u);
      }
      cp_async_commit();
      if (kb >= LAG) {
        cp_async_wait<LAG>();
        fence_proxy_async();
        mbar_arrive(full0 + 8 * ((kb - LAG) % C::STAGES));
      }
    }
    cp_async_wait<0>();
    fence_proxy_async();
    for (int kb = num_kb - LAG < 0 ? 0 : num_kb - LAG; kb < num_kb; ++kb)
      mbar_arrive(full0 + 8 * (kb % C::STAGES));
  } else if (warp < 4) {
    // ---- epilogue: TMEM -> registers -> bias + act -> global ----
    mbar_wait(tmem_full, 0);
    tc_fence_after();
    const int row = warp * 32 + lane;
    const int m = m0 + row;
    const int64_t pix = (g.mode == GM_LC) ? (int64_t)m * g.OH * g.OW + z : (int64_t)m;
    const int goff = (g.mode == GM_CONV) ? z * g.cout_goff : 0;
    const float* bz = bias + (int64_t)z * g.bias_zstride;
#pragma unroll 1
    for (int c = 0; c < BN; c += 16) {
      uint32_t r[16];
      tmem_ld16(tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)c, r);
      tmem_wait_ld();
      const int nb = n0 + c;
      if (m < g.M && nb < g.write_cols) {
        float v[16];
#pragma unroll
        for (int t = 0; t < 16; ++t) {
          const int n = nb + t;
          v[t] = n < g.N ? act_fast(__uint_as_float(r[t]) + __ldg(bz + n), g.act) : 0.f;
        }
        if (g.out_f32) {
          float* yp = reinterpret_cast<float*>(Y) + pix * g.out_pitch + goff + nb;
#pragma unroll
          for (int h = 0; h < 2; ++h)
            if (nb + 8 * h < g.write_cols) {
              reinterpret_cast<float4*>(yp + 8 * h)[0] = make_float4(v[8 * h], v[8 * h + 1], v[8 * h + 2], v[8 * h + 3]);
              reinterpret_cast<float4*>(yp + 8 * h)[1] = make_float4(v[8 * h + 4], v[8 * h + 5], v[8 * h + 6], v[8 * h + 7]);
            }
        } else {
          uint16_t* yp = reinterpret_cast<uint16_t*>(Y) + pix * g.out_pitch + goff + nb;
#pragma unroll
          for (int h = 0; h < 2; ++h)
            if (nb + 8 * h < g.write_cols)
              *reinterpret_cast<uint4*>(yp + 8 * h) =
                  make_uint4(pack2<BF16>(v[8 * h], v[8 * h + 1]), pack2<BF16>(v[8 * h + 2], v[8 * h + 3]),
                             pack2<BF16>(v[8 * h + 4], v[8 * h + 5]), pack2<BF16>(v[8 * h + 6], v[8 * h + 7]));
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == MMA_WARP) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"((uint32_t)C::TMEM_COLS)
                 : "memory");
  }
}

template <int BN, bool GATHER, bool BF16>
cudaError_t launch_inst(const GemmGeom& g, const CUtensorMap* tmA, const CUtensorMap* tmB, const void* A,
                        const float* bias, void* Y, cudaStream_t st) {
  using C = Cfg<BN>;
  static bool attr_set = false;  // benign race: idempotent attribute set
  auto kern = tc_gemm_kernel<BN, GATHER, BF16>;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  dim3 grid((g.M + BM - 1) / BM, (g.N + BN - 1) / BN, g.Z);
  kern<<<grid, GATHER ? 320 : 192, C::SMEM, st>>>(*tmA, *tmB, g, reinterpret_cast<const uint16_t*>(A), bias, Y);
  return cudaGetLastError();
}

template <bool GATHER, bool BF16>
cudaError_t launch_bn(const GemmGeom& g, int bn, const CUtensorMap* tmA, const CUtensorMap* tmB, const void* A,
                      const float* bias, void* Y, cudaStream_t st) {
  switch (bn) {
    case 16: return launch_inst<16, GATHER, BF16>(g, tmA, tmB, A, bias, Y, st);
    case 32: return launch_inst<32, GATHER, BF16>(g, tmA, tmB, A, bias, Y, st);
    case 64: return launch_inst<64, GATHER, BF16>(g, tmA, tmB, A, bias, Y, st);
    case 128: return launch_inst<128, GATHER, BF16>(g, tmA, tmB, A, bias, Y, st);
    case 256: return launch_inst<256, GATHER, BF16>(g, tmA, tmB, A, bias, Y, st);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace

int tc_pick_bn(const GemmGeom& g) {
  const int n = g.N;
  if (n <= 16) return 16;
  if (n <= 32) return 32;
  if (n <= 64) return 64;
  if (n <= 128) return 128;
  const int64_t mt = (g.M + BM - 1) / BM;
  const int64_t ctas256 = mt * ((n + 255) / 256) * g.Z;
  return ctas256 >= 2 * 148 ? 256 : 128;
}

cudaError_t launch_tc_gemm(const GemmGeom& g, int bn, int dt, const CUtensorMap* tmA, const CUtensorMap* tmB,
                           const void* A, const float* bias, void* Y, cudaStream_t st) {
  const bool gather = g.mode != GM_DENSE;
  if (dt == DT_BF16)
    return gather ? launch_bn<true, true>(g, bn, tmA, tmB, A, bias, Y, st)
                  : launch_bn<false, true>(g, bn, tmA, tmB, A, bias, Y, st);
  return gather ? launch_bn<true, false>(g, bn, tmA, tmB, A, bias, Y, st)
                : launch_bn<false, false>(g, bn, tmA, tmB, A, bias, Y, st);
}

}  // namespace djinn
