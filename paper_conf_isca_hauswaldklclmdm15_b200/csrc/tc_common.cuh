// Shared device helpers of the tcgen05 kernels (k_tc.cu, k_stem.cu): PTX wrappers for
// mbarriers, TMA (tiled / im2col, CTA-pair forms), UMMA descriptors, tcgen05.mma / commit /
// ld, MUFU approximations and the fused bias + activation of a 16-column accumulator chunk.
// Included inside each translation unit's anonymous namespace (device code only).
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <stdint.h>

#include "kernels.h"

namespace djinn {
namespace {

constexpr int BM = 128, BK = 64;

// ---------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
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
    if (++iters > (1u << 28)) __trap();  // a lost arrival must fault, never hang the GPU
  } while (!done);
}
// Waiting threads suspend in the barrier until its phase completes (or the hint expires):
// spinning producers / epilogue pollers had been taking issue slots from the epilogue warps
// sharing their SM sub-partition (ncu: branch_resolving + no_inst stalls at the poll loops).
__device__ __forceinline__ void mbar_wait_sleep(uint32_t bar, uint32_t parity) {
  uint32_t done, iters = 0;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(bar), "r"(parity), "r"(0x989680u)
        : "memory");
    if (++iters > (1u << 24)) __trap();  // a lost arrival must fault, never hang the GPU
  } while (!done);
}
// Loaders' stage waits: spin (the default) -- a suspended waiter's wake-up latency was starving
// the MMA of re-armed stages; DJINN_LOADER_SLEEP builds the sleeping variant for comparison.
__device__ __forceinline__ void mbar_wait_ld(uint32_t bar, uint32_t parity) {
#ifdef DJINN_LOADER_SLEEP
  mbar_wait_sleep(bar, parity);
#else
  mbar_wait(bar, parity);
#endif
}
// Polling with a short back-off: for waiters whose stages cover many MMA cycles (slab mode's
// B-only loaders: a stage is 8-16 MMAs), so a ~100 ns late wake-up costs nothing, while a tight
// spin took 17% of the SM's issue slots from the epilogue warps (ncu, IMC conv1+norm1).
__device__ __forceinline__ void mbar_wait_backoff(uint32_t bar, uint32_t parity) {
  uint32_t done, iters = 0;
  for (;;) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(bar), "r"(parity)
        : "memory");
    if (done) break;
    if (++iters > (1u << 26)) __trap();  // a lost arrival must fault, never hang the GPU
    __nanosleep(96);
  }
}
__device__ __forceinline__ void tma_2d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
      "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void tma_3d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(
          dst),
      "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}
__device__ __forceinline__ void tma_4d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1, int c2,
                                       int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];" ::"r"(
          dst),
      "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
      : "memory");
}
// im2col mode: coordinates {c, w, h, n} = channel and the filter window's top-left input
// position of the first of the 128 output pixels; offsets {kx, ky} select the tap.
__device__ __forceinline__ void tma_im2col_4d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c, int w,
                                              int h, int n, uint16_t ox, uint16_t oy) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};" ::"r"(dst),
      "l"((uint64_t)map), "r"(bar), "r"(c), "r"(w), "r"(h), "r"(n), "h"(ox), "h"(oy)
      : "memory");
}
// ---- cta_group::2 (CTA pair) forms.  Both CTAs issue their own half of the operands; the
// transaction bytes land on the LEADER's (rank 0) barrier: its shared::cluster address is the
// local one with the peer bit (bit 24) cleared.
constexpr uint32_t PEER_MASK = 0xFEFFFFFFu;
__device__ __forceinline__ bool elect_one() {
  uint32_t p;
  asm volatile("{\n\t.reg .pred P;\n\telect.sync _|P, 0xffffffff;\n\tselp.u32 %0, 1, 0, P;\n\t}" : "=r"(p));
  return p != 0;
}
__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void tma_2d_2sm(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
      ::"r"(dst), "l"((uint64_t)map), "r"(bar & PEER_MASK), "r"(c0), "r"(c1) : "memory");
}
__device__ __forceinline__ void tma_3d_2sm(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];"
      ::"r"(dst), "l"((uint64_t)map), "r"(bar & PEER_MASK), "r"(c0), "r"(c1), "r"(c2) : "memory");
}
__device__ __forceinline__ void tma_4d_2sm(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1, int c2,
                                           int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];"
      ::"r"(dst), "l"((uint64_t)map), "r"(bar & PEER_MASK), "r"(c0), "r"(c1), "r"(c2), "r"(c3) : "memory");
}
__device__ __forceinline__ void tma_im2col_4d_2sm(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c, int w,
                                                  int h, int n, uint16_t ox, uint16_t oy) {
  asm volatile(
      "cp.async.bulk.tensor.4d.im2col.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};"
      ::"r"(dst), "l"((uint64_t)map), "r"(bar & PEER_MASK), "r"(c), "r"(w), "r"(h), "r"(n), "h"(ox), "h"(oy)
      : "memory");
}
// Relaxed arrives for the TMEM-empty handshake: TMEM reuse is ordered by tcgen05.wait::ld +
// tcgen05.fence::before_thread_sync, and no generic memory needs to be published, so the
// .release form (MEMBAR.ALL.CTA + ERRBAR: the epilogue waited for its global stores to drain,
// ~24% of stall samples) is not needed.
__device__ __forceinline__ void mbar_arrive_leader(uint32_t bar) {
  asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(bar & PEER_MASK) : "memory");
}
__device__ __forceinline__ void mbar_arrive_relaxed(uint32_t bar) {
  asm volatile("mbarrier.arrive.relaxed.cta.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
template <int CG>
__device__ __forceinline__ void tma_a2(uint32_t dst, const CUtensorMap* m, uint32_t bar, int c0, int c1) {
  if (CG == 2) tma_2d_2sm(dst, m, bar, c0, c1); else tma_2d(dst, m, bar, c0, c1);
}
template <int CG>
__device__ __forceinline__ void tma_a3(uint32_t dst, const CUtensorMap* m, uint32_t bar, int c0, int c1, int c2) {
  if (CG == 2) tma_3d_2sm(dst, m, bar, c0, c1, c2); else tma_3d(dst, m, bar, c0, c1, c2);
}
template <int CG>
__device__ __forceinline__ void tma_a4(uint32_t dst, const CUtensorMap* m, uint32_t bar, int c0, int c1, int c2, int c3) {
  if (CG == 2) tma_4d_2sm(dst, m, bar, c0, c1, c2, c3); else tma_4d(dst, m, bar, c0, c1, c2, c3);
}
template <int CG>
__device__ __forceinline__ void tma_i2c(uint32_t dst, const CUtensorMap* m, uint32_t bar, int c, int w, int h, int n,
                                        uint16_t ox, uint16_t oy) {
  if (CG == 2) tma_im2col_4d_2sm(dst, m, bar, c, w, h, n, ox, oy); else tma_im2col_4d(dst, m, bar, c, w, h, n, ox, oy);
}

__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// UMMA shared-memory descriptor of a K-major swizzled tile: rows of `row_bytes` (32/64/128),
// 8-row core groups `8*row_bytes` apart (SBO), LBO unused (1), version 1 (sm_100),
// layout type SW32 = 6, SW64 = 4, SW128 = 2.
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, int row_bytes) {
  const uint64_t layout = row_bytes == 128 ? 2 : (row_bytes == 64 ? 4 : 6);
  return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)((8 * row_bytes) >> 4) << 32) |
         ((uint64_t)1 << 46) | (layout << 61);
}

// Instruction descriptor, kind::f16: D fp32, A/B fp16 (0) or bf16 (1), both K-major, M=128.
template <int BN, bool BF16, int CG = 1>
__device__ __forceinline__ uint32_t idesc_f16() {
  const uint32_t ab = BF16 ? 1u : 0u;
  return (1u << 4) | (ab << 7) | (ab << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)((BM * CG) >> 4) << 24);
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
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mma_f16_2sm(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                            uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accum)
      : "memory");
}
// commit to the barrier at this smem offset in BOTH CTAs of the pair
__device__ __forceinline__ void mma_commit_2sm(uint32_t bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(bar),
      "h"((uint16_t)3)
      : "memory");
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ float tanh_approx(float v) {
  float r;
  asm("tanh.approx.f32 %0, %1;" : "=f"(r) : "f"(v));
  return r;
}
// Bare MUFU approximations with flush-to-zero: exp2f / __log2f / __expf / __fdividef compile to
// MUFU plus an FSETP + FMUL denormal range fixup per call (ncu, IMC conv1+norm1: the fixups were
// ~5 of the LRN epilogue's ~15 instructions per element).  Arguments here are never denormal
// where it matters (LRN: t = k + alpha/n * sum >= k; sigmoid: 1 + e^-x >= 1).
__device__ __forceinline__ float ex2_ftz(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ float lg2_ftz(float x) {
  float r;
  asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
#ifdef DJINN_LRN_POLY
// 2^y on the FMA pipe (see k_misc.cu exp2_fma): relative error <= 4.2e-5, half of the LRN's
// transcendental work moved off the MUFU.
__device__ __forceinline__ float ex2_lrn(float y) {
  y = fmaxf(y, -126.f);
  const float t = y + 12582912.f;
  const float n = t - 12582912.f;
  const float f = y - n;
  float p = fmaf(0.0096181291f, f, 0.0555041087f);
  p = fmaf(p, f, 0.2402265070f);
  p = fmaf(p, f, 0.6931471806f);
  p = fmaf(p, f, 1.0f);
  return __int_as_float(__float_as_int(p) + ((__float_as_int(t) - 0x4B400000) << 23));
}
#else
__device__ __forceinline__ float ex2_lrn(float y) { return ex2_ftz(y); }
#endif
__device__ __forceinline__ float rcp_ftz(float x) {
  float r;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ float sigmoid_fast(float v) { return rcp_ftz(1.f + ex2_ftz(-1.4426950408889634f * v)); }
// Activations on MUFU (16-bit storage tolerates their ~2^-11..2^-21 relative error).
__device__ __forceinline__ float act_fast(float v, int act) {
  switch (act) {
    case ACT_RELU: return fmaxf(v, 0.f);
    case ACT_SIGMOID: return sigmoid_fast(v);
    case ACT_TANH: return tanh_approx(v);
    case ACT_HARDTANH: return fminf(fmaxf(v, -1.f), 1.f);
    case ACT_SIGMOID_C: return sigmoid_fast(v) - 0.5f;  // sigma - 1/2 (abs. err ~1e-7)
    default: return v;
  }
}

// Bias + activation on a 16-vector: the switch is resolved once per vector, the loops are
// branch-free (the per-element runtime switch cost ~17% of issue slots in branch resolution).
__device__ __forceinline__ void bias_act16(float (&v)[16], const uint32_t (&r)[16], const float (&b)[16], int act) {
  // bias add and the sigmoid's scalings on the packed fp32 pipe (FADD2/FMUL2, bitwise equal)
#pragma unroll
  for (int j = 0; j < 16; j += 2) {
    const float2 s = add2(make_float2(__uint_as_float(r[j]), __uint_as_float(r[j + 1])), make_float2(b[j], b[j + 1]));
    v[j] = s.x;
    v[j + 1] = s.y;
  }
  switch (act) {
    case ACT_RELU:
#pragma unroll
      for (int j = 0; j < 16; ++j) v[j] = fmaxf(v[j], 0.f);
      break;
    case ACT_SIGMOID:
    case ACT_SIGMOID_C:
#pragma unroll
      for (int j = 0; j < 16; j += 2) {
        const float2 e = mul2(make_float2(v[j], v[j + 1]), make_float2(-1.4426950408889634f, -1.4426950408889634f));
        const float2 d = add2(make_float2(ex2_ftz(e.x), ex2_ftz(e.y)), make_float2(1.f, 1.f));
        float2 o = make_float2(rcp_ftz(d.x), rcp_ftz(d.y));
        if (act == ACT_SIGMOID_C) o = add2(o, make_float2(-0.5f, -0.5f));
        v[j] = o.x;
        v[j + 1] = o.y;
      }
      break;
    case ACT_TANH:
#pragma unroll
      for (int j = 0; j < 16; ++j) v[j] = tanh_approx(v[j]);
      break;
    case ACT_HARDTANH:
#pragma unroll
      for (int j = 0; j < 16; ++j) v[j] = fminf(fmaxf(v[j], -1.f), 1.f);
      break;
    default:
      break;
  }
}

__device__ __forceinline__ void lds16(float (&b)[16], const float* s) {
#pragma unroll
  for (int q = 0; q < 4; ++q) *reinterpret_cast<float4*>(b + 4 * q) = reinterpret_cast<const float4*>(s)[q];
}
__device__ __forceinline__ uint32_t pack2_f16_sat(float a, float b) {  // fp16 pair, clamped to +-65504
  __half2 h = __floats2half2_rn(fminf(fmaxf(a, -65504.f), 65504.f), fminf(fmaxf(b, -65504.f), 65504.f));
  return *reinterpret_cast<uint32_t*>(&h);
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


}  // namespace
}  // namespace djinn
