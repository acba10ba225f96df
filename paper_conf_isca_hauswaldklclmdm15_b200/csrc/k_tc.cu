// K1/K2/K3: tcgen05 tensor-core implicit GEMM for fully-connected, convolution and
// locally-connected layers, bias + activation (+ optional LRN) fused in the epilogue.
//
// What it computes ("each neuron computes a weighted sum of its inputs";
// L65: "the learned weights are kernels that are convolved with the image"; L185:
// batching "increases the dimensions of the matrix multiplication"):
//     Y[pix(m), goff(z) + n] = act( bias[z][n] + sum_k A[m,k] * B[z][n][k] )
// A = the NHWC activations seen through an implicit im2col, B = packed weights
// [Z][N][Kpad] (K-major, k = (ky, kx, c) with c fastest), fp32 accumulation in TMEM.
//
// Blackwell structure:
//   * persistent CTAs (grid <= #SMs), static tile striding; a tile = (m block of 128 rows,
//     n block of BN columns, a group of zf z-slices accumulated side by side in TMEM)
//   * warp 8: TMA producer.  A arrives in chunks of cw channels (one TMA box each):
//       conv  -> tiled 4D TMA box {cw, bx, by, bn}: the input pixels under tap (kx,ky) of
//                a bx x by x bn block of output pixels (the M tile); out-of-bounds
//                coordinates (the zero padding) are zero-filled by the TMA unit.  (im2col-
//                mode TMA was measured at ~16 B/cycle/SM on B200, tiled boxes stream >90.)
//       LC    -> tiled 4D TMA box {cw, 1, 1, 128 images} at the tap's input pixel
//       dense -> tiled 2D TMA box {64, 128 rows}
//     B arrives as a 3D tiled box {64, BN, 1}, SWIZZLE_128B.
//   * warp 9: TMEM allocator + single-thread tcgen05.mma issuer (M=128, N=BN, K=16),
//     tcgen05.commit frees smem stages and publishes finished accumulators
//   * warps 0-7: epilogue, tcgen05.ld TMEM -> registers, +bias, activation, optional
//     Caffe LRN across the pixel's channels, 16-bit / fp32 vector stores.  Warps w and w+4
//     share TMEM lane quarter w%4 and split the columns; accumulators are double-buffered
//     in TMEM so the epilogue of tile t overlaps the MMAs of tile t+1.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <stdint.h>
#include <stdlib.h>

#include "kernels.h"
#include "tc_common.cuh"
#include <atomic>
#include <algorithm>
#include <type_traits>
#define TC_MAX_DEVICES 64

#ifdef DJINN_TC_STATS
#include <cstdio>
#define STAT_T0() const unsigned long long _t0 = clock64()
#define STAT_ADD(v) (v) += clock64() - _t0
#else
#define STAT_T0()
#define STAT_ADD(v)
#endif

namespace djinn {
namespace {

// Warp roles: 0-7 epilogue, 8-11 TMA loaders, 12 TMEM allocator + MMA issuer.  A warp issues one
// TMA box per ~375 cycles however large the box (tools/tma_bench3.cu: the rate scales with the
// number of issuing warps, not with bytes), so stages are dealt round-robin to four loaders.
#ifndef DJINN_EPI_WG
#define DJINN_EPI_WG 3
#endif
// Epilogue warpgroups take tiles round robin: each has EPI_WG MMA tile-times for its tile (the
// epilogue is latency-bound, ncu: ~45 % issue-active; role timing: the MMA warp waited on TMEM
// slots 44 % of IMC conv1 with 2 warpgroups).
constexpr int EPI_WG = DJINN_EPI_WG;
constexpr int EPI_WARPS = 4 * EPI_WG, LOAD_WARP0 = EPI_WARPS, NLOAD = EPI_WG == 3 ? 3 : 4, MMA_WARP = EPI_WARPS + NLOAD,
              NUM_THREADS = 32 * (MMA_WARP + 1);

constexpr int KTAB_MAX = 256;  // im2col producer: per-K-chunk (channel, kx, ky) table entries
template <int BN, int CG = 1>
struct Cfg {
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = (BN / CG) * BK * 2;  // cta_group::2: each CTA holds half of B
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES = (200 * 1024) / STAGE_BYTES > 8 ? 8 : (200 * 1024) / STAGE_BYTES;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 512;
};

// Diagnostic builds only (tools/): DJINN_DBG_NOSTORE drops the epilogue's
// global stores, DJINN_DBG_NOEPI skips the epilogue work (TMEM slots are released at once).
#ifdef DJINN_DBG_NOEPI
constexpr bool kDbgNoEpi = true;
#else
constexpr bool kDbgNoEpi = false;
#endif
#ifdef DJINN_DBG_LDONLY
constexpr bool kDbgLdOnly = true;  // DJINN_DBG_LDONLY: plain epilogue loads TMEM, computes and stores nothing
#else
constexpr bool kDbgLdOnly = false;
#endif
#ifdef DJINN_DBG_NOB
constexpr bool kDbgNoB = true;  // DJINN_DBG_NOB: the B operand is not loaded
#else
constexpr bool kDbgNoB = false;
#endif
#ifdef DJINN_DBG_NOMMA
constexpr bool kDbgNoMma = true;  // DJINN_DBG_NOMMA: operands stream, no MMA is issued
#else
constexpr bool kDbgNoMma = false;
#endif

// 16-byte epilogue store; DJINN_ST_HINT selects the cache policy (experiment hook:
// 0 plain st.global, 1 .L1::no_allocate, 2 .cs streaming).
#ifndef DJINN_ST_HINT
#define DJINN_ST_HINT 0
#endif
__device__ __forceinline__ void st16(void* p, uint4 v) {
#if DJINN_ST_HINT == 1
  asm volatile("st.global.L1::no_allocate.v4.b32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
#elif DJINN_ST_HINT == 2
  asm volatile("st.global.cs.v4.b32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
#else
  *reinterpret_cast<uint4*>(p) = v;
#endif
}
template <bool BF16>
__device__ __forceinline__ void store16(const GemmGeom& g, void* Y, int64_t off, const float (&v)[16], int nvalid8) {
#ifdef DJINN_DBG_NOSTORE
  if (v[0] != 12345.f) return;
#endif
#ifdef DJINN_DBG_COALESCED
  {  // diagnostic (wrong results): the warp's 16-byte stores land contiguously, same byte count
    const unsigned am = __activemask();
    const int64_t b0 = __shfl_sync(am, off, __ffs(am) - 1);
    off = b0 + (off % g.out_pitch) * 32 + (threadIdx.x & 31) * 8;
  }
#endif
  if (g.out_f32) {
    float* yp = reinterpret_cast<float*>(Y) + off;
#pragma unroll
    for (int h = 0; h < 2; ++h)
      if (h < nvalid8) {
        reinterpret_cast<float4*>(yp + 8 * h)[0] = make_float4(v[8 * h], v[8 * h + 1], v[8 * h + 2], v[8 * h + 3]);
        reinterpret_cast<float4*>(yp + 8 * h)[1] = make_float4(v[8 * h + 4], v[8 * h + 5], v[8 * h + 6], v[8 * h + 7]);
      }
  } else if (BF16 && g.out_half) {
    // a bf16 net's conv output read only by the lrn+pool kernel is kept in fp16 (3 more mantissa
    // bits than bf16; the plan says "fp16-out"), saturated to the fp16 range: a value beyond
    // 65504 becomes +-65504, never inf (then NaN after LRN)
    uint16_t* yp = reinterpret_cast<uint16_t*>(Y) + off;
#pragma unroll
    for (int h = 0; h < 2; ++h)
      if (h < nvalid8)
        st16(yp + 8 * h,
             make_uint4(pack2_f16_sat(v[8 * h], v[8 * h + 1]), pack2_f16_sat(v[8 * h + 2], v[8 * h + 3]),
                        pack2_f16_sat(v[8 * h + 4], v[8 * h + 5]), pack2_f16_sat(v[8 * h + 6], v[8 * h + 7])));
  } else {
    uint16_t* yp = reinterpret_cast<uint16_t*>(Y) + off;
#pragma unroll
    for (int h = 0; h < 2; ++h)
      if (h < nvalid8)
        st16(yp + 8 * h,
             make_uint4(pack2<BF16>(v[8 * h], v[8 * h + 1]), pack2<BF16>(v[8 * h + 2], v[8 * h + 3]),
                        pack2<BF16>(v[8 * h + 4], v[8 * h + 5]), pack2<BF16>(v[8 * h + 6], v[8 * h + 7])));
  }
}

// Store a 16-channel chunk whose first LOGICAL channel is cglob, honouring the output's
// grouped layout (channel c at (c/gsz)*gpitch + c%gsz); the last chunk of a group also
// zero-fills the group's pad channels so that pads never hold stale data.
template <bool BF16>
__device__ __forceinline__ void store_chunk(const GemmGeom& g, void* Y, int64_t pixbase, int cglob,
                                            const float (&v)[16], int nvalid8) {
  const int gsz = g.out_gsz;
  if (gsz == g.out_gpitch) {  // plain layout (or groups stored back to back): no division
    store16<BF16>(g, Y, pixbase + cglob, v, nvalid8);
    return;
  }
  const int grp = cglob / gsz, cin = cglob - grp * gsz;
  const int64_t gbase = pixbase + (int64_t)grp * g.out_gpitch;
  store16<BF16>(g, Y, gbase + cin, v, nvalid8);
  if (g.out_gpitch > gsz && cin + 16 >= gsz && !g.out_f32) {
    uint16_t* yp = reinterpret_cast<uint16_t*>(Y) + gbase + gsz;
    for (int e = 0; e < g.out_gpitch - gsz; e += 8) *reinterpret_cast<uint4*>(yp + e) = make_uint4(0, 0, 0, 0);
  }
}

struct TileCoord {
  int m0, n0, z0;      // m0: first GEMM row (dense / LC); n0: column block; z0: z group
  int x0, y0, i0;      // conv: first output pixel (x, y) and image of the block
};
__device__ __forceinline__ TileCoord tile_coord(const GemmGeom& g, int t, int mt, int nt, int cg = 1) {
  TileCoord c;
  const int tm = t % mt;
  c.m0 = tm * BM * cg;
  t /= mt;
  c.n0 = (t % nt);
  c.z0 = t / nt;
  c.x0 = c.y0 = c.i0 = 0;
  if (g.mode == GM_CONV && g.a_tiled) {
    const int nbx = (g.OW + g.bx - 1) / g.bx, nby = (g.OH + g.by - 1) / g.by;
    c.x0 = (tm % nbx) * g.bx;
    c.y0 = ((tm / nbx) % nby) * g.by;
    c.i0 = (tm / (nbx * nby)) * g.bn;
  }
  return c;
}
// Broadcast lane 0's copy: the values are warp-uniform already; this tells ptxas so.
__device__ __forceinline__ int warp_uniform(int v) { return __shfl_sync(0xffffffffu, v, 0); }
__device__ __forceinline__ TileCoord warp_uniform(TileCoord c) {
  c.m0 = warp_uniform(c.m0); c.n0 = warp_uniform(c.n0); c.z0 = warp_uniform(c.z0);
  c.x0 = warp_uniform(c.x0); c.y0 = warp_uniform(c.y0); c.i0 = warp_uniform(c.i0);
  return c;
}
__device__ __forceinline__ int num_m_tiles(const GemmGeom& g, int cg = 1) {
  if (g.mode == GM_CONV && g.a_tiled)
    return ((g.OW + g.bx - 1) / g.bx) * ((g.OH + g.by - 1) / g.by) * ((g.Nimg + g.bn - 1) / g.bn);
  return (g.M + BM * cg - 1) / (BM * cg);
}

// ---------------------------------------------------------------- the kernel
template <int BN, bool BF16, int CG, bool SLAB, int KSUB = BK / 16>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    tc_gemm_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const GemmGeom g, const float* __restrict__ bias, void* __restrict__ Y) {
  using C = Cfg<BN, CG>;
  pdl_trigger();
  // cta_group::2: a CTA pair computes a (2*128) x BN tile; rank 0 (leader) issues the MMAs.
  const uint32_t rank = CG == 2 ? cluster_rank() : 0;
  const int cid = blockIdx.x / CG, ncl = gridDim.x / CG;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  // non-slab: [A ring][B ring][bars];  slab: [B ring][2 slabs][bars]
  const int NST = SLAB ? g.stages : C::STAGES;  // ring stages
  // slab mode: a stage holds KPS consecutive K blocks of B (one commit per KPS*4 MMAs: a
  // tcgen05.commit costs ~400 cycles of pipe time, tools/mma_cg2_bench.cu)
  const int KPS = SLAB ? g.kps : 1;
  const int SB_BYTES = KPS * C::B_BYTES;  // bytes of one ring stage of B
  const uint32_t slab_chunk = SLAB ? (uint32_t)(g.slab_parts * g.slab_rows * 128) : 0u;  // one 64-channel chunk
  const uint32_t slab_bytes = SLAB ? (uint32_t)(g.zf * (g.Cgp / 64)) * slab_chunk : 0u;
  uint8_t* sA = smem;
  uint8_t* sB = SLAB ? smem : smem + C::STAGES * C::A_BYTES;
  uint8_t* sSlab = smem + ((NST * SB_BYTES + 1023) & ~1023);
  uint64_t* bars = SLAB ? reinterpret_cast<uint64_t*>(sSlab + 2 * slab_bytes)
                        : reinterpret_cast<uint64_t*>(sB + C::STAGES * C::B_BYTES);
  // bars: full[NST], empty[NST], tfull[4], tempty[4], sfull[2], sempty[2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * NST + 12);
  __shared__ uint32_t ktab[KTAB_MAX];
  // per-epilogue-warp bias of the tile being drained, indexed by TMEM column (LRN path: by channel)
  // (one double-buffered table per warpgroup: 6 KB, so the slab ring keeps its stages)
  __shared__ __align__(16) float sbias[EPI_WG][2][256];
  const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + NST);
  const uint32_t tfull0 = smem_u32(bars + 2 * NST), tempty0 = smem_u32(bars + 2 * NST + 4);
  const uint32_t sfull0 = smem_u32(bars + 2 * NST + 8), sempty0 = smem_u32(bars + 2 * NST + 10);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int num_kb = g.ksplit > 1 ? g.kpb : g.Kpad / BK;  // K blocks per tile (split-K: per split)
#ifdef DJINN_TC_STATS
  unsigned long long st_prod_wait = 0, st_prod_issue = 0, st_mma_full = 0, st_mma_tempty = 0, st_mma_issue = 0, st_epi_wait = 0,
                     st_epi_work = 0;
  const unsigned long long st_begin = clock64();
#endif
  const int mt = num_m_tiles(g, CG), nt = (g.N + BN - 1) / BN, zt = g.Z / g.zf;
  const int tiles = mt * nt * zt;
  int slot_cols = 32;  // TMEM columns per accumulator slot (power of two >= zf*BN)
  while (slot_cols < g.zf * BN) slot_cols <<= 1;
  // Accumulator slots.  Every slot is drained by ONE warpgroup (slot = lt % nslots, warpgroup =
  // lt % nwg with nwg dividing nslots), so its tfull / tempty phases are awaited in order and
  // a parity wait can never alias a phase two uses ahead.  nwg = 3 (g.epi_wg, LRN epilogues):
  // 3 slots when they fit (zf * BN <= 128).  nwg = 2: 4 slots when they fit (the MMA may run
  // 3 tiles ahead; IMC conv1: the epilogue's latency had stalled the MMA).  Otherwise 2 slots
  // drained by warpgroups 0-1.  g.tslots = 2 forces two.
  const int wg_req = (EPI_WG == 3 && g.epi_wg == 3) ? 3 : 2;
  const int nslots = g.tslots == 2 || 3 * slot_cols > 512 ? 2 : (wg_req == 3 ? 3 : 4);
  const int nwg = nslots == 3 ? 3 : 2;
  int tcols = 32;
  while (tcols < nslots * slot_cols) tcols <<= 1;

  if (warp == LOAD_WARP0 && lane == 0) {
    // (barriers are initialised before the __syncthreads below; every other role starts after it)
    for (int s = 0; s < NST; ++s) {
      mbar_init(full0 + 8 * s, 1);
      mbar_init(empty0 + 8 * s, 1);
    }
    for (int s = 0; s < 4; ++s) {
      mbar_init(tfull0 + 8 * s, 1);
      mbar_init(tempty0 + 8 * s, 4 * CG);  // one warpgroup per tile; leader's: both CTAs'
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(sfull0 + 8 * s, 1);
      mbar_init(sempty0 + 8 * s, 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    fence_proxy_async();
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmB) : "memory");
  }
  if (warp == MMA_WARP) {
    if (CG == 2) {
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                   "r"((uint32_t)tcols)
                   : "memory");
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    } else {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                   "r"((uint32_t)tcols)
                   : "memory");
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
  }
  tc_fence_before();
  __syncthreads();
  if (CG == 2) cluster_sync();  // peer barriers initialised before any remote arrive / TMA tx
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();  // the previous kernel of the stream has completed: its output is visible

  if (warp >= LOAD_WARP0 && warp < LOAD_WARP0 + NLOAD) {
    // TMA loaders.  Each loader warp runs the whole loop (warp-uniform values stay in uniform
    // registers, (ky, kx, c) of each K chunk advance by counters: no division) and one elected
    // lane issues the stages it owns: stage q belongs to loader q % NLOAD, which loads its A
    // chunk(s) and B box and arms its barrier; in slab mode loader 0 loads the per-tile slabs
    // and the (B-only) stages go round-robin to loaders 1..NLOAD-1.
    const int li = warp - LOAD_WARP0;
    const int cw = g.cw, cbytes = BM * cw * 2;
    const int chunks_per_kb = BK / cw;
    const int nchunks_k = g.K / cw;  // valid chunks along K
    const int oy_per = g.OH * g.OWb;
    const int mode = g.mode, a_tiled = g.a_tiled, lcg = g.lcg, kwp = g.kwp, KW = g.KW, Cgp = g.Cgp, kxs = g.kxs;
    const int Cp_in = g.Cp_in, zf = g.zf;
    const uint32_t sA0 = smem_u32(sA), sB0 = smem_u32(sB);
    const int bn_off = (int)rank * (BN / CG);
    const bool leader = elect_one();
    const uint32_t tx_bytes = CG * ((SLAB ? 0 : C::A_BYTES) + (kDbgNoB ? 0 : C::B_BYTES));
    const int nown = SLAB ? NLOAD - 1 : NLOAD, myq = SLAB ? li - 1 : li;  // stage owner index
    int s = 0, qo = 0;  // ring slot; owner of the current stage (q % nown)
    uint32_t ph = 0;
    auto load_b = [&](uint32_t fb, int kb, int n0, int z) {
      // split-K (dense): z is the K split, B has one z slice
      if (g.ksplit > 1) { kb += z * g.kpb; z = 0; }
      if (!kDbgNoB) tma_a3<CG>(sB0 + (uint32_t)s * C::B_BYTES, &tmB, fb, kb * BK, n0 * BN + bn_off, z);
    };
    auto next_stage = [&]() {
      if (++s == NST) { s = 0; ph ^= 1; }
      if (++qo == nown) qo = 0;
    };
    const int nq = num_kb * chunks_per_kb;
    if (SLAB && li == 0) {
      // one slab per tile: zf groups x (Cgp / 64) channel chunks x slab_parts boxes of
      // slab_rows input pixels starting at the tile's first virtual pixel; double-buffered
      const uint32_t slab0 = smem_u32(sSlab);
      const int nchunk = g.Cgp / 64, parts = g.slab_parts, srows = g.slab_rows, cin_goff = g.cin_goff;
      int lt = 0;
      for (int t = cid; t < tiles; t += ncl, ++lt) {
        const TileCoord tc = warp_uniform(tile_coord(g, t, mt, nt, CG));
        const int my_m0 = tc.m0 + (int)rank * BM;
        const int sb = lt & 1;
        const uint32_t use = (uint32_t)(lt >> 1);
        {
          STAT_T0();
          mbar_wait_sleep(sempty0 + 8 * sb, (use & 1) ^ 1);
          STAT_ADD(st_prod_wait);
        }
        STAT_T0();
        if (leader) {
          if (rank == 0) mbar_arrive_expect_tx(sfull0 + 8 * sb, CG * slab_bytes);
          uint32_t dst = slab0 + (uint32_t)sb * slab_bytes;
          for (int zi = 0; zi < zf; ++zi) {
            const int cbase = (tc.z0 * zf + zi) * cin_goff;
            for (int j = 0; j < nchunk; ++j)
              for (int p = 0; p < parts; ++p, dst += (uint32_t)srows * 128)
                tma_a2<CG>(dst, &tmA, sfull0 + 8 * sb, cbase + 64 * j, my_m0 + p * srows);
          }
        }
        __syncwarp();
        STAT_ADD(st_prod_issue);
      }
    } else if (SLAB) {
      // B-only stages of the slab mode: KPS K blocks (steps u = zi * num_kb + kb) per stage
      const int nsteps = zf * num_kb;
      for (int t = cid; t < tiles; t += ncl) {
        const TileCoord tc = warp_uniform(tile_coord(g, t, mt, nt, CG));
        int zi = 0, kb = 0;  // step counters
        for (int u0 = 0; u0 < nsteps; u0 += KPS) {
          const int cnt = min(KPS, nsteps - u0);
          if (qo == myq) {
            if (g.ldwait == 1) mbar_wait_backoff(empty0 + 8 * s, ph ^ 1);
            else if (g.ldwait == 2) mbar_wait_sleep(empty0 + 8 * s, ph ^ 1);
            else mbar_wait(empty0 + 8 * s, ph ^ 1);
            if (leader) {
              const uint32_t fb = full0 + 8 * s;
              if (rank == 0) mbar_arrive_expect_tx(fb, kDbgNoB ? 0u : (uint32_t)(CG * C::B_BYTES * cnt));
              int zz = zi, kk = kb;
              for (int i = 0; i < cnt; ++i) {
                if (!kDbgNoB)
                  tma_a3<CG>(sB0 + (uint32_t)(s * SB_BYTES + i * C::B_BYTES), &tmB, fb, kk * BK, tc.n0 * BN + bn_off,
                             tc.z0 * zf + zz);
                if (++kk == num_kb) { kk = 0; ++zz; }
              }
            }
            __syncwarp();
          }
          for (int i = 0; i < cnt; ++i)
            if (++kb == num_kb) { kb = 0; ++zi; }
          next_stage();
        }
      }
    } else if (mode == GM_CONV && !a_tiled && nq <= KTAB_MAX) {
      // im2col fast path: the (channel, kx, ky) of every K chunk comes from a table built
      // once, so a stage costs a handful of instructions (the issuing warp's instruction
      // latency, not the TMA unit, had bounded the operand stream: DESIGN.md sec 5).
      const int cpt = Cgp / cw;  // chunks per tap
      if (li == 0) {
        for (int qq = lane; qq < nq; qq += 32) {
          uint32_t e = 0xFFFFu;  // past the valid K: channel = Cp_in (TMA zero-fills)
          if (qq < nchunks_k) {
            const int tap = qq / cpt, kx = tap % KW, ky = tap / KW;
            e = (uint32_t)((qq - tap * cpt) * cw) | ((uint32_t)(kx * kxs) << 16) | ((uint32_t)ky << 24);
          }
          ktab[qq] = e;
        }
      }
      asm volatile("bar.sync 1, %0;" ::"n"(NLOAD * 32) : "memory");  // ktab complete for all loaders
      const int sx = g.xstep, OWb = g.OWb, st = g.stride, pd = g.pad, cin_goff = g.cin_goff;
      for (int t = cid; t < tiles; t += ncl) {
        const TileCoord tc = warp_uniform(tile_coord(g, t, mt, nt, CG));
        const int my_m0 = tc.m0 + (int)rank * BM;
        const int img = warp_uniform(my_m0 / oy_per);
        const int rem = my_m0 - img * oy_per;
        const int oy = rem / OWb;
        const int wy = warp_uniform(oy * st - pd), wx = warp_uniform((rem - oy * OWb) * sx - pd);
        for (int zi = 0; zi < zf; ++zi) {
          const int z = tc.z0 * zf + zi;
          const int cbase = z * cin_goff;
          int q = 0;
          for (int kb = 0; kb < num_kb; ++kb) {
            if (qo == myq) {
              {
                STAT_T0();
                mbar_wait_ld(empty0 + 8 * s, ph ^ 1);
                STAT_ADD(st_prod_wait);
              }
              STAT_T0();
              const uint32_t fb = full0 + 8 * s;
              const uint32_t a_dst = sA0 + (uint32_t)s * C::A_BYTES;
              if (leader) {
                if (rank == 0) mbar_arrive_expect_tx(fb, tx_bytes);
                for (int j = 0; j < chunks_per_kb; ++j) {
                  const uint32_t e = ktab[q + j];
                  const int cr = (int)(e & 0xFFFFu);
                  const int c = cr == 0xFFFF ? Cp_in : cbase + cr;
                  tma_i2c<CG>(a_dst + j * cbytes, &tmA, fb, c, wx, wy, img, (uint16_t)((e >> 16) & 0xFF), (uint16_t)(e >> 24));
                }
                load_b(fb, kb, tc.n0, z);
              }
              __syncwarp();
              STAT_ADD(st_prod_issue);
            }
            q += chunks_per_kb;
            next_stage();
          }
        }
      }
    } else
    for (int t = cid; t < tiles; t += ncl) {
      const TileCoord tc = warp_uniform(tile_coord(g, t, mt, nt, CG));
      const int my_m0 = tc.m0 + (int)rank * BM;  // this CTA's 128 rows of the pair tile
      // conv: top-left input pixel of the filter window of the tile's first output pixel
      int wx = tc.x0 * g.stride - g.pad, wy = tc.y0 * g.stride - g.pad, img = tc.i0;
      if (mode == GM_CONV && !a_tiled) {
        img = my_m0 / oy_per;
        const int rem = my_m0 - img * oy_per;
        const int oy = rem / g.OWb;
        wy = oy * g.stride - g.pad;
        wx = (rem - oy * g.OWb) * g.xstep - g.pad;
      }
      // every lane holds the same values; saying so lets ptxas use plain R2UR for the TMA
      // operands instead of an ELECT/R2UR.BROADCAST waterfall per issue
      wx = warp_uniform(wx);
      wy = warp_uniform(wy);
      img = warp_uniform(img);
      for (int zi = 0; zi < zf; ++zi) {
        const int z = tc.z0 * zf + zi;
        int lcx = 0, lcy = 0;  // LC: input pixel of the location (block)
        if (mode == GM_LC) {
          const int oy = z / g.OWb;
          lcy = warp_uniform(oy * g.stride);
          lcx = warp_uniform((z - oy * g.OWb) * g.xb * g.stride);
        }
        const int cbase = mode == GM_CONV ? z * g.cin_goff : 0;
        int cc = 0, kx = 0, ky = 0, q = 0;  // chunk counters: channel offset, tap, chunk index
        for (int kb = 0; kb < num_kb; ++kb) {
          const bool mine = qo == myq;
          const uint32_t fb = full0 + 8 * s;
          if (mine) {
            {
              STAT_T0();
              mbar_wait_ld(empty0 + 8 * s, ph ^ 1);
              STAT_ADD(st_prod_wait);
            }
            if (leader) {
              if (rank == 0) mbar_arrive_expect_tx(fb, tx_bytes);
              load_b(fb, kb, tc.n0, z);
            }
          }
          STAT_T0();
          const uint32_t a_dst = sA0 + (uint32_t)s * C::A_BYTES;
          const bool iss = mine && leader;
          if (mode == GM_DENSE) {
            if (iss) tma_a2<CG>(a_dst, &tmA, fb, (kb + (g.ksplit > 1 ? z * g.kpb : 0)) * BK, my_m0);
          } else {
            for (int j = 0; j < chunks_per_kb; ++j, ++q) {
              // past the valid K: a channel coordinate beyond the extent -> TMA zero-fills
              const int c = q < nchunks_k ? cbase + cc : Cp_in;
              const uint32_t dst = a_dst + j * cbytes;
              if (mode == GM_CONV) {
                if (a_tiled) {
                  if (iss) tma_a4<CG>(dst, &tmA, fb, c, wx + kx, wy + ky, img);
                } else if (iss) {
                  tma_i2c<CG>(dst, &tmA, fb, c, wx, wy, img, (uint16_t)(kx * kxs), (uint16_t)ky);
                }
              } else if (lcg > 1) {  // LC, lcg taps per row: 3D view {W*C, H, N}
                const int xe = q < nchunks_k ? (lcx + kx) * Cp_in : g.W * Cp_in;  // K tail: OOB
                if (iss) tma_a3<CG>(dst, &tmA, fb, xe, lcy + ky, my_m0);
              } else {  // LC: rows are images at the fixed output location z
                if (iss) tma_a4<CG>(dst, &tmA, fb, c, lcx + kx, lcy + ky, my_m0);
              }
              if (lcg > 1) {
                kx += lcg;
                if (kx >= kwp) { kx = 0; ++ky; }
              } else {
                cc += cw;
                if (cc == Cgp) {
                  cc = 0;
                  if (++kx == KW) { kx = 0; ++ky; }
                }
              }
            }
          }
          __syncwarp();
          STAT_ADD(st_prod_issue);
          next_stage();
        }
      }
    }
  } else if (warp == MMA_WARP) {
    // The whole warp runs the issue loop (warp-uniform control flow lets the compiler keep
    // descriptors and counters in uniform registers); one elected lane issues.  A single-lane
    // loop compiled to ~20 dependent instructions per MMA (ELECT/R2UR.BROADCAST waterfalls),
    // ~100 cycles -- twice the tensor core's time for an N = 96 MMA.
    if (rank == 0) {
      const uint32_t idesc = idesc_f16<BN, BF16, CG>();
      const int cw = g.mode == GM_DENSE ? 64 : g.cw, cbytes = BM * cw * 2;
      // A descriptor of stage s, step k = (desc of the stage base) + adelta[k] (16-byte units).
      uint32_t adelta[BK / 16];
#pragma unroll
      for (int k = 0; k < BK / 16; ++k) {
        const int e = k * 16;
        adelta[k] = (uint32_t)(((e / cw) * cbytes + (e % cw) * 2) >> 4);
      }
      const uint64_t a_hi = sdesc(0, SLAB ? 128 : cw * 2), b_hi = sdesc(0, 128);
      const uint32_t sA0 = (smem_u32(sA) & 0x3FFFFu) >> 4, sB0 = (smem_u32(sB) & 0x3FFFFu) >> 4;
      // slab mode: per step u = zi * num_kb + kb, the A row offset within the slab (16-B units)
      const int nsteps = g.zf * num_kb;
      const uint32_t slab_s16 = (smem_u32(sSlab) & 0x3FFFFu) >> 4;
      if (SLAB) {
        const int nchunk = g.Cgp / 64;
        for (int u = lane; u < nsteps; u += 32) {
          const int zi = u / num_kb, kb = u - zi * num_kb, tap = kb / nchunk, j = kb - tap * nchunk;
          const int ky = tap / g.KW, kx = tap - ky * g.KW;
          const uint32_t off = (uint32_t)((zi * nchunk + j) * (int)(slab_chunk >> 4)) + (uint32_t)((ky * g.Wv + kx) * 8);
          ktab[u] = off | (kb == 0 ? (1u << 22) : 0u) | ((uint32_t)zi << 24);
        }
        __syncwarp();
      }
      int s = 0, lt = 0;
      uint32_t ph = 0;
      for (int t = cid; t < tiles; t += ncl, ++lt) {
        const int slot = lt % nslots;
        const uint32_t use = (uint32_t)(lt / nslots);
        {
          STAT_T0();
          mbar_wait_sleep(tempty0 + 8 * slot, (use & 1) ^ 1);
          STAT_ADD(st_mma_tempty);
        }
        tc_fence_after();
        if (SLAB) {
          // taps are row shifts of the tile's slab: A(tap) = slab chunk + (ky*Wv + kx) rows
          // (the 128B swizzle is address-based: a start 128*r bytes into a 1024-aligned atom
          // reads rows r.. correctly; tools/umma_shift_test.cu).  The issue loop is kept lean --
          // the tensor pipe finishes an N=96..128 MMA in 52..64 cycles, so per-stage bookkeeping
          // was idling it (tools/mma_cg2_bench.cu): the A offset / z slice of every step comes
          // from the table built below.
          const int sb = lt & 1;
          {
            STAT_T0();
            mbar_wait(sfull0 + 8 * sb, (uint32_t)(lt >> 1) & 1);
            STAT_ADD(st_mma_full);
          }
          tc_fence_after();
          const uint32_t abase = slab_s16 + (uint32_t)sb * (slab_bytes >> 4);
          const uint32_t dbase = tmem + (uint32_t)(slot * slot_cols);
          for (int u0 = 0; u0 < nsteps; u0 += KPS) {
            const int cnt = min(KPS, nsteps - u0);
            {
              STAT_T0();
              mbar_wait(full0 + 8 * s, ph);
              STAT_ADD(st_mma_full);
            }
            tc_fence_after();
            STAT_T0();
            if (elect_one()) {
              const uint32_t bstage = sB0 + (uint32_t)s * (uint32_t)(SB_BYTES >> 4);
              for (int i = 0; i < cnt; ++i) {
                const uint32_t e = ktab[u0 + i];  // bits 0-21: A offset (16 B), 22: first K step of its z, 24-31: z slice
                const uint32_t d = dbase + (e >> 24) * BN;
                const uint64_t ad = a_hi | (uint64_t)(abase + (e & 0x3FFFFFu));
                const uint64_t bd = b_hi | (uint64_t)(bstage + (uint32_t)i * (C::B_BYTES >> 4));
                const uint32_t acc0 = (e >> 22) & 1u ? 0u : 1u;
                // KSUB = 3: the K block's last 16 channels are zero padding (g.kv16)
#pragma unroll
                for (int k = 0; k < (kDbgNoMma ? 0 : KSUB); ++k) {
                  if (CG == 2) mma_f16_2sm(d, ad + 2 * k, bd + 2 * k, idesc, k ? 1u : acc0);
                  else mma_f16(d, ad + 2 * k, bd + 2 * k, idesc, k ? 1u : acc0);
                }
              }
              if (CG == 2) mma_commit_2sm(empty0 + 8 * s);
              else mma_commit(empty0 + 8 * s);
            }
            __syncwarp();
            STAT_ADD(st_mma_issue);
            if (++s == NST) { s = 0; ph ^= 1; }
          }
          if (elect_one()) {
            if (CG == 2) { mma_commit_2sm(tfull0 + 8 * slot); mma_commit_2sm(sempty0 + 8 * sb); }
            else { mma_commit(tfull0 + 8 * slot); mma_commit(sempty0 + 8 * sb); }
          }
          __syncwarp();
          continue;
        }
        for (int zi = 0; zi < g.zf; ++zi) {
          const uint32_t d = tmem + (uint32_t)(slot * slot_cols + zi * BN);
          for (int kb = 0; kb < num_kb; ++kb) {
            {
              STAT_T0();
              mbar_wait(full0 + 8 * s, ph);
              STAT_ADD(st_mma_full);
            }
            tc_fence_after();
            STAT_T0();
            if (elect_one()) {
              const uint64_t ad = a_hi | (uint64_t)(sA0 + (uint32_t)s * (C::A_BYTES >> 4));
              const uint64_t bd = b_hi | (uint64_t)(sB0 + (uint32_t)s * (C::B_BYTES >> 4));
#pragma unroll
              for (int k = 0; k < (kDbgNoMma ? 0 : BK / 16); ++k) {
                if (CG == 2) mma_f16_2sm(d, ad + adelta[k], bd + 2 * k, idesc, (kb | k) != 0);
                else mma_f16(d, ad + adelta[k], bd + 2 * k, idesc, (kb | k) != 0);
              }
              if (kDbgNoMma && CG == 1) mbar_arrive(empty0 + 8 * s);  // diagnostic: plain arrive
              else if (CG == 2) mma_commit_2sm(empty0 + 8 * s);
              else mma_commit(empty0 + 8 * s);
            }
            __syncwarp();
            STAT_ADD(st_mma_issue);
            if (++s == NST) { s = 0; ph ^= 1; }
          }
        }
        if (elect_one()) {
          if (CG == 2) mma_commit_2sm(tfull0 + 8 * slot);
          else mma_commit(tfull0 + 8 * slot);
        }
        __syncwarp();
      }
    }
  } else if (warp < EPI_WARPS) {
    // ---- epilogue (warps 0 .. EPI_WARPS-1): TMEM -> registers -> bias + act (+ LRN) -> global ----
    // The warpgroups take tiles round robin: warpgroup h drains local tiles lt with
    // lt % nwg == h (warpgroups >= nwg idle), so every thread owns one whole output row (pixel)
    // of its tile: the LRN channel window slides through registers with no halo recomputation,
    // and each warpgroup has nwg MMA tile-times for its tile.
    const int quarter = warp & 3, wg = warp >> 2;
    const uint32_t lane_base = (uint32_t)(quarter * 32) << 16;
    const int r = quarter * 32 + lane;
    int lt = 0, wtile = 0;
    for (int t = cid; t < tiles; t += ncl, ++lt) {
      if (lt % nwg != wg) continue;
      TileCoord tc = tile_coord(g, t, mt, nt, CG);
      tc.m0 += (int)rank * BM;  // this CTA's rows of the pair tile
      const int slot = lt % nslots;
      const uint32_t use = (uint32_t)(lt / nslots);
      int m;       // GEMM row (dense, LC)
      bool mok;
      // conv: output pixel (img, oy, ox) of the row (ox: first pixel of its x block) and its
      // index in the stored output (zero border obd)
      int img = 0, oy = 0, ox = 0;
      int64_t opix = 0;
      if (g.mode == GM_CONV) {
        if (g.a_tiled) {
          ox = tc.x0 + r % g.bx; oy = tc.y0 + (r / g.bx) % g.by; img = tc.i0 + r / (g.bx * g.by);
          mok = ox < g.OW && oy < g.OH && img < g.Nimg;
        } else {
          // im2col: rows enumerate (img, oy, x block) densely; slab: the stored input grid
          const int hh = SLAB ? g.Hv : g.OH, ww = SLAB ? g.Wv : g.OWb;
          const int mv = tc.m0 + r;
          img = mv / (hh * ww);
          const int rem = mv - img * (hh * ww);
          oy = rem / ww;
          const int xu = rem - oy * ww;
          ox = xu * g.xb;
          mok = img < g.Nimg && oy < g.OH && xu < g.OWb;
        }
        opix = ((int64_t)img * (g.OH + 2 * g.obd) + oy + g.obd) * (g.OW + 2 * g.obd) + ox + g.obd;
        m = (int)opix;
      } else {
        m = tc.m0 + r;
        mok = m < g.M;
      }
      // The tile's bias goes to shared memory before the wait for its accumulator: per-chunk
      // global bias loads in the drain loops had exposed an L2 round trip per 16-32 columns
      // (ncu, IMC conv1: the first FADD after each load was the top stall, ~7k cycles per tile).
      // The warpgroup's 128 threads fill one of its two tables (alternating per tile) and meet
      // at a named barrier; a warp can be at most one tile ahead of the others, so the table it
      // fills is never one that a slower warp still reads.
      float* sb = sbias[wg][wtile & 1];
      ++wtile;
      {
        const int ncols = g.zf * BN;
        for (int c = r; c < ncols; c += 128) {
          float b = 0.f;
          if (g.epi_lrn) {
            if (c < g.zf * g.N) b = __ldg(bias + c);
          } else if (g.xb > 1) {
            const int dx = c / g.out_pitch, co = c - dx * g.out_pitch;
            if (co < g.Co) b = __ldg(g.mode == GM_LC ? bias + (int64_t)tc.z0 * g.bias_zstride + dx * g.Co + co : bias + co);
          } else {
            const int zi = c / BN, nb = tc.n0 * BN + (c - zi * BN);
            if (nb < g.N && g.ksplit <= 1) b = __ldg(bias + (int64_t)(tc.z0 * g.zf + zi) * g.bias_zstride + nb);
          }
          sb[c] = b;
        }
        asm volatile("bar.sync %0, 128;" ::"r"(2 + wg) : "memory");
      }
      {
        // one lane per warp polls the barrier (256 polling threads slowed the whole SM's
        // TMA stream ~3x); the warp then reconverges
        STAT_T0();
        if (lane == 0) mbar_wait_sleep(tfull0 + 8 * slot, use & 1);
        __syncwarp();
        STAT_ADD(st_epi_wait);
      }
      tc_fence_after();
      STAT_T0();
      const uint32_t tbase = tmem + lane_base + (uint32_t)(slot * slot_cols);
      if (kDbgNoEpi) {
      } else if (g.epi_lrn) {
        // Caffe LRN across the pixel's Ctot = zf * N channels (channel zi * N + n lives in
        // column zi * BN + n).  The window [c-2, c+2] is clipped to [0, Ctot): values beyond
        // are zero, so zero-padding is exact.  Chunk i+2 is in flight from TMEM while chunk i
        // is normalised.
        const int N = g.N, Ctot = g.zf * N;
        const int nch = (Ctot + 15) / 16;
        const int64_t obase = opix * g.out_pitch;
        const float ka = g.lrn_alpha_over_n, kk = g.lrn_k, nb = -g.lrn_beta;
        int zi_n = 0, n_n = 0;  // (z slice, column) of the next chunk to load: no division
        auto issue = [&](uint32_t (&rr)[16]) {
          tmem_ld16(tbase + (uint32_t)(zi_n * BN + n_n), rr);
        };
        auto advance = [&]() {
          n_n += 16;
          if (n_n >= N) { n_n = 0; ++zi_n; }
        };
        float bq[16];  // bias of the next chunk to convert (loaded one chunk ahead)
        lds16(bq, sb);
        auto convert = [&](int i, const uint32_t (&rr)[16], float (&v)[16]) {
          const int c0 = i * 16;
          bias_act16(v, rr, bq, g.act);
          if (c0 + 16 < Ctot) lds16(bq, sb + c0 + 16);
          if (c0 + 16 > Ctot) {
#pragma unroll
            for (int j = 0; j < 16; ++j) v[j] = c0 + j < Ctot ? v[j] : 0.f;
          }
        };
        float cur[16], nxt[16];
        uint32_t rr[16];
        issue(rr);
        advance();
        tmem_wait_ld();
        convert(0, rr, cur);
        if (nch > 1) { issue(rr); advance(); }
        float pm2 = 0.f, pm1 = 0.f;
#pragma unroll 1
        for (int i = 0; i < nch; ++i) {
          if (i + 1 < nch) {
            tmem_wait_ld();
            convert(i + 1, rr, nxt);
            if (i + 2 < nch) { issue(rr); advance(); }
          } else {
#pragma unroll
            for (int j = 0; j < 16; ++j) nxt[j] = 0.f;
          }
          // Channel pairs on the packed fp32 pipe (FMUL2/FADD2/FFMA2), same operation order as
          // the scalar form s5 = (sq[j]+sq[j+1]) + (sq[j+2]+sq[j+3]) + sq[j+4]: bitwise equal.
          float sq[20];
          sq[0] = pm2;
          sq[1] = pm1;
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const float2 c2 = make_float2(cur[2 * j], cur[2 * j + 1]);
            const float2 s2 = mul2(c2, c2);
            sq[2 + 2 * j] = s2.x;
            sq[3 + 2 * j] = s2.y;
          }
          {
            const float2 n2 = make_float2(nxt[0], nxt[1]);
            const float2 s2 = mul2(n2, n2);
            sq[18] = s2.x;
            sq[19] = s2.y;
          }
          float q[18];  // q[j] = sq[j] + sq[j+1]
#pragma unroll
          for (int j = 0; j < 18; ++j) q[j] = sq[j] + sq[j + 1];
          const float2 ka2 = make_float2(ka, ka), kk2 = make_float2(kk, kk), nb2 = make_float2(nb, nb);
          float o[16];
#pragma unroll
          for (int j = 0; j < 16; j += 2) {
            const float2 s5 = add2(add2(make_float2(q[j], q[j + 1]), make_float2(q[j + 2], q[j + 3])),
                                   make_float2(sq[j + 4], sq[j + 5]));  // windows c-2 .. c+2
            const float2 c2 = make_float2(cur[j], cur[j + 1]);
#if defined(DJINN_DBG_LRN0)
            const float2 r = fma2(ka2, s5, kk2);  // diagnostic: no MUFU
#else
            const float2 t = fma2(ka2, s5, kk2);
            const float2 l = mul2(nb2, make_float2(lg2_ftz(t.x), lg2_ftz(t.y)));
            const float2 r = make_float2(ex2_lrn(l.x), ex2_lrn(l.y));
#endif
            const float2 ov = mul2(c2, r);
            o[j] = ov.x;
            o[j + 1] = ov.y;
          }
          pm2 = sq[16];
          pm1 = sq[17];
          if (mok) {
            const int c0 = i * 16;
            const int nvalid8 = min(2, (g.write_cols - c0 + 7) / 8);
            if (nvalid8 > 0) store_chunk<BF16>(g, Y, obase, c0, o, nvalid8);
          }
#pragma unroll
          for (int j = 0; j < 16; ++j) cur[j] = nxt[j];
        }
      } else if (g.xb > 1) {
        // x-blocked conv / LC: column c = dx * P + co with P = out_pitch; each 16-column chunk
        // is channels [co0, co0+16) of output pixel block*xb + dx.  Conv: row m = (img, oy,
        // block); LC: row m = image, the block is the tile's z.
        const int P = g.out_pitch, OWb = g.OWb;
        int ox0 = ox;
        int64_t pix0 = opix;  // stored index of pixel ox0
        if (g.mode == GM_LC) {
          const int ly = tc.z0 / OWb;
          ox0 = (tc.z0 - ly * OWb) * g.xb;
          pix0 = ((int64_t)m * g.OH + ly) * g.OW + ox0;
        }
        int dx = 0, co0 = 0;
#pragma unroll 1
        for (int c = 0; c < BN; c += 16) {
          float b[16];
          lds16(b, sb + c);
          uint32_t rr[16];
          tmem_ld16(tbase + (uint32_t)c, rr);
          tmem_wait_ld();
          const int oxd = ox0 + dx;
          if (mok && oxd < g.OW && c < g.N) {
            float v[16];
            bias_act16(v, rr, b, g.act);
            if (co0 + 16 > g.Co) {
#pragma unroll
              for (int j = 0; j < 16; ++j) v[j] = co0 + j < g.Co ? v[j] : 0.f;
            }
            store16<BF16>(g, Y, (pix0 + dx) * P + co0, v, 2);
          }
          co0 += 16;
          if (co0 >= P) { co0 = 0; ++dx; }
        }
      } else {
        for (int zi = 0; zi < g.zf; ++zi) {
          const int z = tc.z0 * g.zf + zi;
          const int64_t pix = (g.mode == GM_LC) ? (int64_t)m * g.OH * g.OW + z
                              : (g.mode == GM_CONV ? opix : (int64_t)m + (g.ksplit > 1 ? (int64_t)z * g.M : 0));
          const int goff = (g.mode == GM_CONV) ? z * g.cout_goff : 0;
          const int nb0 = tc.n0 * BN;
#pragma unroll 1
          for (int c = 0; c < BN; c += 32) {
            const bool two = c + 16 < BN;
            float b0[16], b1[16];
            lds16(b0, sb + zi * BN + c);
            if (two) lds16(b1, sb + zi * BN + c + 16);
            uint32_t r0[16], r1[16];
            tmem_ld16(tbase + (uint32_t)(zi * BN + c), r0);
            if (two) tmem_ld16(tbase + (uint32_t)(zi * BN + c + 16), r1);
            tmem_wait_ld();
            const int nb = nb0 + c;
            if (kDbgLdOnly) continue;
            if (mok && nb < g.write_cols) {
              float v[16];
              bias_act16(v, r0, b0, g.act);
              if (nb + 16 > g.N) {
#pragma unroll
                for (int j = 0; j < 16; ++j) v[j] = nb + j < g.N ? v[j] : 0.f;
              }
              store_chunk<BF16>(g, Y, pix * g.out_pitch, goff + nb, v, min(2, (g.write_cols - nb + 7) / 8));
            }
            if (two && mok && nb + 16 < g.write_cols) {
              float v[16];
              bias_act16(v, r1, b1, g.act);
              if (nb + 32 > g.N) {
#pragma unroll
                for (int j = 0; j < 16; ++j) v[j] = nb + 16 + j < g.N ? v[j] : 0.f;
              }
              store_chunk<BF16>(g, Y, pix * g.out_pitch, goff + nb + 16, v, min(2, (g.write_cols - nb - 16 + 7) / 8));
            }
          }
        }
      }
      STAT_ADD(st_epi_work);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        if (CG == 2) mbar_arrive_leader(tempty0 + 8 * slot);
        else mbar_arrive_relaxed(tempty0 + 8 * slot);
      }
    }
  }
#ifdef DJINN_TC_STATS
  if (blockIdx.x == 0 && (threadIdx.x == LOAD_WARP0 * 32 || threadIdx.x == MMA_WARP * 32 || threadIdx.x == 0))
    printf("[tc BN=%d mode=%d N=%d K=%d tiles=%d grid=%d] warp %d total %llu prod_wait %llu prod_issue %llu mma_full %llu "
           "mma_tempty %llu mma_issue %llu epi_wait %llu epi_work %llu\n",
           BN, g.mode, g.N, g.K, tiles, gridDim.x, warp, clock64() - st_begin, st_prod_wait, st_prod_issue, st_mma_full, st_mma_tempty,
           st_mma_issue, st_epi_wait, st_epi_work);
#endif
  tc_fence_before();
  __syncthreads();
  if (CG == 2) cluster_sync();  // no remote arrive / commit may target a finished peer
  if (warp == MMA_WARP) {
    tc_fence_after();
    if (CG == 2)
      asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"((uint32_t)tcols) : "memory");
    else
      asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"((uint32_t)tcols) : "memory");
  }
}

int g_num_sms = 0;

// dynamic shared memory of a slab-mode launch: B ring + two slabs + barriers (+ alignment slack)
constexpr int SLAB_SMEM_MAX = 227 * 1024 - 1024 - EPI_WG * 2048;  // 227 KB per block minus the static ktab and sbias
template <int BN, int CG>
int slab_smem(const GemmGeom& g, int stages) {
  using C = Cfg<BN, CG>;
  const int ring = (stages * g.kps * C::B_BYTES + 1023) & ~1023;
  const int slab = g.zf * (g.Cgp / 64) * g.slab_parts * g.slab_rows * 128;
  return 1024 + ring + 2 * slab + (2 * stages + 12) * 8 + 16;
}

template <int BN, bool BF16, int CG, bool SLAB, int KSUB = BK / 16>
cudaError_t launch_inst(const GemmGeom& g, const CUtensorMap* tmA, const CUtensorMap* tmB, const float* bias, void* Y,
                        cudaStream_t st) {
  using C = Cfg<BN, CG>;
  // The max-dynamic-smem attribute is per device context: cache it per device ordinal
  // (benign race: the attribute set is idempotent).
  static std::atomic<int> attr_set[TC_MAX_DEVICES];
  auto kern = tc_gemm_kernel<BN, BF16, CG, SLAB, KSUB>;
  const int smem = SLAB ? slab_smem<BN, CG>(g, g.stages) : C::SMEM;
  if (SLAB && (g.stages < 2 || smem > SLAB_SMEM_MAX)) return cudaErrorInvalidValue;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= TC_MAX_DEVICES) return cudaErrorInvalidDevice;
  if (attr_set[dev].load(std::memory_order_relaxed) < smem) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, SLAB ? SLAB_SMEM_MAX : C::SMEM);
    if (e != cudaSuccess) return e;
    attr_set[dev].store(SLAB ? SLAB_SMEM_MAX : C::SMEM, std::memory_order_relaxed);
  }
  const int64_t mtiles = (g.mode == GM_CONV && g.a_tiled)
                             ? (int64_t)((g.OW + g.bx - 1) / g.bx) * ((g.OH + g.by - 1) / g.by) *
                                   ((g.Nimg + g.bn - 1) / g.bn)
                             : (g.M + BM * CG - 1) / (BM * CG);
  const int64_t tiles = mtiles * ((g.N + BN - 1) / BN) * (g.Z / g.zf);
  if (g.zf * BN > 256) return cudaErrorInvalidValue;  // two TMEM accumulator slots needed
  const int max_cl = tc_num_sms() / CG;
  const int clusters = (int)(tiles < max_cl ? tiles : max_cl);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(clusters * CG);
  cfg.blockDim = dim3(NUM_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CG;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, *tmA, *tmB, g, bias, Y);
}

template <bool BF16>
cudaError_t launch_bn(const GemmGeom& g, int bn, const CUtensorMap* tmA, const CUtensorMap* tmB, const float* bias,
                      void* Y, cudaStream_t st) {
  if (g.slab) {  // slab convolutions run on CTA pairs only
    if (g.cg != 2) return cudaErrorInvalidValue;
    if (g.kv16 == 3) {
      switch (bn) {
        case 96: return launch_inst<96, BF16, 2, true, 3>(g, tmA, tmB, bias, Y, st);
        case 128: return launch_inst<128, BF16, 2, true, 3>(g, tmA, tmB, bias, Y, st);
        default: break;
      }
    }
    switch (bn) {
      case 96: return launch_inst<96, BF16, 2, true>(g, tmA, tmB, bias, Y, st);
      case 128: return launch_inst<128, BF16, 2, true>(g, tmA, tmB, bias, Y, st);
      case 192: return launch_inst<192, BF16, 2, true>(g, tmA, tmB, bias, Y, st);
      case 256: return launch_inst<256, BF16, 2, true>(g, tmA, tmB, bias, Y, st);
      default: return cudaErrorInvalidValue;
    }
  }
  if (g.cg == 2) {
    switch (bn) {
      case 96: return launch_inst<96, BF16, 2, false>(g, tmA, tmB, bias, Y, st);
      case 128: return launch_inst<128, BF16, 2, false>(g, tmA, tmB, bias, Y, st);
      case 192: return launch_inst<192, BF16, 2, false>(g, tmA, tmB, bias, Y, st);
      case 256: return launch_inst<256, BF16, 2, false>(g, tmA, tmB, bias, Y, st);
      default: return cudaErrorInvalidValue;
    }
  }
  switch (bn) {
    case 16: return launch_inst<16, BF16, 1, false>(g, tmA, tmB, bias, Y, st);
    case 32: return launch_inst<32, BF16, 1, false>(g, tmA, tmB, bias, Y, st);
    case 64: return launch_inst<64, BF16, 1, false>(g, tmA, tmB, bias, Y, st);
    case 96: return launch_inst<96, BF16, 1, false>(g, tmA, tmB, bias, Y, st);
    case 128: return launch_inst<128, BF16, 1, false>(g, tmA, tmB, bias, Y, st);
    case 192: return launch_inst<192, BF16, 1, false>(g, tmA, tmB, bias, Y, st);
    case 256: return launch_inst<256, BF16, 1, false>(g, tmA, tmB, bias, Y, st);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace

namespace {
// split-K reduction: 8 columns per thread, partial sums added in split order
template <typename T>
__global__ void splitk_reduce_kernel(const float* __restrict__ part, int S, int64_t rows, int N, int ppitch,
                                     const float* __restrict__ bias, int act, T* __restrict__ y, float* __restrict__ yf,
                                     int out_pitch, int write_cols) {
  pdl_trigger();
  pdl_wait();
  const int c8 = (write_cols + 7) / 8;
  const int64_t total = rows * c8, split = rows * (int64_t)ppitch;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t m = i / c8;
    const int n0 = (int)(i - m * c8) * 8;
    float v[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) v[j] = 0.f;
    if (n0 < N) {
      const float* p = part + m * ppitch + n0;
      for (int sidx = 0; sidx < S; ++sidx, p += split) {
        const float4 a = __ldg(reinterpret_cast<const float4*>(p)), b = __ldg(reinterpret_cast<const float4*>(p + 4));
        v[0] += a.x; v[1] += a.y; v[2] += a.z; v[3] += a.w; v[4] += b.x; v[5] += b.y; v[6] += b.z; v[7] += b.w;
      }
#pragma unroll
      for (int j = 0; j < 8; ++j) v[j] = n0 + j < N ? act_fast(v[j] + __ldg(bias + n0 + j), act) : 0.f;
    }
    if (yf) {
      float* o = yf + m * out_pitch + n0;
#pragma unroll
      for (int j = 0; j < 8; ++j)
        if (n0 + j < write_cols) o[j] = v[j];
    } else {
      *reinterpret_cast<uint4*>(y + m * out_pitch + n0) =
          make_uint4(pack2<sizeof(T) == 2 && !std::is_same<T, __half>::value>(v[0], v[1]),
                     pack2<sizeof(T) == 2 && !std::is_same<T, __half>::value>(v[2], v[3]),
                     pack2<sizeof(T) == 2 && !std::is_same<T, __half>::value>(v[4], v[5]),
                     pack2<sizeof(T) == 2 && !std::is_same<T, __half>::value>(v[6], v[7]));
    }
  }
}
}  // namespace

cudaError_t launch_splitk_reduce(const float* part, int S, int64_t rows, int N, int ppitch, const float* bias, int act,
                                 void* y, int out_pitch, int write_cols, int out_f32, int dt, cudaStream_t st) {
  if (rows <= 0) return cudaSuccess;
  if (ppitch % 8 || (!out_f32 && (out_pitch % 8 || write_cols % 8))) return cudaErrorInvalidValue;
  const int64_t total = rows * ((write_cols + 7) / 8);
  const int grid = (int)std::min<int64_t>((total + 255) / 256, 148 * 16);
  if (out_f32)
    return launch_pdl(splitk_reduce_kernel<__half>, dim3(grid), dim3(256), 0, st, part, S, rows, N, ppitch, bias, act,
                      (__half*)nullptr, (float*)y, out_pitch, write_cols);
  if (dt == DT_BF16)
    return launch_pdl(splitk_reduce_kernel<__nv_bfloat16>, dim3(grid), dim3(256), 0, st, part, S, rows, N, ppitch, bias,
                      act, (__nv_bfloat16*)y, (float*)nullptr, out_pitch, write_cols);
  return launch_pdl(splitk_reduce_kernel<__half>, dim3(grid), dim3(256), 0, st, part, S, rows, N, ppitch, bias, act,
                    (__half*)y, (float*)nullptr, out_pitch, write_cols);
}

int tc_num_sms() {
  if (!g_num_sms) {
    int dev = 0, n = 148;
    if (cudaGetDevice(&dev) == cudaSuccess && cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess)
      g_num_sms = n;
    else
      g_num_sms = 148;
  }
  return g_num_sms;
}

bool tc_slab_config(GemmGeom& g, int bn) {
  if (!g.slab || g.cg != 2 || g.Cgp % 64 || g.zf * bn > 256 || g.zf * (g.Kpad / BK) > KTAB_MAX) return false;
  // largest K blocks per stage (fewest commits) that still leaves a ring of >= 3 stages
  // (kps 1 = a commit every 4 MMAs idles the tensor pipe: im2col is then faster, e.g. IMC conv3)
  for (int kps : {4, 2}) {
    int best = 0;
    for (int st = 16; st >= 3 && !best; --st) {
      GemmGeom t = g;
      t.kps = kps;
      int smem;
      switch (bn) {
        case 96: smem = slab_smem<96, 2>(t, st); break;
        case 128: smem = slab_smem<128, 2>(t, st); break;
        case 192: smem = slab_smem<192, 2>(t, st); break;
        case 256: smem = slab_smem<256, 2>(t, st); break;
        default: return false;
      }
      if (smem <= SLAB_SMEM_MAX) best = st;
    }
    if (best) {
      g.kps = kps;
      g.stages = best;
      return true;
    }
  }
  return false;
}

int tc_pick_cg(const GemmGeom& g, int bn) {
  const char* e = getenv("DJINN_CTA_PAIR");
  if (e && e[0] == '0') return 1;
  if (bn < 96 || (g.mode == GM_CONV && g.a_tiled)) return 1;
  return 2;
}

int tc_pick_bn(const GemmGeom& g) {
  const int n = g.N;
  if (n <= 16) return 16;
  if (n <= 32) return 32;
  if (n <= 64) return 64;
  if (n <= 96) return 96;
  if (n <= 128) return 128;
  if (n <= 192) return 192;
  // wider N: the tile (192 or 256) with the least padding, ties to the larger
  // 192 only when it needs no more tiles than 256 (e.g. N = 384); otherwise bigger tiles win
  return (n + 191) / 192 <= (n + 255) / 256 ? 192 : 256;
}

cudaError_t launch_tc_gemm(const GemmGeom& g, int bn, int dt, const CUtensorMap* tmA, const CUtensorMap* tmB,
                           const float* bias, void* Y, cudaStream_t st) {
  if (g.M <= 0) return cudaSuccess;
  if (dt == DT_BF16) return launch_bn<true>(g, bn, tmA, tmB, bias, Y, st);
  return launch_bn<false>(g, bn, tmA, tmB, bias, Y, st);
}

}  // namespace djinn
