// K0 + K2 (+ K4) fused: the first layer of an image net -- a strided convolution over the fp32
// NCHW query images -- as ONE tcgen05 kernel that reads the fp32 input directly.
//
// What it computes ("the learned weights are kernels that are convolved with the
// image"; the image apps' queries are fp32 images, Table 3):
//     y[n, oy, ox, co] = act( b[co] + sum_{c, ky, kx} W[co, c, ky, kx] * x[n, c, s*oy + ky, s*ox + kx] )
// optionally followed by Caffe LRN across the co of a pixel (IMC conv1 + norm1).  The stride-F
// kernel is re-expressed by space-to-depth: pixel (ty, tx) of an Hs x Ws grid
// carries channel (dy*F + dx)*C0 + c = x[c][F*ty + dy][F*tx + dx], and the conv becomes a
// KS x KS stride-1 conv over that grid (IMC: 227^2 x 3, 11x11/4 -> 57^2 x 48, 3x3/1).
//
// Structure (B200, one CTA per tile of 128 virtual output pixels, persistent grid; CTA-local:
// a CTA pair would need cluster-scope acquire/release around the gather's generic-proxy slab
// writes, and the acquire.cluster poll compiled to an L1 invalidation per iteration that
// starved the gather -- measured 690 us vs 336 us without the gather):
//   * warps 8-15 (gather): build each tile's A slab -- the 128 + (KS-1)*Ws + KS-1 consecutive
//     space-to-depth pixels its taps read -- straight from fp32 NCHW with ordinary loads (one
//     slab row per thread, its F*F*C0 loads in flight at once), convert to 16-bit and write the
//     128B-swizzled K-major rows the UMMA descriptors expect; double-buffered.  This replaces the
//     separate pack kernel and its 16-bit s2d tensor round trip through HBM.
//   * warp 8 (also a gather warp): tcgen05.mma.cta_group::1, M = 128, N = BN (IMC: 96, 52 cycles per K = 16 step);
//     every tap is the slab shifted by ky*Ws + kx rows; B (all KS*KS K blocks of the filter
//     bank, 108 KB for IMC) is loaded ONCE by TMA and stays resident in shared memory.
//   * warps 0-7 (epilogue, 2 warpgroups): TMEM -> registers -> bias + act (+ LRN) -> 16-bit ->
//     a per-warp staging tile in swizzled shared memory (conflict-free 16-byte writes) -> TMA
//     tensor stores (cp.async.bulk.tensor) of the warp's 32 consecutive virtual pixels.  The
//     output tensor is the whole virtual Hs x Ws grid per image (IMC: 57^2 instead of 55^2
//     pixels, +7 % bytes): every warp's rows are then one contiguous box, and the consumer (the
//     MAX pool) reads the valid OH x OW corner of the stored grid.  (A 4D store of the exact
//     55^2 tensor needs a negative x for rows continuing on the next image row, which the TMA
//     unit rejects as an illegal instruction on B200.)
// Accumulators: 4 TMEM slots of 128 columns, so the MMA runs up to 3 tiles ahead of the
// epilogue.
#include "tc_common.cuh"
#include <cstdio>

namespace djinn {
namespace {

// 16 warps (4 per SM sub-partition: 128 registers per thread; a 17th warp would put 5 warps on
// one sub-partition and cap every thread at 96).  The first gather warp also allocates TMEM and
// issues the MMAs of each tile right after its own share of the tile's slab.
constexpr int ST_EPI_WARPS = 8, ST_GATHER_WARP0 = 8, ST_GATHER_WARPS = 8, ST_MMA_WARP = ST_GATHER_WARP0;
constexpr int ST_THREADS = 32 * (ST_EPI_WARPS + ST_GATHER_WARPS);
constexpr int ST_SLAB_ROWS = ST_GATHER_WARPS * 32;  // one slab row per gather thread
constexpr int ST_SLAB_BYTES = ST_SLAB_ROWS * 128;

__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, uint32_t src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"((uint64_t)map),
               "r"(src), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
#ifdef DJINN_STEM_STATS
#define SST(v) v = clock64()
#define SACC(acc, v0) acc += clock64() - v0
#else
#define SST(v)
#define SACC(acc, v0)
#endif
// barrier waits of the stem kernel: suspend-with-hint (default) or spin (DJINN_STEM_SPIN)
__device__ __forceinline__ void st_wait(uint32_t bar, uint32_t parity) {
#ifdef DJINN_STEM_SPIN
  mbar_wait(bar, parity);
#else
  mbar_wait_sleep(bar, parity);
#endif
}
__device__ __forceinline__ void sts128(uint32_t addr, uint4 v) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

template <int BN, bool BF16, int F, int C0, int KS>
__global__ void __launch_bounds__(ST_THREADS, 1)
    stem_conv_kernel(const __grid_constant__ CUtensorMap tmB, const __grid_constant__ CUtensorMap tmY0,
                     const __grid_constant__ CUtensorMap tmY1, const StemGeom g, const float* __restrict__ x,
                     const float* __restrict__ bias) {
  constexpr int KB = KS * KS;                   // K blocks: one 64-channel block per tap
  constexpr int CH = F * F * C0;                // real channels of a space-to-depth pixel
  constexpr int KSUB = (CH + 15) / 16;          // 16-channel MMA K steps per tap (IMC: 3 of 4)
  constexpr int B_BLK = BN * 128;               // bytes of one K block of B
  constexpr int NB64 = BN / 64, HAS32 = (BN % 64) == 32;
  constexpr int STG = 32 * BN * 2;              // staging bytes per epilogue warp
  constexpr int NCH = BN / 16;                  // 16-column accumulator chunks
  static_assert(CH <= 64 && CH % 8 == 0, "space-to-depth pixel must fill whole 8-channel chunks of one K block");
  static_assert(BN % 32 == 0 && BN <= 128, "tile width");

  pdl_trigger();
  const int cid = blockIdx.x, ncl = gridDim.x;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sB = smem;
  uint8_t* sSlab = sB + ((KB * B_BLK + 1023) & ~1023);
  uint8_t* sOut = sSlab + 2 * ST_SLAB_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sOut + ST_EPI_WARPS * STG);
  // bars: bfull, sfull[2], sempty[2], tfull[4], tempty[4]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 13);
  __shared__ __align__(16) float sbias[BN];
  const uint32_t bfull = smem_u32(bars), sfull0 = smem_u32(bars + 1), sempty0 = smem_u32(bars + 3);
  const uint32_t tfull0 = smem_u32(bars + 5), tempty0 = smem_u32(bars + 9);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int HW = g.Hs * g.Ws;
  const int64_t M = (int64_t)g.Nimg * HW;
  const int tiles = (int)((M + 127) / 128);

  if (warp == ST_GATHER_WARP0 && lane == 0) {
    mbar_init(bfull, 1);
    for (int s = 0; s < 2; ++s) {
      mbar_init(sfull0 + 8 * s, ST_GATHER_WARPS);  // every gather warp
      mbar_init(sempty0 + 8 * s, 1);
    }
    for (int s = 0; s < 4; ++s) {
      mbar_init(tfull0 + 8 * s, 1);
      mbar_init(tempty0 + 8 * s, 4);  // the draining warpgroup
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");  // (cluster of one)
    fence_proxy_async();
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmB) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmY0) : "memory");
    if (HAS32) asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmY1) : "memory");
  }
  if (warp == ST_MMA_WARP) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)), "r"(512u)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  // weights and bias are never written by an earlier kernel: read before the PDL wait
  for (int c = threadIdx.x; c < BN; c += ST_THREADS) sbias[c] = c < g.N ? __ldg(bias + c) : 0.f;
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  if (warp == ST_GATHER_WARP0 && lane == 0) {
    // the whole filter bank, resident for the kernel: K block kb = tap kb, all BN rows (the
    // tensor map's box holds BN / 2 rows: two boxes per block)
    mbar_arrive_expect_tx(bfull, (uint32_t)(KB * B_BLK));
    for (int kb = 0; kb < KB; ++kb)
      for (int h = 0; h < 2; ++h) tma_3d(smem_u32(sB) + kb * B_BLK + h * (B_BLK / 2), &tmB, bfull, kb * 64, h * (BN / 2), 0);
  }
  pdl_wait();  // the input rows and the output buffer belong to earlier kernels of the stream

  if (warp >= ST_GATHER_WARP0 && warp < ST_GATHER_WARP0 + ST_GATHER_WARPS) {
    // ---- gather: slab row r of tile t = space-to-depth pixel v = t*128 + r.  The loads of a
    // tile are issued BEFORE waiting for its slab buffer (their latency overlaps the wait).
    // Measured alternatives: L2 bulk prefetch of the tile's input rows a few
    // tiles ahead -- no gain (and 300 us lost when its issuing lane is on the MMA path); 16-byte
    // aligned vector loads + warp shuffles (one request per line) -- 2x slower than these
    // scalar loads.
    const int r = threadIdx.x - 32 * ST_GATHER_WARP0;
    const int SR = 128 + (KS - 1) * g.Ws + (KS - 1);  // rows the taps read
    const uint32_t slab0 = smem_u32(sSlab);
    // MMA issue state (warp ST_MMA_WARP only)
    const bool mma_warp = warp == ST_MMA_WARP;
    const uint32_t idesc = idesc_f16<BN, BF16, 1>();
    const uint64_t hi = sdesc(0, 128);
    const uint32_t sB16 = (smem_u32(sB) & 0x3FFFFu) >> 4, slab16 = (smem_u32(sSlab) & 0x3FFFFu) >> 4;
    uint32_t toff[KB];  // A row offset of each tap within the slab, 16-byte units
#pragma unroll
    for (int tap = 0; tap < KB; ++tap) toff[tap] = (uint32_t)(((tap / KS) * g.Ws + tap % KS) * 8);
    if (mma_warp) {
      mbar_wait(bfull, 0);
      tc_fence_after();
    }
    long long c_load = 0, c_sempty = 0, c_store = 0, c_tempty = 0, c_sfull = 0, c_issue = 0, c0 = 0;
    (void)c0;
    int lt = 0;
    for (int t = cid; t < tiles; t += ncl, ++lt) {
      const int sb = lt & 1;
      const uint32_t use = (uint32_t)(lt >> 1);
      SST(c0);
      float val[CH];
      const int64_t v = (int64_t)t * 128 + r;
      const int img = (int)(v / HW);
      const bool act = r < SR && img < g.Nimg;
      int ty = 0, tx = 0;
      if (act) {
        const int rem = (int)(v - (int64_t)img * HW);
        ty = rem / g.Ws;
        tx = rem - ty * g.Ws;
      }
      const int y0 = F * ty, x0 = F * tx;
      const float* p0 = x + ((int64_t)img * C0 * g.H + y0) * g.W + x0;
#ifdef DJINN_STEM_NOGATHER
      if (false) {  // diagnostic build: no input loads
#else
      if (act) {
#endif
#pragma unroll
        for (int c = 0; c < C0; ++c)
#pragma unroll
          for (int dy = 0; dy < F; ++dy)
#pragma unroll
            for (int dx = 0; dx < F; ++dx) {
              const bool ok = (y0 + dy < g.H) && (x0 + dx < g.W);
              val[(dy * F + dx) * C0 + c] = ok ? __ldg(p0 + ((int64_t)c * g.H + dy) * g.W + dx) : 0.f;
            }
      } else {
#pragma unroll
        for (int e = 0; e < CH; ++e) val[e] = 0.f;
      }
#ifdef DJINN_STEM_STATS
      { float acc = 0.f; for (int e = 0; e < CH; ++e) acc += val[e]; if (acc == 1234.5f) printf("x"); }
#endif
      SACC(c_load, c0);
      SST(c0);
      if (lane == 0) st_wait(sempty0 + 8 * sb, (use & 1) ^ 1);
      __syncwarp();
      SACC(c_sempty, c0);
      SST(c0);
      if (r < SR) {
        const uint32_t row = slab0 + (uint32_t)sb * ST_SLAB_BYTES + (uint32_t)r * 128;
#pragma unroll
        for (int j = 0; j < CH / 8; ++j)
          sts128(row + ((uint32_t)(j ^ (r & 7)) << 4),
                 make_uint4(pack2<BF16>(val[8 * j], val[8 * j + 1]), pack2<BF16>(val[8 * j + 2], val[8 * j + 3]),
                            pack2<BF16>(val[8 * j + 4], val[8 * j + 5]), pack2<BF16>(val[8 * j + 6], val[8 * j + 7])));
      }
      fence_proxy_async();  // generic-proxy slab writes -> visible to the tensor core (async proxy)
      __syncwarp();
      if (lane == 0) mbar_arrive(sfull0 + 8 * sb);
      SACC(c_store, c0);
      if (mma_warp) {
        // tile lt: every gather warp's rows are in, and its accumulator slot is drained
        const int slot = lt & 3;
        SST(c0);
        st_wait(tempty0 + 8 * slot, ((uint32_t)(lt >> 2) & 1) ^ 1);
        SACC(c_tempty, c0);
        SST(c0);
        mbar_wait(sfull0 + 8 * sb, use & 1);
        SACC(c_sfull, c0);
        SST(c0);
        tc_fence_after();
        if (elect_one()) {
          const uint32_t d = tmem + (uint32_t)(slot * 128);
          const uint32_t abase = slab16 + (uint32_t)sb * (ST_SLAB_BYTES >> 4);
#pragma unroll
          for (int tap = 0; tap < KB; ++tap) {
            const uint64_t ad = hi | (uint64_t)(abase + toff[tap]);
            const uint64_t bd = hi | (uint64_t)(sB16 + (uint32_t)tap * (B_BLK >> 4));
#pragma unroll
            for (int k = 0; k < KSUB; ++k) mma_f16(d, ad + 2 * k, bd + 2 * k, idesc, (tap | k) != 0);
          }
          mma_commit(sempty0 + 8 * sb);
          mma_commit(tfull0 + 8 * slot);
        }
        __syncwarp();
        SACC(c_issue, c0);
      }
    }
#ifdef DJINN_STEM_STATS
    if (blockIdx.x == 0 && lane == 0)
      printf("[stem gather warp %d] tiles %d load %lld sempty %lld store %lld tempty %lld sfull %lld issue %lld\n", warp, lt,
             c_load, c_sempty, c_store, c_tempty, c_sfull, c_issue);
#endif
  } else if (warp < ST_EPI_WARPS) {
    // ---- epilogue: warpgroup wg drains local tiles lt with lt % 2 == wg; thread = one pixel
    const int quarter = warp & 3, wg = warp >> 2;
    const uint32_t lane_base = (uint32_t)(quarter * 32) << 16;
    const uint32_t stg = smem_u32(sOut) + (uint32_t)warp * STG;  // [NB64 x (32 x 128 B, SW128)] [32 x 64 B, SW64]
    const uint32_t stg32 = stg + NB64 * 4096;
    const int rr = lane;
    auto put16 = [&](int p, uint4 v) {  // 16-byte piece p (channels 8p..8p+7) of this thread's pixel
      if (p < 8 * NB64) {
        const int b = p >> 3, j = p & 7;
        sts128(stg + (uint32_t)b * 4096 + (uint32_t)rr * 128 + ((uint32_t)(j ^ (rr & 7)) << 4), v);
      } else {
        const int j = p - 8 * NB64;
        sts128(stg32 + (uint32_t)rr * 64 + ((uint32_t)(j ^ ((rr >> 1) & 3)) << 4), v);
      }
    };
    auto put_chunk = [&](int i, const float (&o)[16]) {
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        uint4 u;
        if (g.out_half || !BF16)
          u = make_uint4(pack2<false>(o[8 * h], o[8 * h + 1]), pack2<false>(o[8 * h + 2], o[8 * h + 3]),
                         pack2<false>(o[8 * h + 4], o[8 * h + 5]), pack2<false>(o[8 * h + 6], o[8 * h + 7]));
        else
          u = make_uint4(pack2<true>(o[8 * h], o[8 * h + 1]), pack2<true>(o[8 * h + 2], o[8 * h + 3]),
                         pack2<true>(o[8 * h + 4], o[8 * h + 5]), pack2<true>(o[8 * h + 6], o[8 * h + 7]));
        put16(2 * i + h, u);
      }
    };
    long long e_wait = 0, e_work = 0, e_store = 0, e0 = 0;
    (void)e0;
    int lt = 0;
    for (int t = cid; t < tiles; t += ncl, ++lt) {
      if ((lt & 1) != wg) continue;
      const int slot = lt & 3;
      SST(e0);
      if (lane == 0) {
        bulk_wait_read0();  // this warp's previous TMA stores have read the staging tile
        st_wait(tfull0 + 8 * slot, (uint32_t)(lt >> 2) & 1);
      }
      __syncwarp();
      SACC(e_wait, e0);
      SST(e0);
      tc_fence_after();
      const uint32_t tbase = tmem + lane_base + (uint32_t)(slot * 128);
#if defined(DJINN_STEM_NOEPI)
      if (false) {  // diagnostic build: the accumulator is released unread
      } else
#endif
#if defined(DJINN_STEM_NOLRN)
      if (false) {  // diagnostic build: plain bias + act epilogue
#else
      if (g.epi_lrn) {
#endif
        // Caffe LRN across the pixel's N channels, window [c-2, c+2] clipped to [0, N) (values
        // beyond N are zero, so zero padding is exact); chunk i+1 is in flight from TMEM while
        // chunk i is normalised (the same arithmetic, in the same order, as k_tc.cu).
        const float ka = g.lrn_alpha_over_n, kk = g.lrn_k, nb = -g.lrn_beta;
        const int N = g.N;
        float bq[16], cur[16], nxt[16];
        uint32_t rq[16];
        tmem_ld16(tbase, rq);
        tmem_wait_ld();
        lds16(bq, sbias);
        bias_act16(cur, rq, bq, g.act);
        if (NCH > 1) tmem_ld16(tbase + 16, rq);
        float pm2 = 0.f, pm1 = 0.f;
#pragma unroll 1
        for (int i = 0; i < NCH; ++i) {
          if (i + 1 < NCH) {
            tmem_wait_ld();
            lds16(bq, sbias + 16 * (i + 1));
            bias_act16(nxt, rq, bq, g.act);
            if (16 * (i + 1) + 16 > N) {
#pragma unroll
              for (int j = 0; j < 16; ++j) nxt[j] = 16 * (i + 1) + j < N ? nxt[j] : 0.f;
            }
            if (i + 2 < NCH) tmem_ld16(tbase + (uint32_t)(16 * (i + 2)), rq);
          } else {
#pragma unroll
            for (int j = 0; j < 16; ++j) nxt[j] = 0.f;
          }
          float sq[20];
          sq[0] = pm2;
          sq[1] = pm1;
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const float2 s2 = mul2(make_float2(cur[2 * j], cur[2 * j + 1]), make_float2(cur[2 * j], cur[2 * j + 1]));
            sq[2 + 2 * j] = s2.x;
            sq[3 + 2 * j] = s2.y;
          }
          {
            const float2 s2 = mul2(make_float2(nxt[0], nxt[1]), make_float2(nxt[0], nxt[1]));
            sq[18] = s2.x;
            sq[19] = s2.y;
          }
          float q[18];
#pragma unroll
          for (int j = 0; j < 18; ++j) q[j] = sq[j] + sq[j + 1];
          const float2 ka2 = make_float2(ka, ka), kk2 = make_float2(kk, kk), nb2 = make_float2(nb, nb);
          float o[16];
#pragma unroll
          for (int j = 0; j < 16; j += 2) {
            const float2 s5 = add2(add2(make_float2(q[j], q[j + 1]), make_float2(q[j + 2], q[j + 3])),
                                   make_float2(sq[j + 4], sq[j + 5]));
            const float2 t2 = fma2(ka2, s5, kk2);
            const float2 l = mul2(nb2, make_float2(lg2_ftz(t2.x), lg2_ftz(t2.y)));
            const float2 ov = mul2(make_float2(cur[j], cur[j + 1]), make_float2(ex2_ftz(l.x), ex2_ftz(l.y)));
            o[j] = ov.x;
            o[j + 1] = ov.y;
          }
          pm2 = sq[16];
          pm1 = sq[17];
          put_chunk(i, o);
#pragma unroll
          for (int j = 0; j < 16; ++j) cur[j] = nxt[j];
        }
      } else
#if defined(DJINN_STEM_NOEPI)
      if (false)
#endif
      {
#pragma unroll 1
        for (int i = 0; i < NCH; ++i) {
          uint32_t rq[16];
          float bq[16], o[16];
          tmem_ld16(tbase + (uint32_t)(16 * i), rq);
          lds16(bq, sbias + 16 * i);
          tmem_wait_ld();
          bias_act16(o, rq, bq, g.act);
          if (16 * i + 16 > g.N) {
#pragma unroll
            for (int j = 0; j < 16; ++j) o[j] = 16 * i + j < g.N ? o[j] : 0.f;
          }
          put_chunk(i, o);
        }
      }
      // accumulator slot drained: hand it back to the MMA (leader's barrier)
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive_relaxed(tempty0 + 8 * slot);
      SACC(e_work, e0);
      SST(e0);
      // staging tile complete -> one TMA store per 64 / 32 channels of the warp's 32 pixels
      fence_proxy_async();
      __syncwarp();
      if (lane == 0) {
        const int v0 = t * 128 + quarter * 32;  // first virtual pixel of the warp
#pragma unroll
        for (int b = 0; b < NB64; ++b) tma_store_2d(&tmY0, stg + b * 4096, 64 * b, v0);
        if (HAS32) tma_store_2d(&tmY1, stg32, 64 * NB64, v0);
        bulk_commit();
      }
      SACC(e_store, e0);
    }
#ifdef DJINN_STEM_STATS
    if (blockIdx.x == 0 && lane == 0)
      printf("[stem epi warp %d] wait %lld work %lld store %lld\n", warp, e_wait, e_work, e_store);
#endif
    if (lane == 0) bulk_wait0();  // every store of this warp has landed before the grid completes
  }
  tc_fence_before();
  __syncthreads();
  if (warp == ST_MMA_WARP) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512u) : "memory");
  }
}

template <int BN, int KS>
constexpr int stem_smem() {
  return 1024 + ((KS * KS * BN * 128 + 1023) & ~1023) + 2 * ST_SLAB_BYTES + ST_EPI_WARPS * 32 * BN * 2 + 13 * 8 + 16;
}

template <int BN, bool BF16, int F, int C0, int KS>
cudaError_t launch_stem_inst(const StemGeom& g, const CUtensorMap* tmB, const CUtensorMap* tmY0, const CUtensorMap* tmY1,
                             const float* x, const float* bias, cudaStream_t st) {
  auto kern = stem_conv_kernel<BN, BF16, F, C0, KS>;
  constexpr int smem = stem_smem<BN, KS>();
  static_assert(smem <= 227 * 1024 - BN * 4, "stem kernel shared memory");
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  const int64_t tiles = ((int64_t)g.Nimg * g.Hs * g.Ws + 127) / 128;
  const int grid = (int)(tiles < tc_num_sms() ? tiles : tc_num_sms());
  return launch_pdl(kern, dim3(grid), dim3(ST_THREADS), smem, st, *tmB, *tmY0, *tmY1, g, x, bias);
}

}  // namespace

bool stem_supported(int bn, int f, int c0, int ks, int out_pitch) {
  return bn == 96 && out_pitch == 96 && f == 4 && c0 == 3 && ks == 3;
}

cudaError_t launch_stem_conv(const StemGeom& g, int dt, const CUtensorMap* tmB, const CUtensorMap* tmY0,
                             const CUtensorMap* tmY1, const float* x, const float* bias, cudaStream_t st) {
  if (g.Nimg <= 0) return cudaSuccess;
  if (g.N != 96) return cudaErrorInvalidValue;
  if (dt == DT_BF16) return launch_stem_inst<96, true, 4, 3, 3>(g, tmB, tmY0, tmY1, x, bias, st);
  return launch_stem_inst<96, false, 4, 3, 3>(g, tmB, tmY0, tmY1, x, bias, st);
}

}  // namespace djinn
