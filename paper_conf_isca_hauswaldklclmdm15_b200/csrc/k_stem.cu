// K2 (+ K4) for the first layer of an image net, two variants sharing one kernel template:
//
//   GATHER (K0 fused, opt-in DJINN_STEM=1): the strided conv reads the fp32 NCHW query images
//     itself -- 8 gather warps build each tile's space-to-depth slab from ordinary loads.
//   SLAB (the default for IMC conv1 + norm1): the slab of the packed 16-bit space-to-depth
//     tensor (the pack kernel's output) arrives by one TMA box per tile.
//
// What it computes ("the learned weights are kernels that are convolved with the
// image"; the image apps' queries are fp32 images, Table 3):
//     y[n, oy, ox, co] = act( b[co] + sum_{c, ky, kx} W[co, c, ky, kx] * x[n, c, s*oy + ky, s*ox + kx] )
// optionally followed by Caffe LRN across the co of a pixel (IMC conv1 + norm1).  The stride-F
// kernel is re-expressed by space-to-depth: pixel (ty, tx) of an Hs x Ws grid
// carries channel (dy*F + dx)*C0 + c = x[c][F*ty + dy][F*tx + dx], and the conv becomes a
// KS x KS stride-1 conv over that grid (IMC: 227^2 x 3, 11x11/4 -> 57^2 x 48, 3x3/1).  GEMM row
// m = a virtual pixel of the Hs x Ws grid; every tap is the tile's slab (128 + (KS-1)*Ws + KS-1
// consecutive pixels) shifted by ky*Ws + kx rows.
//
// Structure (B200, one CTA per tile of 128 virtual output pixels, persistent grid, CTA-local --
// a CTA pair would need cluster-scope acquire/release around generic-proxy slab writes, and the
// acquire.cluster poll compiled to an L1 invalidation per iteration):
//   * B, all KS*KS K blocks of the filter bank (IMC: 108 KB), is loaded ONCE by TMA and stays
//     resident in shared memory (the generic slab GEMM re-streams it through a ring per tile).
//   * tcgen05.mma.cta_group::1, M = 128, N = BN (IMC: 96) -- KSUB 16-channel K steps per tap
//     (3 of 4 for IMC's 48 real channels).
//   * epilogue warpgroups: TMEM -> registers -> bias + act (+ LRN) -> 16-bit -> a per-warp
//     staging tile in 128B-swizzled shared memory (conflict-free 16-byte writes) -> TMA tensor
//     store (cp.async.bulk.tensor) of the warp's 32 consecutive virtual pixels.  The output
//     tensor is the whole virtual Hs x Ws grid per image (IMC: 57^2 instead of 55^2 pixels, +7 %
//     bytes), so a warp's rows are one contiguous box; the consumer (the MAX pool) reads the
//     valid OH x OW corner of the stored grid.  (A 4D store of the exact 55^2 tensor needs a
//     negative x for rows continuing on the next image row; the TMA unit rejects that as an
//     illegal instruction.)
//   GATHER: warps 0-7 epilogue (2 warpgroups, 4 TMEM slots), warps 8-15 gather (warp 8 also
//     allocates TMEM and issues the MMAs of a tile right after its share of the slab): 16 warps,
//     4 per SM sub-partition, so 128 registers (a 17th warp would cap them at 96).
//   SLAB: warps 0-11 epilogue (3 warpgroups, 3 TMEM slots: the LRN epilogue is the long pole),
//     warp 12 slab TMA producer, warp 13 MMA.  Staging holds the 64-channel box of each warp;
//     the remaining BN - 64 channels are stored from registers.
//   POOL (SLAB + K5 fused, the default for IMC conv1 + norm1 + pool1): the following 3 x 3 /
//     stride-2 MAX pool runs in the epilogue, so the conv output (IMC: 595 MB) never reaches HBM
//     -- only the pooled tensor (4.2x smaller) is written, in the consumer's layout.  A tile is
//     two output rows of one image (2 * Ws <= 128 GEMM rows, starting at row 2r): pool row r
//     takes conv rows 2r, 2r + 1, 2r + 2, so tile r computes the partial max of its rows 2r and
//     2r + 1 (handed to the next tile's warpgroup through shared memory, mbarrier-ordered) and
//     completes pool row r - 1 with its row 2r.  A CTA walks whole bands of pool rows of one
//     image in order (bands split an image only when there are fewer images than SMs).  The
//     epilogue stages each half of the LRN'd channels (16-bit, exactly the values the unfused
//     path stores) in shared memory, pools them, and writes the pooled pixels with coalesced
//     16-byte stores.
#include "tc_common.cuh"
#include <cstdio>

namespace djinn {
namespace {

constexpr int ST_SLAB_ROWS = 248;  // slab buffer rows (>= 128 + (KS-1)*Ws + KS-1; IMC: 244)
// POOL: staged rows per warpgroup -- the pool reads conv rows 2r (tile rows 0 .. Ws-1) and 2r + 1
// (Ws .. 2 Ws - 1) up to column 2 (POW - 1) + 2, i.e. rows < Ws + 2 POW <= POOL_STG_ROWS
constexpr int POOL_STG_ROWS = 112;
// POOL: one hand-off buffer per half (tile lt + 1 reads each item of tile lt's partial pool row and
// then overwrites it with its own, same thread), so no "empty" barrier and half the space
#ifndef DJINN_STEM_HAND1
#define DJINN_STEM_HAND1 1
#endif
constexpr int POOL_HBUF = DJINN_STEM_HAND1 ? 1 : 2;
constexpr int ST_SLAB_BYTES = ST_SLAB_ROWS * 128;

#ifndef DJINN_STEM_NWG
#define DJINN_STEM_NWG 4
#endif
// CB (K-dense B): the resident filter bank is stored dense in K -- tap t's F*F*C0 channels at K
// t*F*F*C0 .. -- in whole 64-channel SW128 blocks (IMC: 9 x 48 = 432 -> 7 blocks, 84 KB) instead
// of one 64-channel block per tap with 16 zero channels (9 blocks, 108 KB), which leaves room for
// a 4th epilogue warpgroup in the pooled variant.  (An SW32 block per 16-channel K step was
// measured first: 27 us slower at 3 warpgroups, 445 vs 418 us.)
#ifndef DJINN_STEM_CB
#define DJINN_STEM_CB 0
#endif
template <bool GATHER, bool POOL = false>
struct StemCfg {
  static constexpr bool CB = DJINN_STEM_CB;
  static constexpr int NWG = GATHER ? 2 : (POOL ? DJINN_STEM_NWG : 3);  // epilogue warpgroups
  static constexpr int EPI_WARPS = 4 * NWG;
  static constexpr int NSLOT = GATHER ? 4 : NWG;            // TMEM accumulator slots (128 columns each)
  static constexpr int GATHER_WARP0 = EPI_WARPS, GATHER_WARPS = GATHER ? 8 : 0;
  static constexpr int PROD_WARP = EPI_WARPS;               // SLAB: TMA producer; GATHER: first gather warp
  static constexpr int MMA_WARP = GATHER ? EPI_WARPS : EPI_WARPS + 1;
  static constexpr int THREADS = 32 * (GATHER ? EPI_WARPS + GATHER_WARPS : EPI_WARPS + 2);
};

#ifdef DJINN_STEM_STATS
#define SST(v) v = clock64()
#define SACC(acc, v0) acc += clock64() - v0
#else
#define SST(v)
#define SACC(acc, v0)
#endif
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, uint32_t src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"((uint64_t)map),
               "r"(src), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void sts128(uint32_t addr, uint4 v) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

template <int BN, bool GATHER>
__host__ __device__ constexpr int stem_stage_bytes() {  // staging bytes per epilogue warp
  return GATHER ? 32 * BN * 2 : (BN / 64) * 4096;
}
// POOL: per warpgroup, one half of the tile's channels staged per pixel at an odd number of
// 16-byte pieces (conflict-free for 8 consecutive pixels); two hand-off buffers of the partial
// pool row, [2 halves][POW_MAX][HP pieces]
constexpr int POW_MAX = 28;
template <int BN>
__host__ __device__ constexpr int pool_pstr() { return ((BN / 2) / 8 + 1) * 16; }
template <int BN>
__host__ __device__ constexpr int pool_hand_bytes() { return 2 * POW_MAX * ((BN / 2) / 8) * 16; }  // one buffer
template <int BN, int KS, int CH, bool GATHER>
__host__ __device__ constexpr int stem_b_bytes() {  // K-dense: ceil(KS*KS*CH / 64) blocks
#ifdef DJINN_STEM_BPAD  // diagnostic: the per-tap bank's footprint whatever the layout
  return KS * KS * BN * 128;
#else
  return StemCfg<GATHER>::CB ? (KS * KS * CH + 63) / 64 * BN * 128 : KS * KS * BN * 128;
#endif
}
template <int BN, int KS, int CH, bool GATHER, bool POOL>
__host__ __device__ constexpr int stem_smem() {
  return 1024 + ((stem_b_bytes<BN, KS, CH, GATHER>() + 1023) & ~1023) + 2 * ST_SLAB_BYTES +
         (POOL ? StemCfg<GATHER, POOL>::NWG * POOL_STG_ROWS * pool_pstr<BN>() + POOL_HBUF * pool_hand_bytes<BN>()
               : StemCfg<GATHER, POOL>::EPI_WARPS * stem_stage_bytes<BN, GATHER>()) +
         32 * 8 + 16;
}
__device__ __forceinline__ uint4 lds128(uint32_t addr) {
  uint4 v;
  asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr) : "memory");
  return v;
}
template <bool BF16>
__device__ __forceinline__ uint4 hmax8(uint4 a, uint4 b) {  // packed 16-bit max (exact)
  uint4 r;
  if (BF16) {
    const __nv_bfloat162* x = reinterpret_cast<const __nv_bfloat162*>(&a);
    const __nv_bfloat162* y = reinterpret_cast<const __nv_bfloat162*>(&b);
    __nv_bfloat162* z = reinterpret_cast<__nv_bfloat162*>(&r);
#pragma unroll
    for (int j = 0; j < 4; ++j) z[j] = __hmax2(x[j], y[j]);
  } else {
    const __half2* x = reinterpret_cast<const __half2*>(&a);
    const __half2* y = reinterpret_cast<const __half2*>(&b);
    __half2* z = reinterpret_cast<__half2*>(&r);
#pragma unroll
    for (int j = 0; j < 4; ++j) z[j] = __hmax2(x[j], y[j]);
  }
  return r;
}

template <int BN, bool BF16, int F, int C0, int KS, bool GATHER, bool POOL>
__global__ void __launch_bounds__(StemCfg<GATHER, POOL>::THREADS, 1)
    stem_conv_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                     const __grid_constant__ CUtensorMap tmBc, const __grid_constant__ CUtensorMap tmY0,
                     const __grid_constant__ CUtensorMap tmY1,
                     const StemGeom g, const float* __restrict__ x, const float* __restrict__ bias,
                     void* __restrict__ Y) {
  using SC = StemCfg<GATHER, POOL>;
  constexpr int KB = KS * KS;                   // K blocks: one 64-channel block per tap
  constexpr int CH = F * F * C0;                // real channels of a space-to-depth pixel
  constexpr int KSUB = (CH + 15) / 16;          // 16-channel MMA K steps per tap (IMC: 3 of 4)
  constexpr int B_BLK = BN * 128;               // bytes of one K block of B (SW128 layout)
  constexpr int KBD = (KB * CH + 63) / 64;      // CB: K-dense blocks of B
  constexpr int NB64 = BN / 64, HAS32 = (BN % 64) == 32;
  constexpr int STG = stem_stage_bytes<BN, GATHER>();
  constexpr int NCH = BN / 16;                  // 16-column accumulator chunks
  constexpr int NSLOT = SC::NSLOT, NWG = SC::NWG;
  static_assert(CH <= 64 && CH % 8 == 0, "space-to-depth pixel must fill whole 8-channel chunks of one K block");
  static_assert(!SC::CB || CH % 16 == 0, "K-dense bank: every 16-channel K step inside one 64-channel block");
  static_assert(BN % 32 == 0 && BN <= 128, "tile width");

  pdl_trigger();
  const int cid = blockIdx.x, ncl = gridDim.x;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
#ifdef DJINN_STEM_SLAB_FIRST  // layout experiment: the two slab buffers at the base, then B
  uint8_t* sSlab = smem;
  uint8_t* sB = sSlab + 2 * ST_SLAB_BYTES;
  uint8_t* sOut = sB + ((stem_b_bytes<BN, KS, CH, GATHER>() + 1023) & ~1023);
#else
  uint8_t* sB = smem;
  uint8_t* sSlab = sB + ((stem_b_bytes<BN, KS, CH, GATHER>() + 1023) & ~1023);
  uint8_t* sOut = sSlab + 2 * ST_SLAB_BYTES;
#endif
  uint8_t* sHand = sOut + (POOL ? NWG * POOL_STG_ROWS * pool_pstr<BN>() : SC::EPI_WARPS * STG);  // POOL: partial pool rows
  uint64_t* bars = reinterpret_cast<uint64_t*>(sHand + (POOL ? POOL_HBUF * pool_hand_bytes<BN>() : 0));
  // bars: bfull, sfull[2], sempty[2], tfull[4], tempty[4], (tmem slot), POOL: hfull[2][2] at 16, hempty[2][2] at 20
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 13);
  __shared__ __align__(16) float sbias[BN];
  const uint32_t bfull = smem_u32(bars), sfull0 = smem_u32(bars + 1), sempty0 = smem_u32(bars + 3);
  const uint32_t tfull0 = smem_u32(bars + 5), tempty0 = smem_u32(bars + 9);
  const uint32_t hfull0 = smem_u32(bars + 16), hempty0 = smem_u32(bars + 20);
  // single hand-off buffer: per half, the local index of the last tile that published its partial
  // pool row (a counter, not an mbarrier phase: warpgroups run up to NSLOT tiles apart, so a
  // parity wait could alias a phase two tiles old)
  const uint32_t hseq0 = smem_u32(bars + 24);
  static_assert(!POOL || !GATHER, "the fused pool runs on the TMA-slab variant");

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int HW = g.Hs * g.Ws;
  const int64_t M = (int64_t)g.Nimg * HW;
  const int tiles = (int)((M + 127) / 128);
  // This CTA's tile sequence, walked identically by the producer, the MMA warp and the
  // epilogue: fn(local tile lt, first GEMM row, image, pool-row index r, first / last tile of a
  // band).  POOL: units (image, band of pool rows [pr0, pr1)), tile r = conv rows 2r, 2r + 1
  // for r = pr0 .. pr1; otherwise 128 consecutive virtual pixels, strided over the grid.
  auto for_each_tile = [&](auto&& fn) {
    int lt = 0;
    if (POOL) {
      const int units = g.Nimg * g.bands;
      for (int u = cid; u < units; u += ncl) {
        const int img = u / g.bands, b = u - img * g.bands;
        const int pr0 = b * g.POH / g.bands, pr1 = (b + 1) * g.POH / g.bands;
        for (int r = pr0; r <= pr1; ++r, ++lt) fn(lt, img * HW + 2 * r * g.Ws, img, r, r == pr0, r == pr1);
      }
    } else {
      for (int t = cid; t < tiles; t += ncl, ++lt) fn(lt, t * 128, 0, 0, false, false);
    }
  };

  if (warp == SC::PROD_WARP && lane == 0) {
    mbar_init(bfull, 1);
    for (int s = 0; s < 2; ++s) {
      mbar_init(sfull0 + 8 * s, GATHER ? SC::GATHER_WARPS : 1);  // every gather warp / the TMA tx
      mbar_init(sempty0 + 8 * s, 1);
    }
    for (int s = 0; s < 4; ++s) {
      mbar_init(tfull0 + 8 * s, 1);
      mbar_init(tempty0 + 8 * s, 4);  // the draining warpgroup
    }
    if (POOL) {
      for (int s = 0; s < 4; ++s) {
        mbar_init(hfull0 + 8 * s, 1);   // writer warpgroup, per (buffer, half)
        mbar_init(hempty0 + 8 * s, 1);  // reader warpgroup, per (buffer, half)
      }
      for (int h = 0; h < 2; ++h) asm volatile("st.shared.s32 [%0], %1;" ::"r"(hseq0 + 4 * h), "r"(-1) : "memory");
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");  // (cluster of one)
    fence_proxy_async();
    if (!GATHER) asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)(SC::CB ? &tmBc : &tmB)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmY0) : "memory");
    if (HAS32 && GATHER) asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmY1) : "memory");
  }
  if (warp == SC::MMA_WARP) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)), "r"(512u)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  // weights and bias are never written by an earlier kernel: read before the PDL wait
  for (int c = threadIdx.x; c < BN; c += SC::THREADS) sbias[c] = c < g.N ? __ldg(bias + c) : 0.f;
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  if (warp == SC::PROD_WARP && lane == 0) {
    // the whole filter bank, resident for the kernel: K block kb = tap kb, all BN rows (the
    // tensor map's box holds BN / 2 rows: two boxes per block)
    if (SC::CB) {  // K-dense bank: KBD blocks of 64 channels, two boxes of BN / 2 rows each
      mbar_arrive_expect_tx(bfull, (uint32_t)(KBD * B_BLK));
      for (int kb = 0; kb < KBD; ++kb)
        for (int h = 0; h < 2; ++h) tma_2d(smem_u32(sB) + kb * B_BLK + h * (B_BLK / 2), &tmBc, bfull, kb * 64, h * (BN / 2));
    } else {
      mbar_arrive_expect_tx(bfull, (uint32_t)(KB * B_BLK));
      for (int kb = 0; kb < KB; ++kb)
        for (int h = 0; h < 2; ++h) tma_3d(smem_u32(sB) + kb * B_BLK + h * (B_BLK / 2), &tmB, bfull, kb * 64, h * (BN / 2), 0);
    }
  }
  pdl_wait();  // the input rows and the output buffer belong to earlier kernels of the stream

  // MMA issue of local tile lt (the MMA warp only): slab sb complete, its TMEM slot drained
  const uint32_t idesc = idesc_f16<BN, BF16, 1>();
  const uint64_t hi = sdesc(0, 128);
  const uint32_t sB16 = (smem_u32(sB) & 0x3FFFFu) >> 4, slab16 = (smem_u32(sSlab) & 0x3FFFFu) >> 4;
  long long m_te = 0, m_sf = 0, m0 = 0;
  (void)m0;
  auto issue_tile = [&](int lt) {
    const int slot = lt % NSLOT, sb = lt & 1;
    SST(m0);
    mbar_wait_sleep(tempty0 + 8 * slot, ((uint32_t)(lt / NSLOT) & 1) ^ 1);
    SACC(m_te, m0);
    SST(m0);
    mbar_wait(sfull0 + 8 * sb, (uint32_t)(lt >> 1) & 1);
    SACC(m_sf, m0);
    tc_fence_after();
    if (elect_one()) {
      const uint32_t d = tmem + (uint32_t)(slot * 128);
      const uint32_t abase = slab16 + (uint32_t)sb * (ST_SLAB_BYTES >> 4);
#pragma unroll
      for (int tap = 0; tap < KB; ++tap) {
        const uint64_t ad = hi | (uint64_t)(abase + (uint32_t)(((tap / KS) * g.Ws + tap % KS) * 8));
        const uint64_t bd = hi | (uint64_t)(sB16 + (uint32_t)tap * (B_BLK >> 4));
#pragma unroll
        for (int k = 0; k < KSUB; ++k) {
          const int kk = tap * CH + 16 * k;  // CB: the K index of this step in the dense bank
          const uint64_t bk =
              SC::CB ? hi | (uint64_t)(sB16 + (uint32_t)(kk >> 6) * (B_BLK >> 4) + (uint32_t)(((kk & 63) * 2) >> 4)) : bd + 2 * k;
          mma_f16(d, ad + 2 * k, bk, idesc, (tap | k) != 0);
        }
      }
      mma_commit(sempty0 + 8 * sb);
      mma_commit(tfull0 + 8 * slot);
    }
    __syncwarp();
  };

  if (GATHER && warp >= SC::GATHER_WARP0 && warp < SC::GATHER_WARP0 + SC::GATHER_WARPS) {
    // ---- gather: slab row r of tile t = space-to-depth pixel v = t*128 + r.  The loads of a
    // tile are issued BEFORE waiting for its slab buffer (their latency overlaps the wait).
    // Measured alternatives: L2 bulk prefetch of the tile's input rows a few
    // tiles ahead -- no gain; 16-byte aligned vector loads + warp shuffles (one request per
    // line) -- 2x slower than these scalar loads.
    const int r = threadIdx.x - 32 * SC::GATHER_WARP0;
    const int SR = 128 + (KS - 1) * g.Ws + (KS - 1);  // rows the taps read
    const uint32_t slab0 = smem_u32(sSlab);
    if (warp == SC::MMA_WARP) {
      mbar_wait(bfull, 0);
      tc_fence_after();
    }
    int lt = 0;
    for (int t = cid; t < tiles; t += ncl, ++lt) {
      const int sb = lt & 1;
      const uint32_t use = (uint32_t)(lt >> 1);
      float val[CH];
      const int64_t v = (int64_t)t * 128 + r;
      const int img = (int)(v / HW);
      if (r < SR && img < g.Nimg) {
        const int rem = (int)(v - (int64_t)img * HW);
        const int ty = rem / g.Ws, tx = rem - ty * g.Ws;
        const int y0 = F * ty, x0 = F * tx;
        const float* p0 = x + ((int64_t)img * C0 * g.H + y0) * g.W + x0;
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
      if (lane == 0) mbar_wait_sleep(sempty0 + 8 * sb, (use & 1) ^ 1);
      __syncwarp();
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
      if (warp == SC::MMA_WARP) issue_tile(lt);
    }
  } else if (!GATHER && warp == SC::PROD_WARP) {
    // ---- slab producer: one TMA box {64 channels, slab rows} of the packed tensor per tile
    if (elect_one()) {
      for_each_tile([&](int lt, int row0, int, int, bool, bool) {
        const int sb = lt & 1;
        mbar_wait_sleep(sempty0 + 8 * sb, ((uint32_t)(lt >> 1) & 1) ^ 1);
        mbar_arrive_expect_tx(sfull0 + 8 * sb, (uint32_t)g.slab_rows * 128u);
        tma_2d(smem_u32(sSlab) + (uint32_t)sb * ST_SLAB_BYTES, &tmA, sfull0 + 8 * sb, 0, row0);
      });
    }
    __syncwarp();
  } else if (!GATHER && warp == SC::MMA_WARP) {
    mbar_wait(bfull, 0);
    tc_fence_after();
    for_each_tile([&](int lt, int, int, int, bool, bool) { issue_tile(lt); });
#ifdef DJINN_STEM_STATS
    if (blockIdx.x == 0 && lane == 0) printf("[stem mma] wait tempty %lld sfull %lld\n", m_te, m_sf);
#endif
  } else if (POOL && warp < SC::EPI_WARPS) {
    // ---- epilogue with the fused 3 x 3 / stride-2 MAX pool (POOL): thread = tile row m
    constexpr int HALF = BN / 2, HP = HALF / 8, PSTR = pool_pstr<BN>(), HB = pool_hand_bytes<BN>();
    constexpr int HHALF = POW_MAX * HP * 16;  // bytes of one half of a hand-off buffer
    static_assert(HALF % 16 == 0, "a staged half is whole 16-column accumulator chunks");
    const int quarter = warp & 3, wg = warp >> 2;
    const int m = quarter * 32 + lane;
    const uint32_t lane_base = (uint32_t)(quarter * 32) << 16;
    const uint32_t stg = smem_u32(sOut) + (uint32_t)(wg * POOL_STG_ROWS * PSTR);
    const uint32_t my_row = stg + (uint32_t)(m * PSTR);
    const uint32_t hand = smem_u32(sHand);
    const int PJ = g.pool_gp / 8;  // output pieces per half (grouped: the group pitch, pads written 0)
    const int OPH = g.POH + 2 * g.obd, OPW = g.POW + 2 * g.obd;
    uint16_t* Yp = reinterpret_cast<uint16_t*>(Y);
    const float ka = g.lrn_alpha_over_n, kk = g.lrn_k, nb = -g.lrn_beta;
    long long p_wait = 0, p_hw = 0, p_pool = 0, p_tot = 0, p0 = 0, p1 = 0, p2 = 0;
    (void)p0; (void)p1; (void)p2;
    for_each_tile([&](int lt, int, int img, int r, bool first, bool last) {
      if (lt % NWG != wg) return;
      const int slot = lt % NSLOT, k = POOL_HBUF == 2 ? (lt & 1) : 0, kp = POOL_HBUF == 2 ? (k ^ 1) : 0;
      SST(p2);
      SST(p0);
      if (lane == 0) mbar_wait_sleep(tfull0 + 8 * slot, (uint32_t)(lt / NSLOT) & 1);
      __syncwarp();
      SACC(p_wait, p0);
      tc_fence_after();
      const uint32_t tbase = tmem + lane_base + (uint32_t)(slot * 128);
      // pool the staged half h of the tile's channels.  Hand-off buffer k carries this tile's
      // partial pool row r (max of conv rows 2r, 2r + 1) to tile lt + 1; each (buffer, half) is
      // rewritten only after its previous reader (tile lt - 1, same half) has released it and
      // is published with one arrival, so no barrier phase can run two uses ahead, and the
      // chain between consecutive tiles is one pool step, not a whole epilogue.  Waits sleep in
      // lane 0 (spinning warps would take issue slots from the other warpgroups' LRN math).
      auto pool_half = [&](int h) {
        SST(p1);
        asm volatile("bar.sync %0, 128;" ::"r"(1 + wg) : "memory");  // half h staged by the warpgroup
        SST(p0);
        if (lane == 0) {
          if (POOL_HBUF == 2) {
            mbar_wait_sleep(hempty0 + 8 * (2 * k + h), ((uint32_t)(lt >> 1) & 1) ^ 1);
            if (lt > 0) mbar_wait_sleep(hfull0 + 8 * (2 * kp + h), (uint32_t)((lt - 1) >> 1) & 1);
          } else if (lt > 0) {  // tile lt - 1 has read the buffer and written its own partial row
            int seen, iters = 0;
            for (;;) {
              asm volatile("ld.acquire.cta.shared.s32 %0, [%1];" : "=r"(seen) : "r"(hseq0 + 4 * h) : "memory");
              if (seen >= lt - 1) break;
              if (++iters > (1 << 24)) __trap();  // a lost publication must fault, never hang
              __nanosleep(64);
            }
          }
        }
        __syncwarp();
        SACC(p_hw, p0);
        const uint32_t hw = hand + (uint32_t)(k * HB + h * HHALF), hr = hand + (uint32_t)(kp * HB + h * HHALF);
        const int64_t orow = ((int64_t)img * OPH + (r - 1) + g.obd) * OPW + g.obd;  // pool row r - 1, column 0
        for (int q = m; q < g.POW * PJ; q += 128) {
          const int pc = q / PJ, j = q - pc * PJ;
          uint4 res = make_uint4(0u, 0u, 0u, 0u);
          if (j < HP) {
            const uint32_t a = stg + (uint32_t)(2 * pc * PSTR + j * 16);
            const uint4 va = hmax8<BF16>(hmax8<BF16>(lds128(a), lds128(a + PSTR)), lds128(a + 2 * PSTR));
            const uint32_t b = a + (uint32_t)(g.Ws * PSTR);
            const uint4 vb = hmax8<BF16>(hmax8<BF16>(lds128(b), lds128(b + PSTR)), lds128(b + 2 * PSTR));
            // read the previous tile's partial row before overwriting it (one buffer: hr == hw)
            if (!first) res = hmax8<BF16>(lds128(hr + (uint32_t)((pc * HP + j) * 16)), va);
            if (!last) sts128(hw + (uint32_t)((pc * HP + j) * 16), hmax8<BF16>(va, vb));
          }
          if (!first) *reinterpret_cast<uint4*>(Yp + (orow + pc) * g.Cpo + h * g.pool_gp + 8 * j) = res;
        }
        asm volatile("bar.sync %0, 128;" ::"r"(1 + wg) : "memory");  // staging read, hand-off half written
        if (m == 0) {
          if (POOL_HBUF == 2) {
            mbar_arrive(hfull0 + 8 * (2 * k + h));
            if (lt > 0) mbar_arrive(hempty0 + 8 * (2 * kp + h));
          } else {
            asm volatile("st.release.cta.shared.s32 [%0], %1;" ::"r"(hseq0 + 4 * h), "r"(lt) : "memory");
          }
        }
        SACC(p_pool, p1);
      };
      auto put_chunk = [&](int i, const float (&o)[16]) {  // 16-bit LRN output -> staged half
        const int p0 = 2 * (i % (HALF / 16));
        if (m >= POOL_STG_ROWS) return;  // rows the pool never reads
#pragma unroll
        for (int hh = 0; hh < 2; ++hh)
          sts128(my_row + (uint32_t)((p0 + hh) * 16),
                 make_uint4(pack2<BF16>(o[8 * hh], o[8 * hh + 1]), pack2<BF16>(o[8 * hh + 2], o[8 * hh + 3]),
                            pack2<BF16>(o[8 * hh + 4], o[8 * hh + 5]), pack2<BF16>(o[8 * hh + 6], o[8 * hh + 7])));
      };
      // Caffe LRN across the pixel's N channels (the same arithmetic, in the same order, as the
      // unfused epilogue below and k_tc.cu)
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
          // every accumulator column has been read: hand the slot back to the MMA
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive_relaxed(tempty0 + 8 * slot);
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
        if (i % (HALF / 16) == HALF / 16 - 1) pool_half(i / (HALF / 16));
#pragma unroll
        for (int j = 0; j < 16; ++j) cur[j] = nxt[j];
      }
      SACC(p_tot, p2);
    });
#ifdef DJINN_STEM_STATS
    if (blockIdx.x == 0 && lane == 0)
      printf("[stem pool-epi warp %d] total %lld tfull-wait %lld pool(incl hand-off) %lld hand-off wait %lld\n", warp,
             p_tot, p_wait, p_pool, p_hw);
#endif
  } else if (!POOL && warp < SC::EPI_WARPS) {
    // ---- epilogue: warpgroup wg drains local tiles lt with lt % NWG == wg; thread = one pixel
    const int quarter = warp & 3, wg = warp >> 2;
    const uint32_t lane_base = (uint32_t)(quarter * 32) << 16;
    const uint32_t stg = smem_u32(sOut) + (uint32_t)warp * STG;  // [NB64 x (32 x 128 B, SW128)] (+ [32 x 64 B, SW64])
    const uint32_t stg32 = stg + NB64 * 4096;
    const int rr = lane;
    const int Cp = g.N;
    uint16_t* Yp = reinterpret_cast<uint16_t*>(Y);
    int64_t vpix = 0;  // this thread's virtual pixel in the current tile
    auto put16 = [&](int p, uint4 v) {  // 16-byte piece p (channels 8p..8p+7) of this thread's pixel
      if (p < 8 * NB64) {
        const int b = p >> 3, j = p & 7;
        sts128(stg + (uint32_t)b * 4096 + (uint32_t)rr * 128 + ((uint32_t)(j ^ (rr & 7)) << 4), v);
      } else if (GATHER) {
        const int j = p - 8 * NB64;
        sts128(stg32 + (uint32_t)rr * 64 + ((uint32_t)(j ^ ((rr >> 1) & 3)) << 4), v);
      } else if (vpix < M) {
        *reinterpret_cast<uint4*>(Yp + vpix * Cp + 8 * p) = v;
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
      if (lt % NWG != wg) continue;
      const int slot = lt % NSLOT;
      vpix = (int64_t)t * 128 + quarter * 32 + lane;
      SST(e0);
      if (lane == 0) {
        bulk_wait_read0();  // this warp's previous TMA stores have read the staging tile
        mbar_wait_sleep(tfull0 + 8 * slot, (uint32_t)(lt / NSLOT) & 1);
      }
      __syncwarp();
      SACC(e_wait, e0);
      SST(e0);
      tc_fence_after();
      const uint32_t tbase = tmem + lane_base + (uint32_t)(slot * 128);
      if (g.epi_lrn) {
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
      } else {
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
      // accumulator slot drained: hand it back to the MMA
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive_relaxed(tempty0 + 8 * slot);
      SACC(e_work, e0);
      SST(e0);
      // staging tile complete -> one TMA store per 64 (/ 32) channels of the warp's 32 pixels
      fence_proxy_async();
      __syncwarp();
      if (lane == 0) {
        const int v0 = t * 128 + quarter * 32;  // first virtual pixel of the warp
#pragma unroll
        for (int b = 0; b < NB64; ++b) tma_store_2d(&tmY0, stg + b * 4096, 64 * b, v0);
        if (HAS32 && GATHER) tma_store_2d(&tmY1, stg32, 64 * NB64, v0);
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
  if (warp == SC::MMA_WARP) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512u) : "memory");
  }
}

template <int BN, bool BF16, int F, int C0, int KS, bool GATHER, bool POOL>
cudaError_t launch_stem_inst(const StemGeom& g, const CUtensorMap* tmA, const CUtensorMap* tmB, const CUtensorMap* tmBc,
                             const CUtensorMap* tmY0, const CUtensorMap* tmY1, const float* x, const float* bias, void* Y,
                             cudaStream_t st) {
  auto kern = stem_conv_kernel<BN, BF16, F, C0, KS, GATHER, POOL>;
  constexpr int smem = stem_smem<BN, KS, F * F * C0, GATHER, POOL>();
  static_assert(smem <= 227 * 1024 - BN * 4, "stem kernel shared memory");
  cudaError_t e = ensure_max_smem((const void*)kern, smem);
  if (e != cudaSuccess) return e;
  const int64_t work = POOL ? (int64_t)g.Nimg * g.bands : ((int64_t)g.Nimg * g.Hs * g.Ws + 127) / 128;
  const int grid = (int)(work < tc_num_sms() ? work : tc_num_sms());
  return launch_pdl(kern, dim3(grid), dim3(StemCfg<GATHER, POOL>::THREADS), smem, st, *tmA, *tmB, *tmBc, *tmY0, *tmY1, g, x,
                    bias, Y);
}

}  // namespace

bool stem_dense_b() { return StemCfg<false>::CB; }

bool stem_supported(int bn, int f, int c0, int ks, int out_pitch) {
  return bn == 96 && out_pitch == 96 && f == 4 && c0 == 3 && ks == 3;
}

bool stem_pool_supported(int n, int ws, int oh, int ow, int kernel, int stride, int pad, int cpo, int gsz, int gpitch,
                         int xu) {
  // tile = two conv rows; pool rows exactly cover the conv rows (no clipped ceil window);
  // output plain at pitch n, or two groups of n / 2 channels at a group pitch (pads written 0)
  if (kernel != 3 || stride != 2 || pad != 0 || xu != 1 || 2 * ws > 128 || oh < 3 || ow < 3) return false;
  if (ws + 2 * ((ow - 3) / 2 + 1) > POOL_STG_ROWS) return false;  // the pooled rows fit the staging
  if ((oh - 3) % 2 || (ow - 3) % 2 || (ow - 3) / 2 + 1 > POW_MAX || ow > ws) return false;
  const bool plain = cpo == n && gsz >= n;
  const bool grouped = gsz == n / 2 && gpitch >= gsz && gpitch % 8 == 0 && cpo == 2 * gpitch;
  return n == 96 && (plain || grouped);
}

int stem_pool_bands(int nimg, int poh) {
  // bands of pool rows per image: minimise the busiest CTA's tiles, ceil(units / SMs) x
  // (rows per band + 1); ties -> fewer bands (fewer extra tiles)
  const int sms = tc_num_sms();
  int best = 1;
  int64_t best_cost = -1;
  for (int b = 1; b <= poh; ++b) {
    const int64_t units = (int64_t)nimg * b;
    const int64_t cost = ((units + sms - 1) / sms) * ((poh + b - 1) / b + 1);
    if (best_cost < 0 || cost < best_cost) { best = b; best_cost = cost; }
  }
  return best;
}

cudaError_t launch_stem_conv(const StemGeom& g, int dt, const CUtensorMap* tmA, const CUtensorMap* tmB,
                             const CUtensorMap* tmBc, const CUtensorMap* tmY0, const CUtensorMap* tmY1, const float* x,
                             const float* bias, void* Y, cudaStream_t st) {
  if (g.Nimg <= 0) return cudaSuccess;
  if (g.N != 96 || (!g.gather && (g.slab_rows < 128 + 2 * g.Ws + 2 || g.slab_rows > ST_SLAB_ROWS)))
    return cudaErrorInvalidValue;
  if (g.pool) {
    if (g.gather || g.out_half || !g.epi_lrn || g.bands < 1 || g.bands > g.POH || g.POW > POW_MAX || 2 * g.Ws > 128)
      return cudaErrorInvalidValue;
    if (dt == DT_BF16) return launch_stem_inst<96, true, 4, 3, 3, false, true>(g, tmA, tmB, tmBc, tmY0, tmY1, x, bias, Y, st);
    return launch_stem_inst<96, false, 4, 3, 3, false, true>(g, tmA, tmB, tmBc, tmY0, tmY1, x, bias, Y, st);
  }
  if (g.gather) {
    if (dt == DT_BF16) return launch_stem_inst<96, true, 4, 3, 3, true, false>(g, tmA, tmB, tmBc, tmY0, tmY1, x, bias, Y, st);
    return launch_stem_inst<96, false, 4, 3, 3, true, false>(g, tmA, tmB, tmBc, tmY0, tmY1, x, bias, Y, st);
  }
  if (dt == DT_BF16) return launch_stem_inst<96, true, 4, 3, 3, false, false>(g, tmA, tmB, tmBc, tmY0, tmY1, x, bias, Y, st);
  return launch_stem_inst<96, false, 4, 3, 3, false, false>(g, tmA, tmB, tmBc, tmY0, tmY1, x, bias, Y, st);
}

}  // namespace djinn
