// The whole forward pass of a two-layer window MLP (the SENNA-style POS / CHK / NER services,
// PAPER.md L104 and Table 1; SURVEY 8(a) a2 + a7 + a8) as ONE kernel:
//     h = act1(x . W1^T + b1),   z = h . W2^T + b2,   p = softmax(z)   (or z / argmax z)
// for a tile of 128 query rows per CTA.  These nets are launch- and latency-bound, not
// bandwidth-bound (4096 windows are 5 MB of input: 0.8 us of HBM time): the unfused path is four
// dependent kernels (pack, l1, l2, softmax) of a few microseconds each ("small
// networks"; L173 on their low GPU occupancy).  Here every intermediate stays on chip:
//   1. all 8 warps load the tile's fp32 rows (coalesced), convert them to 16-bit and write the
//      128B-swizzled K-major A operand of layer 1 into shared memory (pad columns zero);
//   2. one thread streams W1 through a 4-stage ring of 32-column K blocks (TMA, SWIZZLE_64B) and
//      issues tcgen05.mma (M = 128, N = N1p split into 256 + the rest) into TMEM columns
//      [0, N1p); W2 (all of it, K-major SWIZZLE_128B) arrives once at the start;
//   3. all 8 warps drain layer 1 (bias + activation, 16-bit) straight into layer 2's A operand,
//      which overwrites layer 1's (consumed) A in shared memory;
//   4. one thread issues layer 2 into TMEM columns [N1c, N1c + N2p);
//   5. warps 0-3 (one row per thread) read the logits, add the bias and write the probabilities
//      (max-subtracted exp, then normalised), the logits or the argmax (ties -> lowest index).
// Arithmetic per element is the unfused path's: fp32 accumulation of 16-bit products, bias +
// activation in fp32 rounded once to 16 bits, fp32 logits, expf-based softmax.
#include "tc_common.cuh"
#include <cfloat>
#include <cstdio>
#include <cstdlib>
#ifdef DJINN_MLP_STATS
#define MST(i) if (tid == 0) ts[i] = clock64()
#else
#define MST(i)
#endif

namespace djinn {
namespace {

#ifndef DJINN_MLP_THREADS
#define DJINN_MLP_THREADS 512
#endif
constexpr int MLP_THREADS = DJINN_MLP_THREADS;  // 16 warps: 4 per TMEM lane quarter drain layer 1
constexpr int MLP_CG = MLP_THREADS / 128;        // column groups of the layer-1 epilogue
constexpr int MLP_WSTAGES = 4;            // W1 ring stages (whole-net kernel)
constexpr int MLP_MAXST = 12;             // AT: ring stages fitted to MLP_RING_BYTES (smaller stages when split)
constexpr int MLP_RING_BYTES = 160 * 1024;
// ring stages of a launch (host and device agree): the TMA-fed tail keeps ~160 KB in flight
__host__ __device__ inline int mlp_stages(bool at, int sstride) {
#ifdef DJINN_MLP_WK32
  if (!at) return MLP_WSTAGES;
#else
  if (!at) return 2;
#endif
  const int n = MLP_RING_BYTES / sstride;
  return n < 2 ? 2 : (n > MLP_MAXST ? MLP_MAXST : n);
}
constexpr int MLP_WK = 32;                // K columns per W1 stage (SWIZZLE_64B rows), whole-net kernel
constexpr int MLP_WK_AT = 64;             // TMA-fed tail: 128-byte rows (SWIZZLE_128B) -- 64-byte TMA rows
                                          // had capped its stream at ~23 B/clock per SM (DIG: 12 us of layer 1)
// 128-byte W1 rows for the whole-net kernel too (2 ring stages of N1p x 128 B; its A is resident):
// POS 4096 windows 14.5 -> 13.5 us, 65536 75.7 -> 72.4 us on B200.  DJINN_MLP_WK32 restores the
// 4-stage ring of 64-byte rows.
#ifdef DJINN_MLP_WK32
__host__ __device__ constexpr int mlp_wk(bool at) { return at ? MLP_WK_AT : MLP_WK; }
#else
__host__ __device__ constexpr int mlp_wk(bool at) { return MLP_WK_AT; }
#endif

__device__ __forceinline__ uint32_t idesc_rt(int n, bool bf16) {  // kind::f16, D fp32, K-major A/B, M = 128
  const uint32_t ab = bf16 ? 1u : 0u;
  return (1u << 4) | (ab << 7) | (ab << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
}

// AT = false: layer 1's A is built from the fp32 query rows x (the window nets' input);
// AT = true: A is a 16-bit activation tensor (the tail of a larger net, e.g. DIG's pool2 output)
// read by TMA (tmA: 2D {K0p, rows}, box {32, 128}, SWIZZLE_64B) through the W1 ring -- each stage
// carries its 32-column A block beside the W1 block -- and layer 2's A operand reuses the ring.
template <bool BF16, bool AT>
__global__ void __launch_bounds__(MLP_THREADS, 1)
    mlp2_kernel(const __grid_constant__ CUtensorMap tmW1, const __grid_constant__ CUtensorMap tmW2,
                const __grid_constant__ CUtensorMap tmA, const MlpGeom g, const float* __restrict__ x,
                const float* __restrict__ b1, const float* __restrict__ b2, void* __restrict__ out) {
  pdl_trigger();
#ifdef DJINN_MLP_STATS
  long long ts[12] = {0};
  const int tid0 = threadIdx.x;
  if (tid0 == 0) ts[0] = clock64();
#endif
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  // Split (AT only, nsplit = S > 1): a cluster of S CTAs shares a block of 128 rows; CTA q owns
  // layer 1's columns [q N1p, (q + 1) N1p) (N1p = g.N1p / S) -- its slice of W1 -- and computes the
  // partial logits of layer 2 over that K slice; CTA 0 adds the S partials (in rank order, through
  // DSMEM) and the bias, then runs the softmax.  The per-CTA layer-1 work drops S-fold.
  const int S = AT && g.nsplit > 1 ? g.nsplit : 1;
  const uint32_t q = S > 1 ? cluster_rank() : 0u;
  const int N1p = g.N1p / S, n1o = (int)q * N1p;
  const int N1 = min(N1p, g.N1 - n1o);            // real layer-1 columns of this CTA
  const int K1p = S > 1 ? (N1p + 63) / 64 * 64 : g.K1p;
  const int N1c = S > 1 ? (N1p + g.N2p <= 512 ? N1p : 0) : g.N1c;
  const int KB0 = g.K0p / 64, KB1 = K1p / 64;    // 64-column blocks of the two A operands
  constexpr int WK = mlp_wk(AT);                 // K columns per ring stage
  constexpr int ABLK = 128 * WK * 2;             // AT: one stage's A block (128 rows of 128 B)
  const int wstage = N1p * WK * 2;                // one W1 ring stage (N1p rows of 2 WK bytes)
  const int sstride = AT ? ABLK + wstage : wstage;  // ring stage stride
  const int abytes = AT ? 0 : (KB0 > KB1 ? KB0 : KB1) * 128 * 128;
  const int NST = mlp_stages(AT, sstride);
  const int ring = (NST * sstride + 1023) & ~1023;
  uint8_t* sW = smem + abytes;                    // W1 ring (AT: A block + W1 block per stage)
  uint8_t* sA = AT ? sW : smem;                   // A1 (not AT), then A2 (AT: over the drained ring)
  uint8_t* sW2 = sW + ring;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sW2 + KB1 * g.N2p * 128);
  // bars: w2full, wfull[NST], wempty[NST], d1full, d2full, tmem slot
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 3 + 2 * NST);
  __shared__ __align__(16) float sb1[512];
  __shared__ __align__(16) float sb2[256];
  const uint32_t w2full = smem_u32(bars), wfull0 = smem_u32(bars + 1), wempty0 = smem_u32(bars + 1 + NST);
  const uint32_t d1full = smem_u32(bars + 1 + 2 * NST), d2full = smem_u32(bars + 2 + 2 * NST);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, tid = threadIdx.x;
  // rows of this CTA: rpc <= 128 per CTA (the MMAs stay M = 128; rows >= nrows are never
  // stored): small services spread over more SMs, so the per-CTA chain is shorter
  const int rpc = g.rpc > 0 ? g.rpc : 128;
  const int64_t row0 = (int64_t)(blockIdx.x / S) * rpc;
  const int nrows = (int)(g.rows - row0 < rpc ? g.rows - row0 : rpc);
  // Input row i of the CTA is GEMM row arow(i) = (i % 4) * 32 + i / 4: the rows are spread over
  // the four TMEM lane quarters, so every epilogue warp has rows to drain when rpc < 128 (a warp
  // can only read its own quarter's lanes).  Rows arow(i) for i >= nrows are never stored.
  // (AT: the TMA rows are contiguous, so GEMM row = input row and rpc is 128)
  auto arow = [](int i) { return ((i & 3) << 5) | (i >> 2); };
  const int nrows4 = (nrows + 3) & ~3;  // input rows loaded (whole quarters' worth of rows)
  const int nkw = g.K0p / WK;  // W1 ring blocks

  if (tid == 0) {
    mbar_init(w2full, 1);
    for (int s = 0; s < NST; ++s) {
      mbar_init(wfull0 + 8 * s, 1);
      mbar_init(wempty0 + 8 * s, 1);
    }
    mbar_init(d1full, 1);
    mbar_init(d2full, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    fence_proxy_async();
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)), "r"(512u)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  for (int c = tid; c < 512; c += MLP_THREADS) sb1[c] = c < N1 ? __ldg(b1 + n1o + c) : 0.f;
  for (int c = tid; c < 256; c += MLP_THREADS) sb2[c] = c < g.N2 ? __ldg(b2 + c) : 0.f;
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  // weights: W2 whole, and the first ring stages of W1 (never written by earlier kernels)
  auto load_w1 = [&](int kb) {  // (AT: the stage's barrier also expects its A block, load_a)
    const int s = kb % NST;
    const uint32_t dst = smem_u32(sW) + (uint32_t)(s * sstride + (AT ? ABLK : 0));
    mbar_arrive_expect_tx(wfull0 + 8 * s, (uint32_t)(wstage + (AT ? ABLK : 0)));
    const int half = N1p / 2;  // two boxes of N1p / 2 rows
    tma_2d(dst, &tmW1, wfull0 + 8 * s, kb * WK, n1o);
    tma_2d(dst + (uint32_t)(half * WK * 2), &tmW1, wfull0 + 8 * s, kb * WK, n1o + half);
  };
  auto load_a = [&](int kb) {  // AT: rows [row0, row0 + 128) x K columns [32 kb, 32 kb + 32)
    const int s = kb % NST;
    tma_2d(smem_u32(sW) + (uint32_t)(s * sstride), &tmA, wfull0 + 8 * s, kb * WK, (int)row0);
  };
  if (tid == 0) {
    mbar_arrive_expect_tx(w2full, (uint32_t)(KB1 * g.N2p * 128));
    for (int kb = 0; kb < KB1; ++kb) tma_2d(smem_u32(sW2) + (uint32_t)(kb * g.N2p * 128), &tmW2, w2full, n1o + kb * 64, 0);
    for (int kb = 0; kb < NST && kb < nkw; ++kb) load_w1(kb);
  }
  MST(1);
  pdl_wait();  // the input rows and the output buffer belong to earlier kernels of the stream
  MST(2);
  if (AT && tid == 0)
    for (int kb = 0; kb < NST && kb < nkw; ++kb) load_a(kb);

  // ---- 1. fp32 rows -> 16-bit A1 (K-major, 128B swizzle: element (r, k) of block k / 64 at
  // r * 128 + (((k % 64) / 8) ^ (r % 8)) * 16 + (k % 8) * 2); a warp reads one row's floats
  // contiguously, so the global reads are coalesced
  if (!AT) {
    // 4 rows per warp iteration with all their loads in flight before any is used (a row at a
    // time serialised ~80 L2 round trips per warp: 12.5 us of the kernel's 29 us, B200)
    constexpr int RB = 4, KMAX = 384 / 64;  // rows per batch; lane pairs per row (K0p <= 384)
    for (int rb = warp * RB; rb < nrows4; rb += (MLP_THREADS / 32) * RB) {
      float v[RB][KMAX][2];
#pragma unroll
      for (int i = 0; i < RB; ++i) {
        const int r = rb + i;
        const float* xr = x + (row0 + r) * (int64_t)g.K0;
#pragma unroll
        for (int j = 0; j < KMAX; ++j) {
          const int k = lane * 2 + 64 * j;
          v[i][j][0] = (r < nrows && k < g.K0) ? __ldg(xr + k) : 0.f;
          v[i][j][1] = (r < nrows && k + 1 < g.K0) ? __ldg(xr + k + 1) : 0.f;
        }
      }
#pragma unroll
      for (int i = 0; i < RB; ++i) {
        const int r = arow(rb + i);
#pragma unroll
        for (int j = 0; j < KMAX; ++j) {
          const int k = lane * 2 + 64 * j;
          if (k < g.K0p) {
            const int kk = k & 63;
            const uint32_t off = (uint32_t)((k >> 6) * (128 * 128) + r * 128 + (((kk >> 3) ^ (r & 7)) << 4) + (kk & 7) * 2);
            *reinterpret_cast<uint32_t*>(sA + off) = pack2<BF16>(v[i][j][0], v[i][j][1]);
          }
        }
      }
    }
  }
  fence_proxy_async();
  __syncthreads();
  MST(3);

  const uint64_t hi128 = sdesc(0, 128), hi64 = sdesc(0, 64);
  const bool bf = BF16;
  // ---- 2. layer 1 MMAs (thread 0): K steps of 16 over the W1 ring
  if (tid == 0) {
    const int na = N1p > 256 ? 256 : N1p, nb = N1p - na;
    const uint32_t ida = idesc_rt(na, bf), idb = nb ? idesc_rt(nb, bf) : 0u;
    const uint32_t a16 = (smem_u32(sA) & 0x3FFFFu) >> 4, w16 = (smem_u32(sW) & 0x3FFFFu) >> 4;
    for (int kb = 0; kb < nkw; ++kb) {
      const int s = kb % NST;
      mbar_wait(wfull0 + 8 * s, (uint32_t)(kb / NST) & 1);
      tc_fence_after();
#pragma unroll
      for (int k = 0; k < WK / 16; ++k) {
        const int kk = kb * WK + k * 16;  // first K column of this step
        const uint64_t hw = WK == 64 ? hi128 : hi64;  // the ring's swizzle (WK * 2-byte rows)
        const uint64_t ad = AT ? hi128 | (uint64_t)(w16 + (uint32_t)(s * (sstride >> 4)) + (uint32_t)(k * 2))
                               : hi128 | (uint64_t)(a16 + (uint32_t)((kk >> 6) * (128 * 128 / 16) + ((kk & 63) * 2) / 16));
        const uint32_t wb = w16 + (uint32_t)(s * (sstride >> 4) + (AT ? ABLK >> 4 : 0)) + (uint32_t)(k * 2);
        mma_f16(tmem, ad, hw | (uint64_t)wb, ida, (kb | k) != 0);
        if (nb) mma_f16(tmem + (uint32_t)na, ad, hw | (uint64_t)(wb + (uint32_t)((na * WK * 2) >> 4)), idb, (kb | k) != 0);
      }
      mma_commit(wempty0 + 8 * s);
    }
    mma_commit(d1full);
  } else if (tid == 32) {
    // W1 ring refills: stage kb % S is reloaded with block kb + S once its MMAs have completed
    for (int kb = 0; kb + NST < nkw; ++kb) {
      mbar_wait(wempty0 + 8 * (kb % NST), (uint32_t)(kb / NST) & 1);
      load_w1(kb + NST);
      if (AT) load_a(kb + NST);
    }
  }
  MST(4);
  __syncwarp();

  // ---- 3. layer 1 epilogue -> A2 (overwrites A1; its MMAs have completed)
  {
    if (lane == 0) mbar_wait(d1full, 0);
    __syncwarp();
    tc_fence_after();
    const int quarter = warp & 3, cgi = warp >> 2;
    const int r = quarter * 32 + lane;
    const uint32_t tb = tmem + ((uint32_t)(quarter * 32) << 16);
    const int nch = N1p / 16, c0 = cgi * nch / MLP_CG, c1 = (cgi + 1) * nch / MLP_CG;
    uint8_t* a2 = sA;
    // chunk ci: bias + activation -> 16-bit -> A2 (two 16-byte pieces)
    auto emit = [&](int ci, const uint32_t (&rq)[16]) {
      float bq[16], v[16];
      lds16(bq, sb1 + ci * 16);
      bias_act16(v, rq, bq, g.act1);
      const int k = ci * 16;
#pragma unroll
      for (int j = 0; j < 16; ++j) v[j] = k + j < N1 ? v[j] : 0.f;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int kk = (k + 8 * h) & 63;
        const uint32_t off = (uint32_t)(((k + 8 * h) >> 6) * (128 * 128) + r * 128 + (((kk >> 3) ^ (r & 7)) << 4));
        *reinterpret_cast<uint4*>(a2 + off) =
            make_uint4(pack2<BF16>(v[8 * h], v[8 * h + 1]), pack2<BF16>(v[8 * h + 2], v[8 * h + 3]),
                       pack2<BF16>(v[8 * h + 4], v[8 * h + 5]), pack2<BF16>(v[8 * h + 6], v[8 * h + 7]));
      }
    };
    // two chunks per step: the second one's TMEM load is in flight while the first is converted
    // (warps whose 32 rows are all past nrows have nothing to produce)
    const bool act_rows = AT ? quarter * 32 < nrows : quarter < nrows;  // this warp has rows to drain
    for (int ci = c0; ci < c1 && act_rows; ci += 2) {
      uint32_t ra[16], rb2[16];
      tmem_ld16(tb + (uint32_t)(ci * 16), ra);
      if (ci + 1 < c1) tmem_ld16(tb + (uint32_t)((ci + 1) * 16), rb2);
      tmem_wait_ld();
      emit(ci, ra);
      if (ci + 1 < c1) emit(ci + 1, rb2);
    }
    // zero K columns [N1p, K1p) of A2 (W2 is zero there too; 0 * garbage could be NaN)
    for (int k = N1p + 8 * cgi; k < K1p && act_rows; k += 8 * MLP_CG) {
      const int kk = k & 63;
      *reinterpret_cast<uint4*>(a2 + (k >> 6) * (128 * 128) + r * 128 + (((kk >> 3) ^ (r & 7)) << 4)) = make_uint4(0, 0, 0, 0);
    }
  }
  tc_fence_before();
  fence_proxy_async();
  __syncthreads();
  MST(5);

  // ---- 4. layer 2 MMAs (thread 0) into columns [N1c, N1c + N2p)
  const uint32_t d2 = tmem + (uint32_t)N1c;
  if (tid == 0) {
    tc_fence_after();
    mbar_wait(w2full, 0);
    const uint32_t id2 = idesc_rt(g.N2p, bf);
    const uint32_t a16 = (smem_u32(sA) & 0x3FFFFu) >> 4, w16 = (smem_u32(sW2) & 0x3FFFFu) >> 4;
    for (int k = 0; k < K1p; k += 16) {
      const uint64_t ad = hi128 | (uint64_t)(a16 + (uint32_t)((k >> 6) * (128 * 128 / 16) + ((k & 63) * 2) / 16));
      const uint64_t bd = hi128 | (uint64_t)(w16 + (uint32_t)((k >> 6) * (g.N2p * 128 / 16) + ((k & 63) * 2) / 16));
      mma_f16(d2, ad, bd, id2, k != 0);
    }
    mma_commit(d2full);
  }
  MST(8);
  __syncwarp();

  // ---- 5. logits (+ bias) -> shared memory (warps 0-3 own the TMEM lanes: one row each), then
  // every warp takes rows: lanes over the row's N2 <= 64 columns, max / sum by shuffles, and
  // coalesced stores of the probabilities / logits; argmax ties -> lowest index
  float* stg = reinterpret_cast<float*>(sA);  // A's space: layer 2's MMAs have completed
  const int N2 = g.N2, sp = N2 + 1;           // odd pitch: conflict-free column writes
  if (warp < 4 && (AT ? warp * 32 : warp) < nrows) {
    if (lane == 0) mbar_wait(d2full, 0);
    __syncwarp();
    MST(9);
    tc_fence_after();
    const int r = AT ? warp * 32 + lane : 4 * lane + warp;  // the input row of TMEM lane warp * 32 + lane
    const uint32_t tb = d2 + ((uint32_t)(warp * 32) << 16);
    const int nch = g.N2p / 16;
    uint32_t rq[4][16];
#pragma unroll
    for (int ci = 0; ci < 4; ++ci)
      if (ci < nch) tmem_ld16(tb + (uint32_t)(ci * 16), rq[ci]);  // all chunks in flight, one wait
    tmem_wait_ld();
#pragma unroll
    for (int ci = 0; ci < 4; ++ci)
      if (ci < nch) {
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          const int c = ci * 16 + j;
          if (c < N2 && r < nrows) stg[r * sp + c] = __uint_as_float(rq[ci][j]) + (S > 1 ? 0.f : sb2[c]);
        }
      }
  }
  __syncthreads();
  if (S > 1) {
    // split: CTA 0 adds the cluster's partial logits in rank order (DSMEM), then the bias
    cluster_sync();
    if (q == 0)
      for (int e = tid; e < nrows * N2; e += MLP_THREADS) {
        const int r = e / N2, c = e - r * N2;
        const uint32_t a = smem_u32(stg + r * sp + c);
        float z = stg[r * sp + c];
        for (int p = 1; p < S; ++p) {
          uint32_t ra;
          float v;
          asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(a), "r"(p));
          asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(ra) : "memory");
          z += v;
        }
        stg[r * sp + c] = z + sb2[c];
      }
    __syncthreads();
  }
  MST(10);
  // TPR threads per row (interleaved columns; 2 / 4 / 8 as fewer rows leave threads free) for the
  // max / exp / sum, in place in shared memory; shuffles stay within the row's aligned lane group
  if (q == 0) {
    const int rows_max = MLP_THREADS / 2;  // rows covered at 2 threads per row
    const int lt = nrows > rows_max / 2 ? 1 : (nrows > rows_max / 4 ? 2 : (nrows > rows_max / 8 ? 3 : 4)), TPR = 1 << lt;
    const int r = tid >> lt, h = tid & (TPR - 1);
    const bool live = r < nrows;
    float* zr = stg + r * sp;
    float m = -FLT_MAX;
    int mi = 0x7fffffff;
    if (live)
      for (int c = h; c < N2; c += TPR) {
        const float v = zr[c];
        if (v > m || (v == m && c < mi)) { m = v; mi = c; }
      }
    for (int o = 1; o < TPR; o <<= 1) {
      const float m2 = __shfl_xor_sync(0xffffffffu, m, o);
      const int i2 = __shfl_xor_sync(0xffffffffu, mi, o);
      if (m2 > m || (m2 == m && i2 < mi)) { m = m2; mi = i2; }
    }
    if (g.out_mode == 1) {
      if (h == 0 && live) reinterpret_cast<int*>(out)[row0 + r] = mi;
    } else if (g.out_mode == 0) {
      // The row sum in an order that does not depend on TPR (so a row's probabilities are bitwise
      // the same whatever the batch size or rows per CTA): 16 partial sums over the columns
      // c = p (mod 16), each in increasing c, then a fixed binary tree (p + 8, p + 4, p + 2, p + 1);
      // the tree levels of stride >= TPR run inside the thread, the rest by shuffles.
      float part[8];
      const int PPT = 16 / TPR;  // partials per thread: p = h + TPR * j
#pragma unroll
      for (int j = 0; j < 8; ++j) part[j] = 0.f;
      if (live)
        for (int c = h; c < N2; c += TPR) {
          const float e = expf(zr[c] - m);
          zr[c] = e;
          const int j = (c & 15) / TPR;
#pragma unroll
          for (int q = 0; q < 8; ++q)
            if (q == j) part[q] += e;
        }
#pragma unroll
      for (int st = 8; st >= 1; st >>= 1)
        if (st >= TPR) {
#pragma unroll
          for (int j = 0; j < 8; ++j)
            if (j < st / TPR && j < PPT) part[j] = part[j] + part[j + st / TPR];
        }
      float sum = part[0];
      for (int o = TPR / 2; o >= 1; o >>= 1) sum = sum + __shfl_xor_sync(0xffffffffu, sum, o);
      const float inv = 1.f / sum;
      if (live)
        for (int c = h; c < N2; c += TPR) zr[c] *= inv;
    }
  }
  if (g.out_mode != 1 && q == 0) {
    __syncthreads();
    // coalesced stores: a warp writes whole rows (lanes over columns)
    for (int r = warp; r < nrows; r += MLP_THREADS / 32) {
      float* o = reinterpret_cast<float*>(out) + (row0 + r) * N2;
      for (int c = lane; c < N2; c += 32) o[c] = stg[r * sp + c];
    }
  }
  MST(6);
  tc_fence_before();
  if (S > 1) cluster_sync();  // CTA 0 has read every peer's partial logits
  __syncthreads();
  MST(7);
#ifdef DJINN_MLP_STATS
  if (tid == 0 && blockIdx.x == 0)
    printf("[mlp] prologue %lld pdlwait %lld load %lld l1mma %lld l1epi %lld l2issue %lld d2wait %lld logits %lld softmax %lld tail %lld\n",
           ts[1] - ts[0], ts[2] - ts[1], ts[3] - ts[2], ts[4] - ts[3], ts[5] - ts[4], ts[8] - ts[5], ts[9] - ts[8],
           ts[10] - ts[9], ts[6] - ts[10], ts[7] - ts[6]);
#endif
  if (warp == 0) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512u) : "memory");
  }
}

}  // namespace

int mlp2_smem(const MlpGeom& g) {
  const int KB0 = g.K0p / 64, KB1 = g.K1p / 64;
  const int abytes = g.a_tma ? 0 : (KB0 > KB1 ? KB0 : KB1) * 128 * 128;
  const int wk = mlp_wk(g.a_tma);
  const int sstride = g.N1p * wk * 2 + (g.a_tma ? 128 * wk * 2 : 0);
  return 1024 + abytes + ((mlp_stages(g.a_tma, sstride) * sstride + 1023) & ~1023) + KB1 * g.N2p * 128 +
         (4 + 2 * MLP_MAXST) * 8 + 16;
}

int mlp2_rows_per_cta(int64_t rows) {
  static const int env = [] {
    const char* e = getenv("DJINN_MLP_RPC");
    return e ? atoi(e) : 0;
  }();
  if (env > 0) return env;
  const int64_t sms = tc_num_sms();
  for (int rpc = 32; rpc < 128; rpc *= 2)
    if ((rows + rpc - 1) / rpc <= sms) return rpc;
  return 128;
}

int mlp2_wk(int a_tma) { return mlp_wk(a_tma != 0); }

bool mlp2_supported(const MlpGeom& g) {
  const int S = g.nsplit > 1 ? g.nsplit : 1;
  if (S > 1 && (!g.a_tma || S > 8 || g.N1p % (16 * S) || g.N1p / S > 256 || g.N1p / S < 32)) return false;
  return g.K0p % 64 == 0 && g.K1p % 64 == 0 && g.N1p % 16 == 0 && g.N1p >= g.N1 && g.N1p <= 512 &&
         (g.N1p <= 256 || (g.N1p - 256) % 16 == 0) && g.N1p / 2 <= 256 && g.K1p >= g.N1p && g.N2p % 16 == 0 &&
         g.N2p >= g.N2 && g.N2p <= 64 && g.N1c % 16 == 0 && (g.N1c >= g.N1p || g.N1c == 0) &&
         g.N1c + g.N2p <= 512 && (!g.a_tma || mlp_stages(true, (g.N1p + 128) * MLP_WK_AT * 2) * (g.N1p + 128) * MLP_WK_AT * 2 >= g.K1p / 64 * 128 * 128) &&
         mlp2_smem(g) <= 227 * 1024 - 3 * 1024;
}

cudaError_t launch_mlp2(const MlpGeom& g, int dt, const CUtensorMap* tmW1, const CUtensorMap* tmW2, const CUtensorMap* tmA,
                        const float* x, const float* b1, const float* b2, void* out, cudaStream_t st) {
  if (g.rows <= 0) return cudaSuccess;
  if (!mlp2_supported(g)) return cudaErrorInvalidValue;
  const int smem = mlp2_smem(g);
  const int rpc = g.rpc > 0 ? g.rpc : 128;
  if (rpc > 128 || rpc % 8 || (g.a_tma && rpc != 128)) return cudaErrorInvalidValue;
  const unsigned grid = (unsigned)((g.rows + rpc - 1) / rpc);
  // the max-dynamic-smem attribute is set once per (device, kernel): a cudaFuncSetAttribute per
  // call was a measurable part of the ~10 us host cost of a small service's forward
  if (g.a_tma && !tmA) return cudaErrorInvalidValue;
  auto kern = dt == DT_BF16 ? (g.a_tma ? mlp2_kernel<true, true> : mlp2_kernel<true, false>)
                            : (g.a_tma ? mlp2_kernel<false, true> : mlp2_kernel<false, false>);
  cudaError_t e = ensure_max_smem((const void*)kern, 227 * 1024 - 3 * 1024);
  if (e != cudaSuccess) return e;
  const int S = g.nsplit > 1 ? g.nsplit : 1;
  if (S == 1)
    return launch_pdl(kern, dim3(grid), dim3(MLP_THREADS), smem, st, *tmW1, *tmW2, g.a_tma ? *tmA : *tmW1, g, x, b1, b2,
                      out);
  cudaLaunchConfig_t cfg = {};  // split: clusters of S CTAs per 128-row block
  cfg.gridDim = dim3(grid * (unsigned)S);
  cfg.blockDim = dim3(MLP_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = (unsigned)S;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, *tmW1, *tmW2, *tmA, g, x, b1, b2, out);
}

}  // namespace djinn
