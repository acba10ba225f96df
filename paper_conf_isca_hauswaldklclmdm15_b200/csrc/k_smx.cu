// K1 + K6 fused for a wide last layer (ASR's 8000 senones): z = x W^T + b, then the row softmax
// (or the row argmax, or the logits) written straight from the tensor-memory accumulators.
//
// What it computes ("the DNN's output ... probabilities"; Table 3: ASR returns
// a probability vector over the senones per frame; SURVEY.md 8(a) a7 + a8):
//     z[m][n] = b[n] + sum_k x[m][k] W[n][k]          p[m][n] = exp(z[m][n] - max_j z[m][j]) / sum_j exp(...)
// The unfused path writes z in fp32 (ASR: 262 MB) and a softmax kernel reads it back and writes
// p (262 MB): two thirds of the layer's HBM traffic exist only to carry z between two kernels.
//
// Structure (B200): one thread-block CLUSTER of CL CTAs (CL <= 16, non-portable size) owns a
// block of 128 rows and ALL N columns: CTA rank r computes columns [r*NCW, r*NCW + NCW) (NCW <=
// 512 = the whole 512-column tensor memory of its SM) with tcgen05.mma.cta_group::1 (M = 128,
// N <= 256 per instruction, two instructions per K step).  The A tile (128 rows x 32 K) is the
// same for every CTA of the cluster: each CTA loads 128 / CL of its rows and MULTICASTS them to
// all CTAs (one L2 read per cluster instead of CL), so a stage is A 8 KB + B 32 KB (SW64, 5
// stages).  Every CTA's MMA commit arrives on the stage-empty barrier of EVERY CTA (a stage may be
// refilled only when no CTA of the cluster still reads it).
// Epilogue (8 warps: TMEM lane quarter x column half): row max over the CTA's columns -> shared
// memory -> cluster barrier -> each CTA reads the CL x 2 partial maxima of its rows from its peers'
// shared memory (DSMEM) -> e = 2^((z - max) log2 e), row sums, e written back into tensor memory ->
// cluster barrier -> the peers' partial sums -> p = e / sum, staged per warp in shared memory and
// stored as whole 128-byte row segments.  z never reaches HBM.
#include "tc_common.cuh"
#include <cstdio>

namespace djinn {
namespace {

#ifndef DJINN_SMX_BK
#define DJINN_SMX_BK 32
#endif
constexpr int SMX_BK = DJINN_SMX_BK;       // K per stage: 32 (64-byte rows, SW64) or 64 (128-byte rows, SW128)
constexpr int SMX_RB = SMX_BK * 2;         // bytes per operand row of a stage
constexpr int SMX_STAGES = SMX_BK == 32 ? 5 : 2;
constexpr int SMX_A_BYTES = 128 * SMX_RB;  // 128 rows x BK x 2 B
constexpr int SMX_B_BYTES = 512 * SMX_RB;  // 512 rows x BK x 2 B (two 256-row boxes)
constexpr int SMX_STAGE = SMX_A_BYTES + SMX_B_BYTES;
#ifndef DJINN_SMX_MC
#define DJINN_SMX_MC 1
#endif
constexpr bool SMX_MC = DJINN_SMX_MC != 0;  // A multicast across the cluster (else every CTA loads its own A)
constexpr int SMX_THREADS = 320;           // warps 0-7 epilogue, 8 TMA producer, 9 MMA + TMEM owner
constexpr int SMX_STG_PITCH = 36;          // floats per staged row (144 B: odd multiple of 16 B)
constexpr int SMX_SMEM = 1024 + SMX_STAGES * SMX_STAGE + 512 * 4 + 3 * 2 * 128 * 4 + 16 * 8;
static_assert(8 * 32 * 36 * 4 <= SMX_STAGES * SMX_STAGE, "epilogue staging fits in the stage ring");

__device__ __forceinline__ void tma_2d_mc(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1,
                                          uint16_t mask) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster"
      " [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(dst),
      "l"((uint64_t)map), "r"(bar), "r"(c0), "r"(c1), "h"(mask)
      : "memory");
}
__device__ __forceinline__ void mma_commit_mc(uint32_t bar, uint16_t mask) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
                   bar),
               "h"(mask)
               : "memory");
}
__device__ __forceinline__ uint32_t mapa(uint32_t addr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
  return r;
}
__device__ __forceinline__ float ld_dsmem_f32(uint32_t addr) {
  float v;
  asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ int ld_dsmem_s32(uint32_t addr) {
  int v;
  asm volatile("ld.shared::cluster.s32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], "
      "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
      : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#ifdef DJINN_SMX_STATS
#define SMX_T(i) if (threadIdx.x == 0) tt[i] = gtimer()
#else
#define SMX_T(i)
#endif

template <bool BF16>
__global__ void __launch_bounds__(SMX_THREADS, 1)
    smx_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, const SmxGeom g,
               const float* __restrict__ bias, void* __restrict__ out) {
  pdl_trigger();
#ifdef DJINN_SMX_STATS
  uint64_t tt[8] = {0};
#endif
  SMX_T(0);
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  float* sbias = reinterpret_cast<float*>(smem + SMX_STAGES * SMX_STAGE);
  float* xm = sbias + 512;                       // [2 halves][128 rows] partial row max
  int* xi = reinterpret_cast<int*>(xm + 256);    // [2][128] its column (argmax)
  float* xs = reinterpret_cast<float*>(xi + 256);  // [2][128] partial sum of exponentials
  uint64_t* bars = reinterpret_cast<uint64_t*>(xs + 256);
  // bars: full[5], empty[5], tfull, tmem slot
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 11);
  const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + SMX_STAGES), tfull = smem_u32(bars + 2 * SMX_STAGES);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_rank();
  const int CL = g.CL;
  const uint16_t all = (uint16_t)((1u << CL) - 1u);
  const int rblk = blockIdx.x / CL;
  const int64_t row0 = (int64_t)rblk * 128;
  const int c0 = (int)rank * g.NCW;                         // first global column of this CTA
  const int ncc = min(g.NCW, g.N - c0);                     // valid columns (> 0 by construction)
  const int nmma = (ncc + 15) & ~15;                        // MMA width (16-column multiple)
  const int n1 = min(nmma, 256), n2 = nmma - n1;
  const int KB = g.Kpad / SMX_BK;
  const int slice = 128 / CL;                               // A rows this CTA loads and multicasts

  if (warp == 8 && lane == 0) {
    for (int s = 0; s < SMX_STAGES; ++s) {
      mbar_init(full0 + 8 * s, 1);
      mbar_init(empty0 + 8 * s, SMX_MC ? (uint32_t)CL : 1u);  // MC: one commit from every CTA of the cluster
    }
    mbar_init(tfull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmB) : "memory");
  }
  if (warp == 9) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)), "r"(512u)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  // weights and bias are never written by an earlier kernel: read before the PDL wait
  for (int c = threadIdx.x; c < 512; c += SMX_THREADS) sbias[c] = c < ncc ? __ldg(bias + c0 + c) : 0.f;
  tc_fence_before();
  cluster_sync();  // every CTA's barriers are initialised before any peer multicasts into them
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  SMX_T(1);

  if (warp == 8) {
    // ---- producer: A slice (multicast to the cluster) + this CTA's B columns per 32-K stage
    if (elect_one()) {
      pdl_wait();  // x is the previous layer's output
      const uint32_t bbytes = (uint32_t)((nmma + 255) / 256) * 256u * (uint32_t)SMX_RB;
      for (int kb = 0; kb < KB; ++kb) {
        const int s = kb % SMX_STAGES;
        mbar_wait(empty0 + 8 * s, ((uint32_t)(kb / SMX_STAGES) & 1) ^ 1);
        const uint32_t st = smem_u32(smem) + (uint32_t)(s * SMX_STAGE);
        mbar_arrive_expect_tx(full0 + 8 * s, (uint32_t)SMX_A_BYTES + bbytes);
        if (SMX_MC)
          tma_2d_mc(st + (uint32_t)(rank * slice * SMX_RB), &tmA, full0 + 8 * s, kb * SMX_BK, (int)(row0 + rank * slice), all);
        else
          for (int q = 0; q < CL; ++q)
            tma_2d(st + (uint32_t)(q * slice * SMX_RB), &tmA, full0 + 8 * s, kb * SMX_BK, (int)(row0 + q * slice));
        for (int h = 0; 256 * h < nmma; ++h)
          tma_2d(st + SMX_A_BYTES + (uint32_t)(h * 256 * SMX_RB), &tmB, full0 + 8 * s, kb * SMX_BK, c0 + 256 * h);
      }
    }
    __syncwarp();
  } else if (warp == 9) {
    // ---- MMA issue: 2 K steps of 16 per stage, columns [0, n1) and [256, 256 + n2)
    const uint32_t ab = BF16 ? 1u : 0u;
    const uint32_t id1 = (1u << 4) | (ab << 7) | (ab << 10) | ((uint32_t)(n1 >> 3) << 17) | (8u << 24);
    const uint32_t id2 = (1u << 4) | (ab << 7) | (ab << 10) | ((uint32_t)(n2 >> 3) << 17) | (8u << 24);
    for (int kb = 0; kb < KB; ++kb) {
      const int s = kb % SMX_STAGES;
      mbar_wait(full0 + 8 * s, (uint32_t)(kb / SMX_STAGES) & 1);
      tc_fence_after();
      if (elect_one()) {
        const uint32_t st = smem_u32(smem) + (uint32_t)(s * SMX_STAGE);
        const uint64_t ad = sdesc(st, SMX_RB), bd = sdesc(st + SMX_A_BYTES, SMX_RB);
        const uint64_t bd2 = sdesc(st + SMX_A_BYTES + 256 * SMX_RB, SMX_RB);
#pragma unroll
        for (int k = 0; k < SMX_BK / 16; ++k) {
          mma_f16(tmem, ad + 2 * k, bd + 2 * k, id1, (kb | k) != 0);
          if (n2 > 0) mma_f16(tmem + 256, ad + 2 * k, bd2 + 2 * k, id2, (kb | k) != 0);
        }
        if (SMX_MC) mma_commit_mc(empty0 + 8 * s, all);  // stage s free in every CTA once all have committed
        else mma_commit(empty0 + 8 * s);
        if (kb == KB - 1) mma_commit(tfull);
      }
      __syncwarp();
    }
  }

  // ---- epilogue: thread = row 32 * quarter + lane, columns [256 h, 256 h + 256) of the CTA's
  const int quarter = warp & 3, h = warp >> 2;
  const int r = quarter * 32 + lane;
  const int64_t grow = row0 + r;
  const bool epi = warp < 8;
  const uint32_t tb = tmem + ((uint32_t)(quarter * 32) << 16);
  const int cb = 256 * h, ce = min(cb + 256, ncc);          // this warp's columns (CTA-local)
  const float L2E = 1.4426950408889634f;
  float* stg = reinterpret_cast<float*>(smem) + warp * 32 * SMX_STG_PITCH;  // stages are drained by then
  // 32 columns [c, c + 32) of this thread's row (v[j] for column c + j) -> HBM as whole 128-byte
  // row segments: staged per warp, then each instruction writes 4 rows x 128 B
  auto store32 = [&](int c, const float (&v)[32]) {
    __syncwarp();
#pragma unroll
    for (int q = 0; q < 8; ++q)
      *reinterpret_cast<float4*>(stg + lane * SMX_STG_PITCH + 4 * q) = make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
    __syncwarp();
    const int gc = c0 + c + 4 * (lane & 7);
    float* o = reinterpret_cast<float*>(out);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int rr = 4 * i + (lane >> 3);
      const int64_t orow = row0 + quarter * 32 + rr;
      const float4 x4 = *reinterpret_cast<const float4*>(stg + rr * SMX_STG_PITCH + 4 * (lane & 7));
      if (orow < g.M && gc < g.N) *reinterpret_cast<float4*>(o + orow * g.N + gc) = x4;  // N % 4 == 0
    }
  };
  auto load32 = [&](int c, float (&v)[32]) {  // z = acc + b (fp32), columns >= ncc -> -inf
    uint32_t a0[16], a1[16];
    tmem_ld16(tb + (uint32_t)c, a0);
    tmem_ld16(tb + (uint32_t)(c + 16), a1);
    tmem_wait_ld();
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      v[j] = c + j < ncc ? __uint_as_float(a0[j]) + sbias[c + j] : -INFINITY;
      v[16 + j] = c + 16 + j < ncc ? __uint_as_float(a1[j]) + sbias[c + 16 + j] : -INFINITY;
    }
  };

  float m = -INFINITY;
  int mi = 0x7fffffff;
  if (epi) {
    if (lane == 0) mbar_wait_sleep(tfull, 0);
    __syncwarp();
    SMX_T(2);
    tc_fence_after();
    for (int c = cb; c < ce; c += 32) {
      float v[32];
      load32(c, v);
      if (g.out_mode == 2) {
        store32(c, v);
        continue;
      }
#pragma unroll
      for (int j = 0; j < 32; ++j)
        if (v[j] > m) { m = v[j]; mi = c0 + c + j; }  // first (lowest) column of the maximum
    }
    xm[h * 128 + r] = m;
    xi[h * 128 + r] = mi;
  }
  SMX_T(3);
  cluster_sync();  // #1: every CTA's partial maxima are published
  SMX_T(4);
  if (g.out_mode != 2 && epi) {
    // the row's maximum over the cluster's columns, peers in column order (ties -> lowest column)
    m = -INFINITY;
    mi = 0x7fffffff;
    const uint32_t am = smem_u32(xm + r), ai = smem_u32(xi + r);
    for (int p = 0; p < CL; ++p)
#pragma unroll
      for (int hh = 0; hh < 2; ++hh) {
        const float pm = ld_dsmem_f32(mapa(am + 512u * hh, (uint32_t)p));
        const int pi = ld_dsmem_s32(mapa(ai + 512u * hh, (uint32_t)p));
        if (pm > m || (pm == m && pi < mi)) { m = pm; mi = pi; }
      }
    if (g.out_mode == 1) {
      if (rank == 0 && h == 0 && grow < g.M) reinterpret_cast<int*>(out)[grow] = mi;
    } else {
      // e = 2^(z log2e - max log2e) kept in tensor memory; partial sums
      const float mb = -m * L2E;
      float s = 0.f;
      for (int c = cb; c < ce; c += 32) {
        float v[32];
        load32(c, v);
        uint32_t e0[16], e1[16];
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          const float x0 = ex2_ftz(fmaf(v[j], L2E, mb)), x1 = ex2_ftz(fmaf(v[16 + j], L2E, mb));
          s += x0 + x1;
          e0[j] = __float_as_uint(x0);
          e1[j] = __float_as_uint(x1);
        }
        tmem_st16(tb + (uint32_t)c, e0);
        tmem_st16(tb + (uint32_t)(c + 16), e1);
      }
      tmem_wait_st();
      xs[h * 128 + r] = s;
    }
  }
  SMX_T(5);
  cluster_sync();  // #2: partial sums published (and every peer is done reading xm / xi)
  SMX_T(6);
  if (g.out_mode == 0 && epi) {
    float S = 0.f;
    const uint32_t as = smem_u32(xs + r);
    for (int p = 0; p < CL; ++p)
#pragma unroll
      for (int hh = 0; hh < 2; ++hh) S += ld_dsmem_f32(mapa(as + 512u * hh, (uint32_t)p));
    const float inv = 1.f / S;
    tc_fence_after();
    for (int c = cb; c < ce; c += 32) {
      uint32_t a0[16], a1[16];
      tmem_ld16(tb + (uint32_t)c, a0);
      tmem_ld16(tb + (uint32_t)(c + 16), a1);
      tmem_wait_ld();
      float v[32];
#pragma unroll
      for (int j = 0; j < 16; ++j) {
        v[j] = __uint_as_float(a0[j]) * inv;
        v[16 + j] = __uint_as_float(a1[j]) * inv;
      }
      store32(c, v);
    }
  }
  SMX_T(7);
#ifdef DJINN_SMX_STATS
  if (threadIdx.x == 0 && (blockIdx.x < 2 || blockIdx.x == 500 || blockIdx.x == 1023))
    printf("[smx cta %d] setup %llu mainloop %llu phase1 %llu sync1 %llu phase2 %llu sync2 %llu phase3 %llu ns (start %llu)\n",
           blockIdx.x, tt[1] - tt[0], tt[2] - tt[1], tt[3] - tt[2], tt[4] - tt[3], tt[5] - tt[4], tt[6] - tt[5],
           tt[7] - tt[6], tt[0] % 100000000ull);
#endif
  tc_fence_before();
  cluster_sync();  // #3: no CTA leaves while a peer may still read its shared memory
  if (warp == 9) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512u) : "memory");
  }
}

template <bool BF16>
cudaError_t launch_smx_inst(const SmxGeom& g, const CUtensorMap* tmA, const CUtensorMap* tmB, const float* bias,
                            void* out, cudaStream_t st) {
  auto kern = smx_kernel<BF16>;
  cudaError_t e = ensure_max_smem((const void*)kern, SMX_SMEM);
  if (e != cudaSuccess) return e;
  static int np_set[64] = {0};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 64 && !np_set[dev]) {
    e = cudaFuncSetAttribute((const void*)kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) return e;
    np_set[dev] = 1;
  }
  const int rblocks = (int)((g.M + 127) / 128);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(rblocks * g.CL));
  cfg.blockDim = dim3(SMX_THREADS);
  cfg.dynamicSmemBytes = SMX_SMEM;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = (unsigned)g.CL;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, *tmA, *tmB, g, bias, out);
}

}  // namespace

int smx_bk() { return SMX_BK; }
bool smx_plan(int N, int Kpad, int* CL, int* NCW) {
  if (N < 1024 || N % 4 || Kpad % SMX_BK) return false;
  const int need = (N + 511) / 512;
  int cl = 1;
  while (cl < need) cl *= 2;
  if (cl > 16) return false;
  const int ncw = (((N + cl - 1) / cl) + 15) & ~15;
  if (ncw > 512 || (int64_t)(cl - 1) * ncw >= N) return false;  // every CTA owns >= 1 column
  *CL = cl;
  *NCW = ncw;
  return true;
}

int smx_max_active_clusters(int dt, int CL) {
  auto kern = dt == DT_BF16 ? smx_kernel<true> : smx_kernel<false>;
  if (ensure_max_smem((const void*)kern, SMX_SMEM) != cudaSuccess) return 0;
  if (cudaFuncSetAttribute((const void*)kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(CL * 8));
  cfg.blockDim = dim3(SMX_THREADS);
  cfg.dynamicSmemBytes = SMX_SMEM;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = (unsigned)CL;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, (const void*)kern, &cfg) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return n;
}

cudaError_t launch_smx(const SmxGeom& g, int dt, const CUtensorMap* tmA, const CUtensorMap* tmB, const float* bias,
                       void* out, cudaStream_t st) {
  if (g.M <= 0) return cudaSuccess;
  if (g.CL < 1 || g.CL > 16 || (g.CL & (g.CL - 1)) || g.NCW > 512 || g.NCW % 16 || g.N % 4 || g.Kpad % SMX_BK ||
      (int64_t)(g.CL - 1) * g.NCW >= g.N || (int64_t)g.CL * g.NCW < g.N || g.out_mode < 0 || g.out_mode > 2)
    return cudaErrorInvalidValue;
  if (dt == DT_BF16) return launch_smx_inst<true>(g, tmA, tmB, bias, out, st);
  return launch_smx_inst<false>(g, tmA, tmB, bias, out, st);
}

}  // namespace djinn
