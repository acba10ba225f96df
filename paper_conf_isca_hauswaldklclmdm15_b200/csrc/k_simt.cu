// K7: SIMT fp32 implicit GEMM for conv / locally-connected / fully-connected layers
// (SURVEY.md sec 2.3 "fp32 reference GPU path").  Exact fp32 FFMA accumulation (never
// TF32: SURVEY.md sec 8(c) shows 1xTF32 misses the 1e-4 fp32 contract by 100x).
// The layer algebra is that of PAPER.md L63-65 (weighted sums over a neuron's inputs,
// kernels convolved with the image) in Caffe's definitions (L77): see kernels.h GemmGeom.
#include <math.h>

#include "kernels.h"

namespace djinn {

namespace {
constexpr int TM = 64, TN = 64, TK = 16, NT = 256;

__device__ __forceinline__ float act_f32(float v, int act) {
  switch (act) {
    case ACT_RELU: return v > 0.f ? v : 0.f;
    case ACT_SIGMOID: return 1.f / (1.f + expf(-v));
    case ACT_TANH: return tanhf(v);
    case ACT_HARDTANH: return fminf(fmaxf(v, -1.f), 1.f);
    default: return v;
  }
}

__global__ void __launch_bounds__(NT) simt_gemm_kernel(GemmGeom g, const float* __restrict__ A,
                                                       const float* __restrict__ B,
                                                       const float* __restrict__ bias,
                                                       float* __restrict__ Y) {
  pdl_trigger();
  pdl_wait();
  __shared__ float As[TK][TM + 4];
  __shared__ float Bs[TK][TN + 4];
  const int t = threadIdx.x;
  const int m0 = blockIdx.x * TM, n0 = blockIdx.y * TN, z = blockIdx.z;
  const int tx = t % 16, ty = t / 16;

  // Per-thread A-load rows (4 rows of the tile, fixed across the K loop).
  int a_img[4], a_iy0[4], a_ix0[4];
  bool a_ok[4];
  const int kk_local = t % 16;
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    const int row = (t + NT * e) / 16;
    const int m = m0 + row;
    a_ok[e] = m < g.M;
    int img = m, oy = 0, ox = 0;
    if (g.mode == GM_CONV) {
      img = m / (g.OH * g.OW);
      const int rem = m - img * g.OH * g.OW;
      oy = rem / g.OW;
      ox = rem - oy * g.OW;
    } else if (g.mode == GM_LC) {
      oy = z / g.OW;
      ox = z - oy * g.OW;
    }
    a_img[e] = img;
    a_iy0[e] = oy * g.stride - g.pad;
    a_ix0[e] = ox * g.stride - g.pad;
  }
  const int cin_off = (g.mode == GM_CONV) ? z * g.cin_goff : 0;
  const float* Bz = B + (int64_t)z * g.N * g.K;

  float acc[4][4] = {};
  for (int k0 = 0; k0 < g.K; k0 += TK) {
    // A tile: element (row, kk) with kk = t % 16.
    const int k = k0 + kk_local;
    int ky = 0, kx = 0, c = k;
    if (g.mode != GM_DENSE) {
      const int tap = k / g.Cgp;
      c = k - tap * g.Cgp;
      ky = tap / g.KW;
      kx = tap - ky * g.KW;
    }
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int row = (t + NT * e) / 16;
      float v = 0.f;
      if (a_ok[e] && k < g.K) {
        if (g.mode == GM_DENSE) {
          v = __ldg(A + (int64_t)a_img[e] * g.a_pitch + k);
        } else {
          const int iy = a_iy0[e] + ky, ix = a_ix0[e] + kx;
          if (iy >= 0 && iy < g.H && ix >= 0 && ix < g.W)
            v = __ldg(A + (((int64_t)a_img[e] * g.H + iy) * g.W + ix) * g.Cp_in + cin_off + c);
        }
      }
      As[kk_local][row] = v;
    }
    // B tile: (n, kk)
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int idx = t + NT * e;
      const int n = idx / 16, kk = idx % 16;
      const int gn = n0 + n, gk = k0 + kk;
      Bs[kk][n] = (gn < g.N && gk < g.K) ? __ldg(Bz + (int64_t)gn * g.K + gk) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < TK; ++kk) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[kk][ty * 4 + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) b[j] = Bs[kk][tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }

#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int m = m0 + ty * 4 + i;
    if (m >= g.M) continue;
    const int64_t pix = (g.mode == GM_LC) ? (int64_t)m * g.OH * g.OW + z : m;
    float* yrow = Y + pix * g.out_pitch + (int64_t)z * g.cout_goff * (g.mode == GM_CONV);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int n = n0 + tx * 4 + j;
      if (n < g.N) yrow[n] = act_f32(acc[i][j] + bias[(int64_t)z * g.bias_zstride + n], g.act);
      else if (n < g.write_cols) yrow[n] = 0.f;
    }
  }
}
}  // namespace

cudaError_t launch_simt_gemm(const GemmGeom& g, const float* A, const float* B, const float* bias,
                             float* Y, cudaStream_t st) {
  dim3 grid((g.M + TM - 1) / TM, (max(g.N, g.write_cols) + TN - 1) / TN, g.Z);
  launch_pdl(simt_gemm_kernel, dim3(grid), dim3(NT), 0, st, g, A, B, bias, Y);
  return cudaGetLastError();
}

}  // namespace djinn
