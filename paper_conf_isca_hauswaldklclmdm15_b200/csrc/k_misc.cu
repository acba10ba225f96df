// Memory-bound kernels of the hot path:
//   K0 input pack, K4 LRN, K5 pooling, K6 softmax/argmax.
// All activations are NHWC with channel pitch Cp; math is fp32 whatever the storage type.
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <float.h>
#include <stdlib.h>

#include <algorithm>

#include "kernels.h"

namespace djinn {

template <typename T> __device__ __forceinline__ float ld(const T* p);
template <> __device__ __forceinline__ float ld<float>(const float* p) { return *p; }
template <> __device__ __forceinline__ float ld<__half>(const __half* p) { return __half2float(*p); }
template <> __device__ __forceinline__ float ld<__nv_bfloat16>(const __nv_bfloat16* p) {
  return __bfloat162float(*p);
}
template <typename T> __device__ __forceinline__ T cvt(float v);
template <> __device__ __forceinline__ float cvt<float>(float v) { return v; }
template <> __device__ __forceinline__ __half cvt<__half>(float v) { return __float2half_rn(v); }
template <> __device__ __forceinline__ __nv_bfloat16 cvt<__nv_bfloat16>(float v) {
  return __float2bfloat16_rn(v);
}

static inline int nblocks(int64_t n, int t) { return (int)((n + t - 1) / t); }

// ------------------------------------------------------------------------------------------
// K0: fp32 NCHW [rows][C][H][W] -> NHWC [rows][Ho][Wo][Cp] (16-bit), 8 channels per thread,
// with the optional first-layer transforms (space-to-depth, kx-unroll) that give the first
// convolution a dense, 16-element-aligned K (DESIGN.md sec 5 "first layer").
// Vector inputs (C x 1 x 1: ASR frames, NLP windows): one thread per 8-channel chunk of the
// flattened (row, chunk) space, two float4 loads when the row is 16-byte aligned.  The general
// kernel below gives each row its own block, and a 448-channel row is only 56 chunks (ASR pack
// 13.5 us for 8192 frames: mostly idle warps).
template <typename T>
__global__ void pack16_vec_kernel(const float* __restrict__ x, T* __restrict__ y, int64_t rows, int C, int Cp) {
  pdl_trigger();
  pdl_wait();
  const int chunks = Cp / 8;
  const int64_t total = rows * chunks;
  const bool vec = (C % 4) == 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / chunks;
    const int c0 = (int)(i - r * chunks) * 8;
    const float* src = x + r * C + c0;
    float f[8];
    if (vec && c0 + 8 <= C) {
      const float4 a = __ldg(reinterpret_cast<const float4*>(src)), b = __ldg(reinterpret_cast<const float4*>(src + 4));
      f[0] = a.x; f[1] = a.y; f[2] = a.z; f[3] = a.w; f[4] = b.x; f[5] = b.y; f[6] = b.z; f[7] = b.w;
    } else {
#pragma unroll
      for (int j = 0; j < 8; ++j) f[j] = c0 + j < C ? __ldg(src + j) : 0.f;
    }
    __align__(16) T v[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) v[j] = cvt<T>(f[j]);
    reinterpret_cast<uint4*>(y)[i] = *reinterpret_cast<const uint4*>(v);
  }
}

template <typename T>
__global__ void pack16_kernel(const float* __restrict__ x, T* __restrict__ y, int64_t rows, int C, int H, int W,
                              int mode, int f, int xs, int Ho, int Wo, int Cp) {
  pdl_trigger();
  pdl_wait();
  const int chunks = Cp / 8;
  const int per_row = Ho * Wo * chunks;  // 32-bit index math inside a row
  for (int64_t r = blockIdx.y; r < rows; r += gridDim.y) {
    const float* src = x + r * C * (int64_t)H * W;
    T* dst = y + r * (int64_t)per_row * 8;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < per_row; i += gridDim.x * blockDim.x) {
      const int ch = i % chunks;
      const int pix = i / chunks;
      const int yo = pix / Wo, xo = pix - (pix / Wo) * Wo;
      __align__(16) T v[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const int cc = ch * 8 + j;
        int c = cc, yy = yo, xx = xo;
        bool ok;
        if (mode == 0) {
          ok = cc < C;
        } else if (mode == 1) {
          const int d = cc / C;
          c = cc - d * C;
          yy = yo * f + d / f;
          xx = xo * f + d % f;
          ok = d < f * f && yy < H && xx < W;
        } else {
          const int kx = cc / C;
          c = cc - kx * C;
          xx = xo * xs + kx;
          ok = kx < f && xx < W;
        }
        v[j] = cvt<T>(ok ? __ldg(src + (c * H + yy) * W + xx) : 0.f);
      }
      *reinterpret_cast<uint4*>(dst + i * 8) = *reinterpret_cast<uint4*>(v);
    }
  }
}

// fp32 storage: one element per thread, (row, pixel, c) order -> coalesced writes.
__global__ void pack32_kernel(const float* __restrict__ x, float* __restrict__ y, int64_t rows,
                              int C, int HW, int Cp) {
  pdl_trigger();
  pdl_wait();
  const int64_t total = rows * (int64_t)HW * Cp;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int c = (int)(i % Cp);
    const int64_t t = i / Cp;
    const int pix = (int)(t % HW);
    const int64_t r = t / HW;
    y[i] = c < C ? __ldg(x + (r * C + c) * (int64_t)HW + pix) : 0.f;
  }
}

// First-layer transforms (mode 1 space-to-depth by f, mode 2 kx-unroll of width f): one thread
// per OUTPUT pixel writes all Cp channels; the (tap, channel) pair of each output channel is
// tracked with incremental counters (no integer division per element).
template <typename T>
__global__ void pack_xform_kernel(const float* __restrict__ x, T* __restrict__ y, int64_t rows, int C, int H, int W,
                                  int mode, int f, int xs, int Ho, int Wo, int Cp) {
  pdl_trigger();
  pdl_wait();
  const int per_row = Ho * Wo;
  for (int64_t r = blockIdx.y; r < rows; r += gridDim.y) {
    const float* src = x + r * C * (int64_t)H * W;
    for (int pix = blockIdx.x * blockDim.x + threadIdx.x; pix < per_row; pix += gridDim.x * blockDim.x) {
      const int yo = pix / Wo, xo = pix - (pix / Wo) * Wo;
      T* dst = y + (r * per_row + pix) * (int64_t)Cp;
      int a = 0, b = 0, c = 0;  // mode 1: (dy, dx, c); mode 2: (kx, -, c); mode 3: (kx, ky, c)
      const int kh = H - Ho + 1;  // mode 3: window rows
      for (int ch = 0; ch < Cp; ch += 8) {
        __align__(16) T v[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int yy = mode == 1 ? yo * f + a : (mode == 3 ? yo + b : yo);
          const int xx = mode == 1 ? xo * f + b : xo * xs + a;
          const bool ok = (mode == 3 ? b < kh : a < f) && yy < H && xx < W;
          v[j] = cvt<T>(ok ? __ldg(src + ((int64_t)c * H + yy) * W + xx) : 0.f);
          if (++c == C) {
            c = 0;
            if (mode == 1) {
              if (++b == f) { b = 0; ++a; }
            } else if (mode == 3) {
              if (++a == f) { a = 0; ++b; }
            } else {
              ++a;
            }
          }
        }
        *reinterpret_cast<uint4*>(dst + ch) = *reinterpret_cast<const uint4*>(v);
      }
    }
  }
}

// Compile-time specialisation of the first-layer transforms for the Tonic nets: every source
// offset is a constant relative to the pixel's base address, so each output channel costs one
// load and one convert (the generic kernel spent its time in index bookkeeping).
template <typename T, int MODE, int C, int F, int CP, int XS>
__global__ void pack_xform_fixed_kernel(const float* __restrict__ x, T* __restrict__ y, int64_t rows, int H, int W,
                                        int Ho, int Wo) {
  // Stores are staged per warp in shared memory: a thread's pixel is CP*2 contiguous bytes, so
  // direct 16-byte stores from 32 lanes would touch 32 separate lines per instruction; after
  // the (XOR-swizzled, bank-conflict-free) staging each store instruction writes 512
  // consecutive bytes of the warp's 32 consecutive output pixels.
  constexpr int CPC = CP / 8;  // 16-byte chunks per pixel (power of two)
  __shared__ uint4 stage[4][32 * CPC];
  pdl_trigger();
  pdl_wait();
  const int per_row = Ho * Wo;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint4* st = stage[wid];
  for (int64_t r = blockIdx.y; r < rows; r += gridDim.y) {
    const float* src = x + r * C * (int64_t)H * W;
    uint4* dst_row = reinterpret_cast<uint4*>(y + r * per_row * (int64_t)CP);
    for (int base = blockIdx.x * blockDim.x + wid * 32; base < per_row; base += gridDim.x * blockDim.x) {
      const int pix = base + lane;
      if (pix < per_row) {
        const int yo = pix / Wo, xo = pix - (pix / Wo) * Wo;
        const int y0 = MODE == 1 ? yo * F : yo, x0 = MODE == 1 ? xo * F : xo * XS;
        const float* p0 = src + (int64_t)y0 * W + x0;
#pragma unroll
        for (int ch = 0; ch < CP; ch += 8) {
          __align__(16) T v[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const int cc = ch + j;
            float val = 0.f;
            if (MODE == 1) {
              const int d = cc / C, c = cc % C, dy = d / F, dx = d % F;
              if (d < F * F && y0 + dy < H && x0 + dx < W) val = __ldg(p0 + ((int64_t)c * H + dy) * W + dx);
            } else if (MODE == 3) {  // window unroll: channel (ky * F + kx) * C + c, KH = H - Ho + 1 rows
              const int ky = cc / (F * C), rr = cc % (F * C), kx = rr / C, c = rr % C;
              if (ky < H - Ho + 1 && x0 + kx < W) val = __ldg(p0 + ((int64_t)c * H + ky) * W + kx);
            } else {
              const int kx = cc / C, c = cc % C;
              if (kx < F && x0 + kx < W) val = __ldg(p0 + (int64_t)c * H * W + kx);
            }
            v[j] = cvt<T>(val);
          }
          st[lane * CPC + ((ch / 8) ^ (lane & (CPC - 1)))] = *reinterpret_cast<const uint4*>(v);
        }
      }
      __syncwarp();
      const int nv = min(32, per_row - base) * CPC;
      uint4* dst = dst_row + (int64_t)base * CPC;
#pragma unroll
      for (int i = 0; i < CPC; ++i) {
        const int e = i * 32 + lane;
        const int p = e / CPC, k = e % CPC;
        if (e < nv) dst[e] = st[p * CPC + (k ^ (p & (CPC - 1)))];
      }
      __syncwarp();
    }
  }
}

// kx-unroll (mode 2) with one WARP per input row: the warp reads the row's C x W floats with
// coalesced loads into shared memory, then writes the row's Wo packed pixels as whole 16-byte
// chunks (consecutive lanes, consecutive chunks).  The per-pixel kernel above reads each input
// float from up to U / XS pixels' threads with 32-byte-strided lanes (FACE: ~32 sectors per load
// instruction).  FACE's 152 x 3 rows: 62.5 -> 51.0 us on B200.
template <typename T, int C, int U, int CP, int XS>
__global__ void __launch_bounds__(256) pack_kx_rows_kernel(const float* __restrict__ x, T* __restrict__ y, int64_t rows,
                                                           int H, int W, int Wo) {
  pdl_trigger();
  pdl_wait();
  extern __shared__ float srow[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  float* sr = srow + wid * C * W;
  const int64_t total = rows * H;  // (image, row) pairs: kx-unroll keeps the rows
  constexpr int CPC = CP / 8;
  for (int64_t t = (int64_t)blockIdx.x * nw + wid; t < total; t += (int64_t)gridDim.x * nw) {
    const int64_t img = t / H;
    const int yy = (int)(t - img * H);
    const float* src = x + (img * C * H + yy) * (int64_t)W;
#pragma unroll
    for (int c = 0; c < C; ++c)
      for (int i = lane; i < W; i += 32) sr[c * W + i] = __ldg(src + (int64_t)c * H * W + i);
    __syncwarp();
    uint4* dst = reinterpret_cast<uint4*>(y + t * (int64_t)Wo * CP);
    for (int e = lane; e < Wo * CPC; e += 32) {
      const int xo = e / CPC, j = e - xo * CPC;
      __align__(16) T v[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const int cc = 8 * j + q, kx = cc / C, c = cc - kx * C, xx = xo * XS + kx;
        v[q] = cvt<T>(kx < U && xx < W ? sr[c * W + xx] : 0.f);
      }
      dst[e] = *reinterpret_cast<const uint4*>(v);
    }
    __syncwarp();
  }
}

template <typename T>
static bool launch_pack_fixed(const float* x, void* y, int64_t rows, int C, int H, int W, int mode, int f, int xs, int Ho,
                              int Wo, int Cp, cudaStream_t st) {
  static const bool rows_on = [] {  // DJINN_PACK_ROWS=0: the per-pixel kx-unroll kernel
    const char* e = getenv("DJINN_PACK_ROWS");
    return !(e && e[0] == '0');
  }();
  if (rows_on && mode == 2 && Ho == H && C * W * 4 * 8 <= 48 * 1024) {
    const int64_t total = rows * H;
    const unsigned gb = (unsigned)std::min<int64_t>((total + 7) / 8, 148 * 16);
    const size_t smem = (size_t)8 * C * W * 4;
    if (C == 3 && f == 18 && xs == 8 && Cp == 64) {
      launch_pdl(pack_kx_rows_kernel<T, 3, 18, 64, 8>, dim3(gb), dim3(256), smem, st, x, (T*)y, rows, H, W, Wo);
      return true;
    }
    // (DIG's 28 x 1 rows: 16.2 us vs 10.0 for the per-pixel kernel, so it keeps that one)
  }
  dim3 g(min(nblocks(Ho * Wo, 128), 1024), (unsigned)(rows < 65535 ? rows : 65535));
  if (mode == 2 && C == 3 && f == 18 && xs == 8 && Cp == 64)
    launch_pdl(pack_xform_fixed_kernel<T, 2, 3, 18, 64, 8>, dim3(g), dim3(128), 0, st, x, (T*)y, rows, H, W, Ho, Wo);
  else if (mode == 2 && C == 1 && f == 12 && xs == 8 && Cp == 16)
    launch_pdl(pack_xform_fixed_kernel<T, 2, 1, 12, 16, 8>, dim3(g), dim3(128), 0, st, x, (T*)y, rows, H, W, Ho, Wo);
  else if (mode == 3 && C == 1 && f == 12 && xs == 8 && Cp == 64)
    launch_pdl(pack_xform_fixed_kernel<T, 3, 1, 12, 64, 8>, dim3(g), dim3(128), 0, st, x, (T*)y, rows, H, W, Ho, Wo);
  else if (mode == 1 && C == 3 && f == 4 && Cp == 64)
    launch_pdl(pack_xform_fixed_kernel<T, 1, 3, 4, 64, 1>, dim3(g), dim3(128), 0, st, x, (T*)y, rows, H, W, Ho, Wo);
  else
    return false;
  return true;
}

cudaError_t launch_pack_input(const float* x, void* y, int64_t rows, int C, int H, int W, int mode, int f, int xs,
                              int Ho, int Wo, int Cp, int dt, cudaStream_t st) {
  if (dt != DT_F32 && mode != 0) {
    const bool done = dt == DT_F16 ? launch_pack_fixed<__half>(x, y, rows, C, H, W, mode, f, xs, Ho, Wo, Cp, st)
                                   : launch_pack_fixed<__nv_bfloat16>(x, y, rows, C, H, W, mode, f, xs, Ho, Wo, Cp, st);
    if (done) return cudaGetLastError();
  }
  const int T = 256;
  if (dt == DT_F32) {
    int64_t n = rows * (int64_t)H * W * Cp;
    launch_pdl(pack32_kernel, dim3(min(nblocks(n, T), 148 * 32)), dim3(T), 0, st, x, (float*)y, rows, C, H * W, Cp);
  } else if (mode != 0) {
    dim3 g(min(nblocks(Ho * Wo, T), 1024), (unsigned)(rows < 65535 ? rows : 65535));
    if (dt == DT_F16)
      launch_pdl(pack_xform_kernel<__half>, dim3(g), dim3(T), 0, st, x, (__half*)y, rows, C, H, W, mode, f, xs, Ho, Wo, Cp);
    else
      launch_pdl(pack_xform_kernel<__nv_bfloat16>, dim3(g), dim3(T), 0, st, x, (__nv_bfloat16*)y, rows, C, H, W, mode, f, xs, Ho, Wo, Cp);
  } else if (mode == 0 && H == 1 && W == 1 && Ho == 1 && Wo == 1) {
    const int64_t total = rows * (Cp / 8);
    const unsigned g = (unsigned)std::min<int64_t>((total + T - 1) / T, 148 * 16);
    if (dt == DT_F16)
      launch_pdl(pack16_vec_kernel<__half>, dim3(g), dim3(T), 0, st, x, (__half*)y, rows, C, Cp);
    else
      launch_pdl(pack16_vec_kernel<__nv_bfloat16>, dim3(g), dim3(T), 0, st, x, (__nv_bfloat16*)y, rows, C, Cp);
  } else {
    const int per_row = Ho * Wo * (Cp / 8);
    dim3 g(min(nblocks(per_row, T), 1024), (unsigned)(rows < 65535 ? rows : 65535));
    if (dt == DT_F16)
      launch_pdl(pack16_kernel<__half>, dim3(g), dim3(T), 0, st, x, (__half*)y, rows, C, H, W, mode, f, xs, Ho, Wo, Cp);
    else
      launch_pdl(pack16_kernel<__nv_bfloat16>, dim3(g), dim3(T), 0, st, x, (__nv_bfloat16*)y, rows, C, H, W, mode, f, xs, Ho, Wo, Cp);
  }
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------
// djinn_forward16: widen 16-bit input rows to fp32 (exact), 8 elements per thread when aligned.
template <typename T>
__global__ void widen16_kernel(const T* __restrict__ x, float* __restrict__ y, int64_t n) {
  pdl_trigger();
  pdl_wait();
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t n8 = ((reinterpret_cast<uintptr_t>(x) & 15) == 0) ? n / 8 : 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n8; i += stride) {
    const uint4 v = __ldg(reinterpret_cast<const uint4*>(x) + i);
    const T* h = reinterpret_cast<const T*>(&v);
    float4 a, b;
    a.x = ld(h + 0); a.y = ld(h + 1); a.z = ld(h + 2); a.w = ld(h + 3);
    b.x = ld(h + 4); b.y = ld(h + 5); b.z = ld(h + 6); b.w = ld(h + 7);
    reinterpret_cast<float4*>(y)[2 * i] = a;
    reinterpret_cast<float4*>(y)[2 * i + 1] = b;
  }
  for (int64_t i = n8 * 8 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += stride) y[i] = ld(x + i);
}

cudaError_t launch_widen16(const void* x, float* y, int64_t n, int dt, cudaStream_t st) {
  const int T = 256;
  const int g = min(nblocks((n + 7) / 8, T), 148 * 16);
  if (dt == DT_F16) launch_pdl(widen16_kernel<__half>, dim3(g), dim3(T), 0, st, (const __half*)x, y, n);
  else launch_pdl(widen16_kernel<__nv_bfloat16>, dim3(g), dim3(T), 0, st, (const __nv_bfloat16*)x, y, n);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------
// SENNA window lookup (kernels.h launch_embed).  One thread per output column: consecutive
// threads copy consecutive elements of one table row, so each (word, table) lookup is one
// coalesced read of dim[t] elements; the row's indices are L1-resident broadcasts.
template <typename T>
__global__ void embed_kernel(const float* __restrict__ x, const T* __restrict__ tab, T* __restrict__ y, int64_t rows,
                             EmbedGeom eg, int Cp) {
  pdl_trigger();
  pdl_wait();
  const int in_row = eg.window * eg.T, Dw = eg.window * eg.D;
  const int64_t total = rows * Cp;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / Cp;
    const int c = (int)(i - r * Cp);
    T v = cvt<T>(0.f);
    if (c < Dw) {
      const int w = c / eg.D;
      int j = c - w * eg.D, t = 0;
      while (j >= eg.dim[t]) j -= eg.dim[t++];
      const float id = __ldg(x + r * in_row + w * eg.T + t);
      if (id >= 0.f && id < (float)eg.vocab[t] && id == floorf(id))
        v = tab[eg.toff[t] + (int64_t)id * eg.dim[t] + j];
    }
    y[i] = v;
  }
}

cudaError_t launch_embed(const float* x, const void* tables, void* y, int64_t rows, const EmbedGeom& eg, int Cp, int dt,
                         cudaStream_t st) {
  const int T = 256;
  const int g = min(nblocks(rows * Cp, T), 148 * 16);
  if (dt == DT_F32)
    launch_pdl(embed_kernel<float>, dim3(g), dim3(T), 0, st, x, (const float*)tables, (float*)y, rows, eg, Cp);
  else if (dt == DT_F16)
    launch_pdl(embed_kernel<__half>, dim3(g), dim3(T), 0, st, x, (const __half*)tables, (__half*)y, rows, eg, Cp);
  else
    launch_pdl(embed_kernel<__nv_bfloat16>, dim3(g), dim3(T), 0, st, x, (const __nv_bfloat16*)tables,
               (__nv_bfloat16*)y, rows, eg, Cp);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------
// K4: Caffe LRN across channels.  y = x * (k + alpha/size * sum_{window} x^2)^-beta.
// One thread per (pixel, channel); the channel window is contiguous in NHWC.
template <typename T>
__global__ void lrn_kernel(const T* __restrict__ x, T* __restrict__ y, int64_t pixels, int C, int Cp, int gsz,
                           int gpitch, int size, float alpha_over_n, float beta, float k) {
  pdl_trigger();
  pdl_wait();
  const int half = (size - 1) / 2;
  const int64_t total = pixels * Cp;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int p = (int)(i % Cp);  // storage position -> logical channel
    const int grp = p / gpitch, cin = p - grp * gpitch;
    const int c = grp * gsz + cin;
    if (cin >= gsz || c >= C) { y[i] = cvt<T>(0.f); continue; }
    const T* px = x + (i - p);
    const int lo = max(c - half, 0), hi = min(c + half, C - 1);
    float s = 0.f;
    for (int cc = lo; cc <= hi; ++cc) {
      const float v = ld(px + (cc / gsz) * gpitch + cc % gsz);
      s += v * v;
    }
    const float v = ld(px + p);
    y[i] = cvt<T>(v * powf(k + alpha_over_n * s, -beta));
  }
}

cudaError_t launch_lrn(const void* x, void* y, int64_t pixels, int C, int Cp, int gsz, int gpitch, int size,
                       float alpha, float beta, float k, int dt, cudaStream_t st) {
  const int T = 256;
  const int64_t n = pixels * Cp;
  const int g = min(nblocks(n, T), 148 * 32);
  const float an = alpha / size;
  if (gsz > C) { gsz = C; gpitch = Cp; }
  if (dt == DT_F32) launch_pdl(lrn_kernel<float>, dim3(g), dim3(T), 0, st, (const float*)x, (float*)y, pixels, C, Cp, gsz, gpitch, size, an, beta, k);
  else if (dt == DT_F16) launch_pdl(lrn_kernel<__half>, dim3(g), dim3(T), 0, st, (const __half*)x, (__half*)y, pixels, C, Cp, gsz, gpitch, size, an, beta, k);
  else launch_pdl(lrn_kernel<__nv_bfloat16>, dim3(g), dim3(T), 0, st, (const __nv_bfloat16*)x, (__nv_bfloat16*)y, pixels, C, Cp, gsz, gpitch, size, an, beta, k);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------
// K4+K5 fused: y = maxpool(LRN(x)), Caffe LRN across channels (window c-2..c+2 clipped to
// [0, C)) in fp32, then Caffe MAX pooling with kernel 3 / stride 2 / pad 0 (AlexNet norm1+pool1,
// norm2+pool2).  The conv before it stores its bias+ReLU output in fp16 (plain layout, pitch
// Cpi, channels >= C zero).
//
// Every input element's LRN is evaluated once (the MUFU work -- lg2 + ex2 per element at 16
// per clock per SM -- is the kernel's floor).  One block walks down the input rows of one image
// band; each row (W pixels x Cpi channels, contiguous) is staged in shared memory by cp.async,
// NBUF-1 rows ahead, with a 16-byte pad per pixel so that lanes reading consecutive pixels hit
// distinct banks (direct global loads with a 32-lane pixel stride had run L1-bound at 90%).
// Warp (seg, chunk) owns channels 16*chunk .. +15 of the 32 columns starting at 30*seg: the
// vertical window max (rows 2oy, 2oy+1, 2oy+2; row 2oy+2 also opens window oy+1) lives in
// registers, the horizontal one takes two warp shuffles, and the even lanes 0..28 store output
// pixels ox = (30*seg + lane) / 2.
constexpr int LRNPOOL_NBUF = 4;
// 2^y on the FMA pipe (y >= -126): y = n + f with n = rint(y), |f| <= 1/2, 2^f by its degree-4
// Taylor polynomial (relative error <= 4.2e-5), 2^n added to the exponent field.  Moves half of
// the LRN's transcendental work off the MUFU (16 results per clock per SM).
__device__ __forceinline__ float exp2_fma(float y) {
  y = fmaxf(y, -126.f);
  const float t = y + 12582912.f;  // 1.5 * 2^23: rint(y) in the low mantissa bits
  const float n = t - 12582912.f;
  const float f = y - n;
  float p = fmaf(0.0096181291f, f, 0.0555041087f);
  p = fmaf(p, f, 0.2402265070f);
  p = fmaf(p, f, 0.6931471806f);
  p = fmaf(p, f, 1.0f);
  return __int_as_float(__float_as_int(p) + ((__float_as_int(t) - 0x4B400000) << 23));
}
template <typename TO>
__global__ void __launch_bounds__(1024) lrn_pool_kernel(const __half* __restrict__ x, TO* __restrict__ y, int C, int Cpi,
                                                        int H, int W, int OH, int OW, int bands, int gsz, int gpitch,
                                                        int Cpo, int obd, float an, float nbeta, float k) {
  pdl_trigger();
  pdl_wait();
  extern __shared__ __align__(16) uint8_t srows[];
  const int RP = Cpi * 2 + 16;  // bytes per staged pixel
  const int nch = C / 16;
  const int lane = threadIdx.x, seg = threadIdx.y / nch, chunk = threadIdx.y - seg * nch;
  const int c0 = chunk * 16;
  const int xx = seg * 30 + lane;
  const int64_t r = blockIdx.x;
  const int per_band = (OH + bands - 1) / bands;
  const int oy0 = blockIdx.y * per_band, oy1 = min(OH, oy0 + per_band);
  if (oy0 >= oy1) return;
  const int tid = threadIdx.y * 32 + lane, nthr = blockDim.y * 32;
  // staging: thread tid copies 16-byte piece q of pixels px0, px0 + pstep, ... (the launch makes
  // the block size a multiple of the pieces per pixel, so (px, q) need no division per copy)
  const int pieces_px = Cpi / 8, pstep = nthr / pieces_px;
  const int q_st = tid % pieces_px, px0 = tid / pieces_px;
  const __half* xr = x + r * H * (int64_t)W * Cpi + px0 * Cpi + q_st * 8;
  const uint32_t sm0 = (uint32_t)__cvta_generic_to_shared(srows) + px0 * RP + q_st * 16;
  auto stage = [&](int yy) {
    const uint32_t dst0 = sm0 + (yy % LRNPOOL_NBUF) * W * RP;
    const __half* src0 = xr + (int64_t)yy * W * Cpi;
    for (int px = px0, i = 0; px < W; px += pstep, ++i)
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst0 + i * pstep * RP),
                   "l"(src0 + (int64_t)i * pstep * Cpi)
                   : "memory");
  };
  const bool xin = xx < W;
  const int grp = c0 / gsz, cin = c0 - grp * gsz;  // 16 | gsz: a chunk never straddles groups
  TO* yr = y + (r * (OH + 2 * obd) + obd) * (int64_t)(OW + 2 * obd) * Cpo + grp * gpitch + cin;
  const bool pad_writer = gpitch > gsz && cin + 16 == gsz;
  const bool has_lo = c0 >= 2, has_hi = c0 + 16 < C;
  __half2 acc[8];
  int emitted = oy0 - 1;
  auto emit = [&](int oy) {
    // horizontal window: columns 2ox .. 2ox+2 (clipped to W - 1: a duplicate cannot change a max)
    __half2 m[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const uint32_t u = *reinterpret_cast<const uint32_t*>(&acc[j]);
      const uint32_t u1 = __shfl_down_sync(0xffffffffu, u, 1), u2 = __shfl_down_sync(0xffffffffu, u, 2);
      __half2 v = acc[j];
      if (xx + 1 < W) v = __hmax2(v, *reinterpret_cast<const __half2*>(&u1));
      if (xx + 2 < W) v = __hmax2(v, *reinterpret_cast<const __half2*>(&u2));
      m[j] = v;
    }
    const int ox = xx >> 1;
    if (!(lane & 1) && lane <= 28 && ox < OW) {
      TO* yo = yr + ((int64_t)oy * (OW + 2 * obd) + ox + obd) * Cpo;
      __align__(16) TO o[16];
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const float2 f = __half22float2(m[j]);
        o[2 * j] = cvt<TO>(f.x);
        o[2 * j + 1] = cvt<TO>(f.y);
      }
      reinterpret_cast<uint4*>(yo)[0] = reinterpret_cast<const uint4*>(o)[0];
      reinterpret_cast<uint4*>(yo)[1] = reinterpret_cast<const uint4*>(o)[1];
      if (pad_writer)
        for (int e = 16; e < 16 + gpitch - gsz; e += 8) *reinterpret_cast<uint4*>(yo + e) = make_uint4(0, 0, 0, 0);
    }
    emitted = oy;
  };
  const int yfirst = 2 * oy0, ylast = min(2 * oy1, H - 1);
  for (int yy = yfirst; yy < yfirst + LRNPOOL_NBUF - 1; ++yy) {
    if (yy <= ylast) stage(yy);
    asm volatile("cp.async.commit_group;" ::: "memory");
  }
  for (int yy = yfirst; yy <= ylast; ++yy) {
    asm volatile("cp.async.wait_group %0;" ::"n"(LRNPOOL_NBUF - 2) : "memory");  // row yy has landed
    __syncthreads();  // ... for every thread, and every warp is done reading row yy - 1's buffer
    if (yy + LRNPOOL_NBUF - 1 <= ylast) stage(yy + LRNPOOL_NBUF - 1);  // refills row yy - 1's buffer
    asm volatile("cp.async.commit_group;" ::: "memory");
    const uint8_t* px = srows + (yy % LRNPOOL_NBUF) * W * RP + (xin ? xx : W - 1) * RP + c0 * 2;
    const uint4 ua = reinterpret_cast<const uint4*>(px)[0];
    const uint4 ub = reinterpret_cast<const uint4*>(px)[1];
    const uint32_t ulo = has_lo ? *reinterpret_cast<const uint32_t*>(px - 4) : 0u;
    const uint32_t uhi = has_hi ? *reinterpret_cast<const uint32_t*>(px + 32) : 0u;
    float v[20];
    {
      const float2 lo = __half22float2(*reinterpret_cast<const __half2*>(&ulo));
      const float2 hi = __half22float2(*reinterpret_cast<const __half2*>(&uhi));
      v[0] = lo.x; v[1] = lo.y; v[18] = hi.x; v[19] = hi.y;
      const __half2* ha = reinterpret_cast<const __half2*>(&ua);
      const __half2* hb = reinterpret_cast<const __half2*>(&ub);
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const float2 fa = __half22float2(ha[j]), fb = __half22float2(hb[j]);
        v[2 + 2 * j] = fa.x; v[3 + 2 * j] = fa.y; v[10 + 2 * j] = fb.x; v[11 + 2 * j] = fb.y;
      }
    }
    float sq[20];
#pragma unroll
    for (int j = 0; j < 20; ++j) sq[j] = v[j] * v[j];
    // sliding window sums s[j] = sq[j] + ... + sq[j + 4] (all terms >= 0: no cancellation)
    float sw[16];
    sw[0] = (sq[0] + sq[1]) + (sq[2] + sq[3]) + sq[4];
#pragma unroll
    for (int j = 1; j < 16; ++j) sw[j] = (sw[j - 1] - sq[j - 1]) + sq[j + 4];
    __half2 l[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float s0 = sw[2 * j], s1 = sw[2 * j + 1];
      float r0, r1;
      asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(r0) : "f"(fmaf(an, s0, k)));
      asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(r1) : "f"(fmaf(an, s1, k)));
#ifdef DJINN_LRN_POLY
      r0 = exp2_fma(nbeta * r0);
      r1 = exp2_fma(nbeta * r1);
#else
      asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r0) : "f"(nbeta * r0));
      asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r1) : "f"(nbeta * r1));
#endif
      l[j] = __floats2half2_rn(v[2 + 2 * j] * r0, v[3 + 2 * j] * r1);
    }
    if ((yy & 1) == 0) {
      const int j = yy >> 1;
      if (j - 1 >= oy0) {  // row 2(j-1)+2 closes window j-1
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q] = __hmax2(acc[q], l[q]);
        emit(j - 1);
      }
      if (j < oy1) {
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q] = l[q];
      }
    } else {
#pragma unroll
      for (int q = 0; q < 8; ++q) acc[q] = __hmax2(acc[q], l[q]);
    }
  }
  if (emitted < oy1 - 1) emit(oy1 - 1);  // last window clipped at the bottom edge (ceil geometry)
}

cudaError_t launch_lrn_pool(const void* x, void* y, int64_t rows, int C, int Cpi, int H, int W, int OH, int OW,
                            int kernel, int stride, int pad, int out_gsz, int out_gpitch, int Cpo, int obd, int size,
                            float alpha, float beta, float k, int dt, cudaStream_t st) {
  const int segs = (W + 29) / 30;
  if (size != 5 || kernel != 3 || stride != 2 || pad != 0 || C % 16 || Cpi % 8 || Cpi < C || Cpo % 8 ||
      rows > 65535 || obd < 0 || segs * (C / 16) * 32 > 1024)
    return cudaErrorInvalidValue;
  if (out_gsz >= C) { out_gsz = C; out_gpitch = Cpo; }
  if (out_gsz % 16 || out_gpitch % 8) return cudaErrorInvalidValue;
  const size_t smem = (size_t)LRNPOOL_NBUF * W * (Cpi * 2 + 16);
  if (smem > 100 * 1024) return cudaErrorInvalidValue;
  // bands of output rows: enough blocks for ~4 waves (each band re-reads one boundary input row)
  const int threads = segs * (C / 16) * 32;
  if (threads % (Cpi / 8)) return cudaErrorInvalidValue;  // the staging loop's piece mapping
  const int per_sm = std::max(1, std::min(2048 / threads, (int)((200 * 1024) / smem)));
  int bands = (int)std::min<int64_t>(std::max<int64_t>(1, (4LL * 148 * per_sm + rows - 1) / rows), OH);
  dim3 g((unsigned)rows, bands), b(32, segs * (C / 16));
  const float an = alpha / size;
  cudaError_t e;
  if (dt == DT_F16) {
    e = ensure_max_smem((const void*)lrn_pool_kernel<__half>, 100 * 1024);
    if (e == cudaSuccess)
      e = launch_pdl(lrn_pool_kernel<__half>, g, b, smem, st, (const __half*)x, (__half*)y, C, Cpi, H, W, OH, OW, bands,
                     out_gsz, out_gpitch, Cpo, obd, an, -beta, k);
  } else {
    e = ensure_max_smem((const void*)lrn_pool_kernel<__nv_bfloat16>, 100 * 1024);
    if (e == cudaSuccess)
      e = launch_pdl(lrn_pool_kernel<__nv_bfloat16>, g, b, smem, st, (const __half*)x, (__nv_bfloat16*)y, C, Cpi, H, W,
                     OH, OW, bands, out_gsz, out_gpitch, Cpo, obd, an, -beta, k);
  }
  return e != cudaSuccess ? e : cudaGetLastError();
}

// ------------------------------------------------------------------------------------------
// K5: Caffe pooling (MAX / AVE), ceil geometry; window clipped to the image, AVE divisor is
// the window area clipped to H+pad but not to the image.
template <typename T>
__global__ void pool_kernel(const T* __restrict__ x, T* __restrict__ y, int64_t rows, int Cp, int H,
                            int W, int OH, int OW, int kern, int stride, int pad, int is_max) {
  pdl_trigger();
  pdl_wait();
  const int64_t total = rows * (int64_t)OH * OW * Cp;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int c = (int)(i % Cp);
    int64_t t = i / Cp;
    const int ox = (int)(t % OW);
    t /= OW;
    const int oy = (int)(t % OH);
    const int64_t r = t / OH;
    int hs = oy * stride - pad, ws = ox * stride - pad;
    int he = min(hs + kern, H + pad), we = min(ws + kern, W + pad);
    const float area = (float)((he - hs) * (we - ws));
    hs = max(hs, 0); ws = max(ws, 0); he = min(he, H); we = min(we, W);
    const T* base = x + r * (int64_t)H * W * Cp + c;
    float acc = is_max ? -FLT_MAX : 0.f;
    for (int h = hs; h < he; ++h)
      for (int w = ws; w < we; ++w) {
        const float v = ld(base + ((int64_t)h * W + w) * Cp);
        acc = is_max ? fmaxf(acc, v) : acc + v;
      }
    y[i] = cvt<T>(is_max ? acc : acc / area);
  }
}

// 16-bit storage: 8 channels (16 B) per thread, fp32 math.
// x-unrolled output (out_xu > 1): each pooled pixel is computed once and stored into slot s
// of pixel x - s for every s; slots past the right edge are zero-filled by pixel x's thread.
template <typename T>
__global__ void pool16_xu_kernel(const T* __restrict__ x, T* __restrict__ y, int64_t rows, int Cp, int H, int W,
                                 int OH, int OW, int kern, int stride, int pad, int is_max, int out_xu) {
  pdl_trigger();
  pdl_wait();
  const int cchunks = Cp / 8;
  const int per_row = OH * OW * cchunks, Cpo = out_xu * Cp;
  for (int64_t r = blockIdx.y; r < rows; r += gridDim.y) {
    const T* xr = x + r * (int64_t)H * W * Cp;
    T* yr = y + r * (int64_t)OH * OW * Cpo;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < per_row; i += gridDim.x * blockDim.x) {
      const int ch = i % cchunks;
      const int pix = i / cchunks;
      const int oy = pix / OW, ox = pix - oy * OW;
      int hs = oy * stride - pad, ws = ox * stride - pad;
      int he = min(hs + kern, H + pad), we = min(ws + kern, W + pad);
      const float area = (float)((he - hs) * (we - ws));
      hs = max(hs, 0); ws = max(ws, 0); he = min(he, H); we = min(we, W);
      const T* base = xr + ch * 8;
      float acc[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[j] = is_max ? -FLT_MAX : 0.f;
      for (int h = hs; h < he; ++h)
        for (int w = ws; w < we; ++w) {
          const uint4 u = __ldg(reinterpret_cast<const uint4*>(base + (h * W + w) * Cp));
          const T* v = reinterpret_cast<const T*>(&u);
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[j] = is_max ? fmaxf(acc[j], ld(v + j)) : acc[j] + ld(v + j);
        }
      __align__(16) T o[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) o[j] = cvt<T>(is_max ? acc[j] : acc[j] / area);
      const uint4 ov = *reinterpret_cast<const uint4*>(o);
      for (int sl = 0; sl < out_xu; ++sl) {
        if (ox - sl >= 0)
          *reinterpret_cast<uint4*>(yr + ((int64_t)oy * OW + ox - sl) * Cpo + sl * Cp + ch * 8) = ov;
        if (sl > 0 && ox + sl >= OW)
          *reinterpret_cast<uint4*>(yr + ((int64_t)oy * OW + ox) * Cpo + sl * Cp + ch * 8) = make_uint4(0, 0, 0, 0);
      }
    }
  }
}

template <typename T>
__global__ void pool16_kernel(const T* __restrict__ x, T* __restrict__ y, int64_t rows, int Cp, int H, int W,
                              int OH, int OW, int kern, int stride, int pad, int is_max, int out_xu) {
  pdl_trigger();
  pdl_wait();
  const int cchunks = Cp / 8, chunks = cchunks * out_xu;
  const int per_row = OH * OW * chunks;
  for (int64_t r = blockIdx.y; r < rows; r += gridDim.y) {
    const T* xr = x + r * (int64_t)H * W * Cp;
    T* yr = y + r * (int64_t)per_row * 8;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < per_row; i += gridDim.x * blockDim.x) {
      const int chx = i % chunks;
      const int pix = i / chunks;
      const int oy = pix / OW;
      const int slot = chx / cchunks, ch = chx - slot * cchunks;
      const int ox = pix - oy * OW + slot;  // x-unrolled output: slot s holds pixel x + s
      if (ox >= OW) {
        *reinterpret_cast<uint4*>(yr + (int64_t)i * 8) = make_uint4(0, 0, 0, 0);
        continue;
      }
      int hs = oy * stride - pad, ws = ox * stride - pad;
      int he = min(hs + kern, H + pad), we = min(ws + kern, W + pad);
      const float area = (float)((he - hs) * (we - ws));
      hs = max(hs, 0); ws = max(ws, 0); he = min(he, H); we = min(we, W);
      const T* base = xr + ch * 8;
      float acc[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[j] = is_max ? -FLT_MAX : 0.f;
      for (int h = hs; h < he; ++h)
        for (int w = ws; w < we; ++w) {
          const uint4 u = __ldg(reinterpret_cast<const uint4*>(base + (h * W + w) * Cp));
          const T* v = reinterpret_cast<const T*>(&u);
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[j] = is_max ? fmaxf(acc[j], ld(v + j)) : acc[j] + ld(v + j);
        }
      __align__(16) T o[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) o[j] = cvt<T>(is_max ? acc[j] : acc[j] / area);
      *reinterpret_cast<uint4*>(yr + i * 8) = *reinterpret_cast<const uint4*>(o);
    }
  }
}

// K5 MAX pooling with a channel-layout change: one thread per (output pixel, 8-channel chunk of
// the OUTPUT layout); input and output layouts may differ (plain / grouped / x-unrolled), so the
// pool's producer writes its natural pitch and the pool writes the consumer's layout.  Block =
// (chunks of one output pixel) x (PIX consecutive output pixels of one image); the channel
// mapping is computed once per block; the max runs on packed 16-bit pairs (exact).
__device__ __forceinline__ uint4 max8(uint4 a, uint4 b, __half) {
  uint4 r;
  const __half2* x = reinterpret_cast<const __half2*>(&a);
  const __half2* y = reinterpret_cast<const __half2*>(&b);
  __half2* z = reinterpret_cast<__half2*>(&r);
#pragma unroll
  for (int j = 0; j < 4; ++j) z[j] = __hmax2(x[j], y[j]);
  return r;
}
__device__ __forceinline__ uint4 max8(uint4 a, uint4 b, __nv_bfloat16) {
  uint4 r;
  const __nv_bfloat162* x = reinterpret_cast<const __nv_bfloat162*>(&a);
  const __nv_bfloat162* y = reinterpret_cast<const __nv_bfloat162*>(&b);
  __nv_bfloat162* z = reinterpret_cast<__nv_bfloat162*>(&r);
#pragma unroll
  for (int j = 0; j < 4; ++j) z[j] = __hmax2(x[j], y[j]);
  return r;
}

template <typename T, int K>
__global__ void pool_max_remap_kernel(const T* __restrict__ x, T* __restrict__ y, int C, int Cpi, int gsz_i,
                                      int gpitch_i, int H, int W, int Hst, int Wst, int OH, int OW, int kern, int stride,
                                      int pad, int Cpo, int gsz_o, int gpitch_o, int xu, int obd) {
  pdl_trigger();
  pdl_wait();
  __shared__ int in_off[64];  // per output chunk: input channel offset, -1 = zero chunk
  const int P = Cpo / xu, chunks = P / 8;
  if (threadIdx.y == 0 && threadIdx.x < chunks) {
    const int pos = threadIdx.x * 8, grp = pos / gpitch_o, within = pos - grp * gpitch_o, c0 = grp * gsz_o + within;
    in_off[threadIdx.x] = (within < gsz_o && c0 < C) ? (c0 / gsz_i) * gpitch_i + c0 % gsz_i : -1;
  }
  __syncthreads();
  const int pix = blockIdx.x * blockDim.y + threadIdx.y;
  if (pix >= OH * OW) return;
  const int oy = pix / OW, ox = pix - oy * OW;
  const int64_t r = blockIdx.y;
  const int off = in_off[threadIdx.x];
  T* yo = y + ((r * (OH + 2 * obd) + oy + obd) * (OW + 2 * obd) + ox + obd) * (int64_t)Cpo + threadIdx.x * 8;
  uint4 ov = make_uint4(0, 0, 0, 0);
  if (off >= 0) {
    const T* base = x + r * (int64_t)Hst * Wst * Cpi + off;
    int hs = oy * stride - pad, ws = ox * stride - pad;
    int he = min(hs + kern, H + pad), we = min(ws + kern, W + pad);
    hs = max(hs, 0); ws = max(ws, 0); he = min(he, H); we = min(we, W);
    if (K > 0) {
      // all K*K loads issued together; taps outside the clipped window re-read a tap inside
      // it (a duplicate cannot change a max)
      uint4 v[K > 0 ? K * K : 1];
#pragma unroll
      for (int a = 0; a < K; ++a)
#pragma unroll
        for (int b = 0; b < K; ++b) {
          const int h = min(hs + a, he - 1), w = min(ws + b, we - 1);
          v[a * K + b] = __ldg(reinterpret_cast<const uint4*>(base + ((int64_t)h * Wst + w) * Cpi));
        }
      ov = v[0];
#pragma unroll
      for (int j = 1; j < K * K; ++j) ov = max8(ov, v[j], T());
    } else {
      ov = __ldg(reinterpret_cast<const uint4*>(base + ((int64_t)hs * Wst + ws) * Cpi));
      for (int h = hs; h < he; ++h)
        for (int w = ws; w < we; ++w)
          ov = max8(ov, __ldg(reinterpret_cast<const uint4*>(base + ((int64_t)h * Wst + w) * Cpi)), T());
    }
  }
  *reinterpret_cast<uint4*>(yo) = ov;
  for (int sl = 1; sl < xu; ++sl) {
    if (ox - sl >= 0) *reinterpret_cast<uint4*>(yo - (int64_t)sl * Cpo + sl * P) = ov;  // pixel ox-sl, slot sl
    if (ox + sl >= OW) *reinterpret_cast<uint4*>(yo + sl * P) = make_uint4(0, 0, 0, 0);  // past the row end
  }
}

// 3x3 / stride-2 / pad-0 MAX pooling (IMC pool1/pool2/pool5, FACE M2) with the same layout change
// as pool_max_remap_kernel, but each thread walks a band of R output rows of one column: the
// horizontal max of an input row is computed once and the row shared by output rows oy and oy+1
// (input row 2oy+2) is carried over, so each output row costs 6 loads instead of 9.  Windows
// clip to the image (Caffe ceil geometry); clipped taps re-read the last row/column (exact).
template <typename T, int R>
__global__ void pool_max_k3s2_band_kernel(const T* __restrict__ x, T* __restrict__ y, int C, int Cpi, int gsz_i,
                                          int gpitch_i, int H, int W, int Hst, int Wst, int OH, int OW, int Cpo,
                                          int gsz_o, int gpitch_o, int xu, int obd, int xblocks) {
  pdl_trigger();
  pdl_wait();
  __shared__ int in_off[64];
  const int P = Cpo / xu, chunks = P / 8;
  if (threadIdx.y == 0 && threadIdx.x < chunks) {
    const int pos = threadIdx.x * 8, grp = pos / gpitch_o, within = pos - grp * gpitch_o, c0 = grp * gsz_o + within;
    in_off[threadIdx.x] = (within < gsz_o && c0 < C) ? (c0 / gsz_i) * gpitch_i + c0 % gsz_i : -1;
  }
  __syncthreads();
  const int band = blockIdx.x / xblocks, xb = blockIdx.x - band * xblocks;
  const int ox = xb * blockDim.y + threadIdx.y;
  if (ox >= OW) return;
  const int oy0 = band * R, oy1 = min(oy0 + R, OH);
  const int64_t r = blockIdx.y;
  const int off = in_off[threadIdx.x];
  const int64_t orow = (int64_t)(OW + 2 * obd) * Cpo;
  T* yo = y + ((r * (OH + 2 * obd) + oy0 + obd) * (OW + 2 * obd) + ox + obd) * (int64_t)Cpo + threadIdx.x * 8;
  if (off < 0) {
    for (int oy = oy0; oy < oy1; ++oy, yo += orow) {
      *reinterpret_cast<uint4*>(yo) = make_uint4(0, 0, 0, 0);
      for (int sl = 1; sl < xu; ++sl) {
        if (ox - sl >= 0) *reinterpret_cast<uint4*>(yo - (int64_t)sl * Cpo + sl * P) = make_uint4(0, 0, 0, 0);
        if (ox + sl >= OW) *reinterpret_cast<uint4*>(yo + sl * P) = make_uint4(0, 0, 0, 0);
      }
    }
    return;
  }
  const T* base = x + r * (int64_t)Hst * Wst * Cpi + off;
  const int ws = ox * 2, w1 = min(ws + 1, W - 1), w2 = min(ws + 2, W - 1);
  auto hrow = [&](int h) {
    const T* p = base + (int64_t)h * Wst * Cpi;
    const uint4 a = __ldg(reinterpret_cast<const uint4*>(p + (int64_t)ws * Cpi));
    const uint4 b = __ldg(reinterpret_cast<const uint4*>(p + (int64_t)w1 * Cpi));
    const uint4 c = __ldg(reinterpret_cast<const uint4*>(p + (int64_t)w2 * Cpi));
    return max8(max8(a, b, T()), c, T());
  };
  uint4 prev = hrow(2 * oy0);
  for (int oy = oy0; oy < oy1; ++oy, yo += orow) {
    const int hs = 2 * oy;
    const uint4 m1 = hrow(min(hs + 1, H - 1));
    const uint4 m2 = hrow(min(hs + 2, H - 1));
    const uint4 ov = max8(max8(prev, m1, T()), m2, T());
    prev = m2;
    *reinterpret_cast<uint4*>(yo) = ov;
    for (int sl = 1; sl < xu; ++sl) {
      if (ox - sl >= 0) *reinterpret_cast<uint4*>(yo - (int64_t)sl * Cpo + sl * P) = ov;
      if (ox + sl >= OW) *reinterpret_cast<uint4*>(yo + sl * P) = make_uint4(0, 0, 0, 0);
    }
  }
}

cudaError_t launch_pool_remap(const void* x, void* y, int64_t rows, int C, int Cpi, int gsz_i, int gpitch_i, int H,
                              int W, int Hst, int Wst, int OH, int OW, int kernel, int stride, int pad, int Cpo, int gsz_o,
                              int gpitch_o, int xu, int obd, int dt, cudaStream_t st) {
  if (xu < 1 || Cpo % xu || obd < 0 || (obd > 0 && xu > 1) || Hst < H || Wst < W) return cudaErrorInvalidValue;
  // plain layouts: one group spanning every position (channel c at c; pads read as zeros)
  const bool gi = gsz_i < C, go = gsz_o < C;
  if (!gi) gsz_i = gpitch_i = 1 << 30;
  if (!go) gsz_o = gpitch_o = 1 << 30;
  if (xu > 1 && go) return cudaErrorInvalidValue;
  if (dt == DT_F32 || Cpi % 8 || Cpo % 8 || (gi && (gsz_i % 8 || gpitch_i % 8)) || (go && (gsz_o % 8 || gpitch_o % 8)) ||
      kernel > stride + 1)
    return cudaErrorInvalidValue;
  const int chunks = Cpo / xu / 8;
  if (chunks > 64) return cudaErrorInvalidValue;
  static const bool band_on = [] {
    const char* e = getenv("DJINN_POOL_BAND");
    return !e || atoi(e) != 0;
  }();
  if (band_on && kernel == 3 && stride == 2 && pad == 0) {
    static const int R = [] {  // output rows per band (DJINN_POOL_R = 2 / 4 / 8)
      const char* e = getenv("DJINN_POOL_R");
      const int r = e ? atoi(e) : 4;
      return (r == 2 || r == 8) ? r : 4;
    }();
    const int xblocks = (OW + 256 / chunks - 1) / (256 / chunks);
    const int bpix = (OW + xblocks - 1) / xblocks;  // balanced column blocks
    const int bands = (OH + R - 1) / R;
    for (int64_t r0 = 0; r0 < rows; r0 += 65535) {
      const int64_t nr = rows - r0 < 65535 ? rows - r0 : 65535;
      dim3 blk(chunks, bpix), g(xblocks * bands, (unsigned)nr);
      const size_t xo = (size_t)r0 * Hst * Wst * Cpi, yo = (size_t)r0 * (OH + 2 * obd) * (OW + 2 * obd) * Cpo;
#define DJ_BAND_LAUNCH(T, RR)                                                                                      \
  launch_pdl(pool_max_k3s2_band_kernel<T, RR>, dim3(g), dim3(blk), 0, st, (const T*)x + xo, (T*)y + yo, C, Cpi, gsz_i, \
             gpitch_i, H, W, Hst, Wst, OH, OW, Cpo, gsz_o, gpitch_o, xu, obd, xblocks)
      if (dt == DT_F16) {
        if (R == 2) DJ_BAND_LAUNCH(__half, 2);
        else if (R == 8) DJ_BAND_LAUNCH(__half, 8);
        else DJ_BAND_LAUNCH(__half, 4);
      } else {
        if (R == 2) DJ_BAND_LAUNCH(__nv_bfloat16, 2);
        else if (R == 8) DJ_BAND_LAUNCH(__nv_bfloat16, 8);
        else DJ_BAND_LAUNCH(__nv_bfloat16, 4);
      }
#undef DJ_BAND_LAUNCH
    }
    return cudaGetLastError();
  }
  const int pix = 256 / chunks;
  for (int64_t r0 = 0; r0 < rows; r0 += 65535) {  // grid.z <= 65535 images per launch
    const int64_t nr = rows - r0 < 65535 ? rows - r0 : 65535;
    dim3 blk(chunks, pix), g((OH * OW + pix - 1) / pix, (unsigned)nr);
    const size_t xo = (size_t)r0 * Hst * Wst * Cpi, yo = (size_t)r0 * (OH + 2 * obd) * (OW + 2 * obd) * Cpo;
#define DJ_POOL_LAUNCH(T, KK)                                                                                   \
  launch_pdl(pool_max_remap_kernel<T, KK>, dim3(g), dim3(blk), 0, st, (const T*)x + xo, (T*)y + yo, C, Cpi, gsz_i, gpitch_i, H, W, Hst, Wst, OH, OW, \
                                                  kernel, stride, pad, Cpo, gsz_o, gpitch_o, xu, obd)
    if (dt == DT_F16) {
      if (kernel == 3) DJ_POOL_LAUNCH(__half, 3);
      else if (kernel == 2) DJ_POOL_LAUNCH(__half, 2);
      else DJ_POOL_LAUNCH(__half, 0);
    } else {
      if (kernel == 3) DJ_POOL_LAUNCH(__nv_bfloat16, 3);
      else if (kernel == 2) DJ_POOL_LAUNCH(__nv_bfloat16, 2);
      else DJ_POOL_LAUNCH(__nv_bfloat16, 0);
    }
#undef DJ_POOL_LAUNCH
  }
  return cudaGetLastError();
}

cudaError_t launch_pool(const void* x, void* y, int64_t rows, int C, int Cp, int H, int W, int OH,
                        int OW, int kernel, int stride, int pad, int is_max, int out_xu, int dt, cudaStream_t st) {
  (void)C;
  const int T = 256;
  if (dt != DT_F32 && Cp % 8 == 0 && out_xu > 1) {
    const int per_row = OH * OW * (Cp / 8);
    dim3 g(min(nblocks(per_row, T), 1024), (unsigned)(rows < 65535 ? rows : 65535));
    if (dt == DT_F16)
      launch_pdl(pool16_xu_kernel<__half>, dim3(g), dim3(T), 0, st, (const __half*)x, (__half*)y, rows, Cp, H, W, OH, OW, kernel, stride, pad, is_max, out_xu);
    else
      launch_pdl(pool16_xu_kernel<__nv_bfloat16>, dim3(g), dim3(T), 0, st, (const __nv_bfloat16*)x, (__nv_bfloat16*)y, rows, Cp, H, W, OH, OW, kernel, stride, pad, is_max, out_xu);
    return cudaGetLastError();
  }
  if (dt != DT_F32 && Cp % 8 == 0) {
    const int per_row = OH * OW * (Cp / 8) * out_xu;
    dim3 g(min(nblocks(per_row, T), 1024), (unsigned)(rows < 65535 ? rows : 65535));
    if (dt == DT_F16)
      launch_pdl(pool16_kernel<__half>, dim3(g), dim3(T), 0, st, (const __half*)x, (__half*)y, rows, Cp, H, W, OH, OW, kernel, stride, pad, is_max, out_xu);
    else
      launch_pdl(pool16_kernel<__nv_bfloat16>, dim3(g), dim3(T), 0, st, (const __nv_bfloat16*)x, (__nv_bfloat16*)y, rows, Cp, H, W, OH, OW, kernel, stride, pad, is_max, out_xu);
    return cudaGetLastError();
  }
  const int64_t n = rows * (int64_t)OH * OW * Cp;
  const int g = min(nblocks(n, T), 148 * 32);
  if (dt == DT_F32) launch_pdl(pool_kernel<float>, dim3(g), dim3(T), 0, st, (const float*)x, (float*)y, rows, Cp, H, W, OH, OW, kernel, stride, pad, is_max);
  else if (dt == DT_F16) launch_pdl(pool_kernel<__half>, dim3(g), dim3(T), 0, st, (const __half*)x, (__half*)y, rows, Cp, H, W, OH, OW, kernel, stride, pad, is_max);
  else launch_pdl(pool_kernel<__nv_bfloat16>, dim3(g), dim3(T), 0, st, (const __nv_bfloat16*)x, (__nv_bfloat16*)y, rows, Cp, H, W, OH, OW, kernel, stride, pad, is_max);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------
// K6: row softmax p_i = exp(z_i - max) / sum_j exp(z_j - max); argmax (ties -> lowest index).
// One CTA of 256 threads per row.
__device__ __forceinline__ void argmax_combine(float& v, int& i, float v2, int i2) {
  if (v2 > v || (v2 == v && i2 < i)) { v = v2; i = i2; }
}

__global__ void softmax_kernel(const float* __restrict__ z, int64_t rows, int N, int pitch,
                               void* __restrict__ out, int mode) {
  pdl_trigger();
  pdl_wait();
  __shared__ float s_v[32];
  __shared__ int s_i[32];
  const int64_t r = blockIdx.x;
  if (r >= rows) return;
  const float* zr = z + r * pitch;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (mode == 2) {
    float* o = (float*)out + r * N;
    for (int i = threadIdx.x; i < N; i += blockDim.x) o[i] = zr[i];
    return;
  }
  float m = -FLT_MAX;
  int mi = 0x7fffffff;
  for (int i = threadIdx.x; i < N; i += blockDim.x) argmax_combine(m, mi, zr[i], i);
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    const float v2 = __shfl_xor_sync(0xffffffffu, m, o);
    const int i2 = __shfl_xor_sync(0xffffffffu, mi, o);
    argmax_combine(m, mi, v2, i2);
  }
  if (lane == 0) { s_v[wid] = m; s_i[wid] = mi; }
  __syncthreads();
  if (wid == 0) {
    m = lane < nw ? s_v[lane] : -FLT_MAX;
    mi = lane < nw ? s_i[lane] : 0x7fffffff;
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      const float v2 = __shfl_xor_sync(0xffffffffu, m, o);
      const int i2 = __shfl_xor_sync(0xffffffffu, mi, o);
      argmax_combine(m, mi, v2, i2);
    }
    if (lane == 0) { s_v[0] = m; s_i[0] = mi; }
  }
  __syncthreads();
  m = s_v[0];
  mi = s_i[0];
  if (mode == 1) {
    if (threadIdx.x == 0) ((int*)out)[r] = mi;
    return;
  }
  __syncthreads();
  float s = 0.f;
  for (int i = threadIdx.x; i < N; i += blockDim.x) s += expf(zr[i] - m);
#pragma unroll
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) s_v[wid] = s;
  __syncthreads();
  if (wid == 0) {
    s = lane < nw ? s_v[lane] : 0.f;
#pragma unroll
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) s_v[0] = s;
  }
  __syncthreads();
  const float inv = 1.f / s_v[0];
  float* o = (float*)out + r * N;
  for (int i = threadIdx.x; i < N; i += blockDim.x) o[i] = expf(zr[i] - m) * inv;
}

// Single pass, values held in registers: one warp per row (N <= 32*VPT).
template <int VPT>
__global__ void softmax_warp_kernel(const float* __restrict__ z, int64_t rows, int N, int pitch, float* __restrict__ out) {
  pdl_trigger();
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int64_t r = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5);
  if (r >= rows) return;
  const float* zr = z + r * pitch;
  float v[VPT];
  float m = -FLT_MAX;
#pragma unroll
  for (int j = 0; j < VPT; ++j) {
    const int i = lane + 32 * j;
    v[j] = i < N ? zr[i] : -FLT_MAX;
    m = fmaxf(m, v[j]);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  float s = 0.f;
#pragma unroll
  for (int j = 0; j < VPT; ++j) {
    v[j] = (lane + 32 * j) < N ? expf(v[j] - m) : 0.f;
    s += v[j];
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  const float inv = 1.f / s;
  float* orow = out + r * N;
#pragma unroll
  for (int j = 0; j < VPT; ++j) {
    const int i = lane + 32 * j;
    if (i < N) orow[i] = v[j] * inv;
  }
}

// Single pass for long rows (N <= 256*4*VQ, e.g. the 8000 ASR senones): one CTA of 256 threads
// per row, float4 loads, exp values kept in registers between the reductions.
template <int VQ>
__global__ void softmax_block_kernel(const float* __restrict__ z, int64_t rows, int N, int pitch, float* __restrict__ out) {
  pdl_trigger();
  pdl_wait();
  __shared__ float red[8];
  const int64_t r = blockIdx.x;
  const int t = threadIdx.x, lane = t & 31, wid = t >> 5;
  const float* zr = z + r * pitch;
  float4 v[VQ];
  float m = -FLT_MAX;
#pragma unroll
  for (int j = 0; j < VQ; ++j) {
    const int i = 4 * (t + 256 * j);
    if (i + 3 < N) {
      v[j] = *reinterpret_cast<const float4*>(zr + i);
    } else {
      v[j].x = i < N ? zr[i] : -FLT_MAX;
      v[j].y = i + 1 < N ? zr[i + 1] : -FLT_MAX;
      v[j].z = i + 2 < N ? zr[i + 2] : -FLT_MAX;
      v[j].w = -FLT_MAX;
    }
    m = fmaxf(fmaxf(m, fmaxf(v[j].x, v[j].y)), fmaxf(v[j].z, v[j].w));
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  if (lane == 0) red[wid] = m;
  __syncthreads();
  m = red[0];
#pragma unroll
  for (int k = 1; k < 8; ++k) m = fmaxf(m, red[k]);
  __syncthreads();
  float s = 0.f;
#pragma unroll
  for (int j = 0; j < VQ; ++j) {
    const int i = 4 * (t + 256 * j);
    v[j].x = i < N ? expf(v[j].x - m) : 0.f;
    v[j].y = i + 1 < N ? expf(v[j].y - m) : 0.f;
    v[j].z = i + 2 < N ? expf(v[j].z - m) : 0.f;
    v[j].w = i + 3 < N ? expf(v[j].w - m) : 0.f;
    s += (v[j].x + v[j].y) + (v[j].z + v[j].w);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) red[wid] = s;
  __syncthreads();
  s = 0.f;
#pragma unroll
  for (int k = 0; k < 8; ++k) s += red[k];
  const float inv = 1.f / s;
  float* orow = out + r * N;
  const bool vec = (N % 4) == 0;
#pragma unroll
  for (int j = 0; j < VQ; ++j) {
    const int i = 4 * (t + 256 * j);
    float4 p = make_float4(v[j].x * inv, v[j].y * inv, v[j].z * inv, v[j].w * inv);
    if (vec && i + 3 < N) {
      *reinterpret_cast<float4*>(orow + i) = p;
    } else {
      if (i < N) orow[i] = p.x;
      if (i + 1 < N) orow[i + 1] = p.y;
      if (i + 2 < N) orow[i + 2] = p.z;
      if (i + 3 < N) orow[i + 3] = p.w;
    }
  }
}

cudaError_t launch_softmax(const float* logits, int64_t rows, int N, int pitch, void* out, int mode,
                           cudaStream_t st) {
  if (rows <= 0) return cudaSuccess;
  if (mode == 0 && N <= 256 && pitch % 4 == 0) {
    const int rpb = 8;  // rows (warps) per 256-thread block
    const unsigned g = (unsigned)((rows + rpb - 1) / rpb);
    if (N <= 64) launch_pdl(softmax_warp_kernel<2>, dim3(g), dim3(256), 0, st, logits, rows, N, pitch, (float*)out);
    else launch_pdl(softmax_warp_kernel<8>, dim3(g), dim3(256), 0, st, logits, rows, N, pitch, (float*)out);
  } else if (mode == 0 && N <= 8192 && pitch % 4 == 0) {
    launch_pdl(softmax_block_kernel<8>, dim3((unsigned)rows), dim3(256), 0, st, logits, rows, N, pitch, (float*)out);
  } else {
    launch_pdl(softmax_kernel, dim3((unsigned)rows), dim3(256), 0, st, logits, rows, N, pitch, out, mode);
  }
  return cudaGetLastError();
}

}  // namespace djinn
