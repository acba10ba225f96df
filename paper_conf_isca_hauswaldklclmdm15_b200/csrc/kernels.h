// Kernel launch interface of libdjinn (host side).  Every function enqueues work on
// `stream` and returns cudaError_t of the launch.  Layouts: activations are NHWC per
// row with a channel pitch Cp (PAPER.md L63-65 layers; DESIGN.md sec 4 "data layout").
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace djinn {

// ---- programmatic dependent launch (PDL) --------------------------------------------------
// Every kernel of a forward pass is launched with programmatic stream serialization: kernel i+1
// may be scheduled while kernel i drains its last wave, runs its prologue (barrier init, TMEM
// allocation, tensor-map prefetch) and then blocks in pdl_wait() -- griddepcontrol.wait returns
// once kernel i has COMPLETED and its memory is visible -- before its first global access.
// Each kernel calls pdl_trigger() on entry.  DJINN_PDL=0 disables the attribute (plain stream order).
#if defined(__CUDACC__)
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
// Packed fp32 pairs (sm_100 FFMA2/FMUL2/FADD2: two IEEE round-to-nearest fp32 results per issue
// slot, bitwise equal to the scalar ops).  The LRN epilogues are issue-bound, not MUFU-bound.
__device__ __forceinline__ float2 fma2(float2 a, float2 b, float2 c) {
  float2 r;
  asm("{.reg .b64 a, b, c, d;\n\tmov.b64 a, {%2, %3};\n\tmov.b64 b, {%4, %5};\n\tmov.b64 c, {%6, %7};\n\t"
      "fma.rn.f32x2 d, a, b, c;\n\tmov.b64 {%0, %1}, d;}"
      : "=f"(r.x), "=f"(r.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y), "f"(c.x), "f"(c.y));
  return r;
}
__device__ __forceinline__ float2 mul2(float2 a, float2 b) {
  float2 r;
  asm("{.reg .b64 a, b, d;\n\tmov.b64 a, {%2, %3};\n\tmov.b64 b, {%4, %5};\n\t"
      "mul.rn.f32x2 d, a, b;\n\tmov.b64 {%0, %1}, d;}"
      : "=f"(r.x), "=f"(r.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
  return r;
}
__device__ __forceinline__ float2 add2(float2 a, float2 b) {
  float2 r;
  asm("{.reg .b64 a, b, d;\n\tmov.b64 a, {%2, %3};\n\tmov.b64 b, {%4, %5};\n\t"
      "add.rn.f32x2 d, a, b;\n\tmov.b64 {%0, %1}, d;}"
      : "=f"(r.x), "=f"(r.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
  return r;
}
#endif
bool pdl_enabled();
// cudaFuncSetAttribute(MaxDynamicSharedMemorySize, bytes) once per (device, kernel, bytes)
cudaError_t ensure_max_smem(const void* kernel, int bytes);
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

enum DType { DT_F32 = 0, DT_BF16 = 1, DT_F16 = 2 };
// ACT_SIGMOID_C stores sigma(x) - 1/2 ("centered" storage, an exact reparametrisation: the
// consumer's bias absorbs + 1/2 * rowsum(W)); it keeps 16-bit activations near 0 where their
// relative precision is best.
enum Act { ACT_NONE = 0, ACT_RELU = 1, ACT_SIGMOID = 2, ACT_TANH = 3, ACT_HARDTANH = 4, ACT_SIGMOID_C = 5 };
enum GemmMode { GM_DENSE = 0, GM_CONV = 1, GM_LC = 2 };

// One convolution / locally-connected / fully-connected layer as an implicit GEMM:
//   Y[pix(m), goff + n] = act( bias + sum_k A[m,k] * B[z][n][k] )
// m enumerates output pixels (conv: (img,oy,ox); LC: img at location z; dense: row),
// k enumerates (ky, kx, c) with c fastest (NHWC), z = group (conv) or location (LC).
struct GemmGeom {
  int mode;
  int M;              // GEMM rows
  int N;              // valid output channels per z (Cog / Co / No)
  int Z;              // groups (conv), locations (LC) or 1
  int K;              // valid K (conv/LC: KH*KW*Cgp; dense: row length)
  int Kpad;           // K rounded up to the k-block (64) -- B row length
  // gather geometry (conv / LC)
  int H, W, Cp_in;    // input image per row and its channel pitch
  int OH, OW;
  int KH, KW, stride, pad;
  int Cgp;            // channels per group used in K (multiple of 8 on 16-bit paths)
  int cin_goff;       // input channel offset between groups
  // dense A
  int a_pitch;        // dense: elements per A row
  // output
  int out_pitch;      // elements per output pixel (Cp_out) or per row (dense)
  int cout_goff;      // output channel offset between groups
  int write_cols;     // columns written per z: valid N plus zero-filled pad up to here
  int bias_zstride;   // bias elements between z (LC: Co per location; conv: Cog)
  int act;
  int out_f32;        // 1: fp32 output (logits), 0: same 16-bit type as input
  int out_gsz, out_gpitch;  // output channel c stored at (c/out_gsz)*out_gpitch + c%out_gsz
  // tensor-core path only
  int cw;             // A chunk width in elements (16 / 32 / 64): one TMA box per chunk
  int Nimg;           // conv: images in the batch
  int xb, OWb;        // conv x-blocking: one GEMM row = xb adjacent output pixels (OWb blocks per
                      // output row); columns are (dx, co) with co < out_pitch; 1 = off
  int Co;             // real output channels (x-blocked conv: per dx)
  int lcg, kwp;       // LC: taps per TMA row (box {Cgp, lcg, 1, 128}) and KW padded to lcg
  int kxs;            // conv: x offset between consecutive taps (x-unrolled input: xu), default 1
  int xstep;          // conv: input-x offset between consecutive GEMM-row pixels (blocks):
                      //   stride, or xb when x-blocked, or 1 over a block-packed first layer
  int cg;             // 1: one CTA per 128-row tile; 2: cta_group::2 CTA pair per 256-row tile (B split)
  int out_half;       // 16-bit output stored as fp16 whatever the path type (an LRN-only consumer)
  int a_tiled;        // conv: 0 = im2col-mode TMA over linear output pixels (default), 1 = tiled
                      //       4D boxes over bx x by x bn pixel blocks (DJINN_CONV_A=tiled)
  int bx, by, bn;     // conv: output-pixel block of one M tile (bx*by*bn == 128), x fastest
  int zf;             // z values fused per CTA (groups computed by one CTA; TMEM columns zf*BN)
  int epi_lrn;        // 1: Caffe LRN across the zf*N channels of a pixel in the epilogue
  // slab convolution (stride 1, 64-channel chunks): GEMM row m = virtual pixel of the stored
  // (bordered) input grid Hv x Wv, m = (img * Hv + y) * Wv + x; a tile's rows read ONE
  // contiguous slab of input pixels [m0, m0 + 128 + (KH-1)*Wv + KW-1) loaded once by TMA, and
  // filter tap (ky, kx) is the UMMA A descriptor shifted by ky*Wv + kx rows.  Rows with
  // y >= OH or x >= OWb are computed and discarded.
  int slab, Hv, Wv;
  int slab_parts, slab_rows;  // the slab is loaded as slab_parts TMA boxes of slab_rows rows
  int stages;         // slab mode: B ring stages (runtime; set by tc_slab_config)
  int kv16;           // slab mode, one 64-channel chunk per tap: 16-channel K sub-steps holding
                      //   real channels (3 for 48 of 64: the 4th is zero padding and gets no MMA,
                      //   a compile-time variant of the kernel); 4 otherwise
  int kps;            // slab mode: K blocks of B per ring stage (one MMA commit per stage)
  int tslots;         // TMEM accumulator slots: 0 = as many as fit (<= 4), 2 = two (DJINN_TSLOTS=2)
  int epi_wg;         // epilogue warpgroups draining tiles: 3 (3 slots) or 2 (up to 4 slots)
  int ldwait;         // slab mode: B-loader stage wait (0 spin, 1 poll + nanosleep back-off, 2 suspend hint)
  int obd;            // conv output: zero border of the stored output tensor (its consumer's pad)
  int ksplit, kpb;    // dense split-K: z = K split (ksplit > 1), kpb K blocks each; the launch writes
                      // fp32 partial sums [ksplit][M][out_pitch] with no bias / activation
  int lrn_size;
  float lrn_alpha_over_n, lrn_beta, lrn_k;
};

// --- pack (K0): fp32 NCHW rows -> NHWC with channel pitch Cp, type dt -------------------
// mode 0: y[r][h][w][c] = x[r][c][h][w];  mode 1 (space-to-depth by f):
// y[r][ty][tx][(dy*f+dx)*C + c] = x[r][c][f*ty+dy][f*tx+dx];  mode 2 (kx-unroll of width f,
// packed pixels xs input pixels apart -- xs = the conv's x-block, so only the pixels the
// GEMM rows start at are written): y[r][h][j][kx*C + c] = x[r][c][h][j*xs+kx].
// Out-of-range sources and pad channels are 0.
cudaError_t launch_pack_input(const float* x, void* y, int64_t rows, int C, int H, int W, int mode, int f, int xs,
                              int Ho, int Wo, int Cp, int dt, cudaStream_t st);

// --- djinn_forward16: 16-bit input rows (the path's type dt) -> fp32, exact ----------------
cudaError_t launch_widen16(const void* x, float* y, int64_t n, int dt, cudaStream_t st);

// --- SENNA window lookup (K0 variant) ------------------------------------
// x: float32 [rows][window * T] feature indices, word-major (x[r][w*T + t]);
// tables: the path's type, table t = [vocab[t]][dim[t]] at element offset toff[t];
// y[r][w*D + sum(dim[:t]) + j] = tables_t[x[r][w*T+t]][j], D = sum(dim), pitch Cp (pad
// columns zero).  An index that is not an integer in [0, vocab[t]) gives the zero vector.
constexpr int EMBED_MAX_TABLES = 8;
struct EmbedGeom {
  int window, T, D;
  int vocab[EMBED_MAX_TABLES], dim[EMBED_MAX_TABLES];
  long long toff[EMBED_MAX_TABLES];
};
cudaError_t launch_embed(const float* x, const void* tables, void* y, int64_t rows, const EmbedGeom& eg, int Cp, int dt,
                         cudaStream_t st);

// --- SIMT fp32 implicit GEMM (K7; exact fp32 FFMA accumulation) --------------------------
// B: [Z][N][K] fp32 (K unpadded), bias fp32.
cudaError_t launch_simt_gemm(const GemmGeom& g, const float* A, const float* B, const float* bias,
                             float* Y, cudaStream_t st);

// --- tcgen05 tensor-core implicit GEMM (K1/K2/K3) -----------------------------------------
// tmB: 3D tensor map over B [Z][N][Kpad] (16-bit, SWIZZLE_128B, box {64, BN, 1}).
// tmA: conv -> 4D tiled map over the NHWC input, box {cw, bx*s, by*s, bn}, element strides
//              {1, s, s, 1}: the tap (kx,ky) of a bx x by x bn block of output pixels;
//      LC   -> 4D tiled map over the NHWC input, box {cw, 1, 1, 128};
//      dense-> 2D tiled map over [rows][a_pitch], box {64, 128}.
// Swizzle of A boxes: cw*2 bytes (32B / 64B / 128B).
int tc_pick_bn(const GemmGeom& g);
int tc_pick_cg(const GemmGeom& g, int bn);  // 2 when a CTA pair (cta_group::2) pays off
int tc_num_sms();
// Slab mode feasibility for tile width bn (CTA pair): sets g.stages; false = use im2col.
bool tc_slab_config(GemmGeom& g, int bn);
cudaError_t launch_tc_gemm(const GemmGeom& g, int bn, int dt, const CUtensorMap* tmA,
                           const CUtensorMap* tmB, const float* bias, void* Y, cudaStream_t st);

// --- first-layer strided conv with a resident filter bank (K2 [+ K4], k_stem.cu): space-to-depth
// by the stride F into an Hs x Ws grid, KS x KS stride-1 taps, bias + act [+ Caffe LRN], 16-bit
// NHWC output over the whole virtual grid [Nimg * Hs * Ws][N] written by TMA tensor stores.
// gather = 1: reads the fp32 NCHW images x itself (K0 fused); gather = 0: reads the packed
// 16-bit space-to-depth tensor through tmA (2D {64, rows * Hs * Ws}, box {64, slab_rows}).
// tmB: as launch_tc_gemm (box {64, N/2, 1}); tmY0: 2D map {Cp, rows * Hs * Ws} of the output,
// box {64, 32}, SWIZZLE_128B; tmY1: the same map with box {32, 32}, SWIZZLE_64B (gather only;
// otherwise channels past 64 are stored from registers into Y).
struct StemGeom {
  int Nimg;            // images in this launch
  int H, W;            // fp32 input image (C0 channels)
  int Hs, Ws;          // space-to-depth grid (virtual GEMM rows per image = Hs * Ws)
  int OH, OW;          // valid output pixels
  int N;               // output channels (= tile width, = output pitch)
  int act, epi_lrn, out_half;
  int gather, slab_rows;
  float lrn_alpha_over_n, lrn_beta, lrn_k;
  // pool = 1: the following 3 x 3 / stride-2 MAX pool is fused (requires epi_lrn, !gather,
  // !out_half): Y is the pooled tensor [Nimg][POH + 2 obd][POW + 2 obd][Cpo] (the border is
  // never written), channel c of half h = c / (N / 2) at h * pool_gp + c % (N / 2), the rest of
  // each half's pool_gp channels written 0; bands = pool-row bands per image (stem_pool_bands)
  int pool, POH, POW, bands, Cpo, pool_gp, obd;
};
bool stem_supported(int bn, int f, int c0, int ks, int out_pitch);
bool stem_pool_supported(int n, int ws, int oh, int ow, int kernel, int stride, int pad, int cpo, int gsz, int gpitch,
                         int xu);
int stem_pool_bands(int nimg, int poh);
// stem_dense_b(): the filter bank of a stem op is stored dense in K (tap t, channel c at K index
// t * F*F*C0 + c, zeros from KS*KS*F*F*C0 to Kpad) instead of one 64-channel block per tap; tmBc is
// then a 2D {rup(KS*KS*F*F*C0, 64), N} map of it (row pitch Kpad), box {64, N / 2}, SWIZZLE_128B
// (IMC: 7 resident K blocks, 84 KB, instead of 9, 108 KB).
bool stem_dense_b();
cudaError_t launch_stem_conv(const StemGeom& g, int dt, const CUtensorMap* tmA, const CUtensorMap* tmB,
                             const CUtensorMap* tmBc, const CUtensorMap* tmY0, const CUtensorMap* tmY1, const float* x,
                             const float* bias, void* Y, cudaStream_t st);

// --- fused two-layer MLP + softmax (k_mlp.cu; the SENNA window nets): fp32 rows x [rows][K0]
// -> h = act1(x W1^T + b1) (N1) -> z = h W2^T + b2 (N2) -> out (mode 0 prob fp32 [rows][N2],
// 1 argmax int32 [rows], 2 logits fp32 [rows][N2]).  W1 / W2 are the arena's [N][Kpad] 16-bit
// matrices; tmW1: 2D {K0p, N1}, box {32, N1p / 2}, SWIZZLE_64B; tmW2: 2D {K1p, N2}, box {64, N2p},
// SWIZZLE_128B.
struct MlpGeom {
  int64_t rows;
  int K0, K0p;         // input row length, padded to 64 (W1's Kpad)
  int N1, N1p, N1c;    // layer 1 outputs, padded to 16; TMEM column of layer 2's accumulator
  int K1p;             // W2's Kpad (layer 1 outputs padded to 64)
  int N2, N2p;         // logits, padded to 16 (<= 64)
  int act1, out_mode;
  int rpc;             // rows per CTA (<= 128, multiple of 8; 0 = 128)
  int a_tma;           // 1: layer 1's A is a 16-bit tensor [rows][K0p] read by TMA (tmA), x unused;
                       //    N1c = 0 then lets layer 2 reuse layer 1's TMEM columns
  int nsplit;          // a_tma: clusters of nsplit CTAs split layer 1's N1p columns (tmW1's box is
                       //    then {32, N1p / nsplit / 2}); CTA 0 sums the partial logits (0/1: no split)
};
// rows per CTA for a forward of `rows` rows: the smallest of 128 / 64 / 32 that keeps the grid
// within one wave of SMs (DJINN_MLP_RPC overrides)
int mlp2_rows_per_cta(int64_t rows);
int mlp2_smem(const MlpGeom& g);
int mlp2_wk(int a_tma);  // K columns per ring stage: 32 (SW64 boxes) or, TMA-fed, 64 (SW128)
bool mlp2_supported(const MlpGeom& g);
cudaError_t launch_mlp2(const MlpGeom& g, int dt, const CUtensorMap* tmW1, const CUtensorMap* tmW2, const CUtensorMap* tmA,
                        const float* x, const float* b1, const float* b2, void* out, cudaStream_t st);

// --- dense layer + row softmax fused over a thread-block cluster (k_smx.cu; ASR's output
// layer): z = x W^T + b for M rows x N columns (x: 16-bit [rows][>= Kpad], W: the arena's
// [N][Kpad]), then mode 0 p = softmax(z) fp32 [M][N], 1 argmax int32 [M], 2 z fp32 [M][N].
// A cluster of CL CTAs owns 128 rows; CTA r computes columns [r NCW, r NCW + NCW) in its tensor
// memory.  tmA: 2D {Kpad, rows}, box {32, 128 / CL}, SWIZZLE_64B; tmB: 2D {Kpad, N}, box
// {32, 256}, SWIZZLE_64B.  smx_plan: CL (power of two <= 16) and NCW for N (false: unsupported).
struct SmxGeom {
  int64_t M;
  int N, Kpad, CL, NCW, out_mode;
};
bool smx_plan(int N, int Kpad, int* CL, int* NCW);
int smx_bk();  // K per pipeline stage (the A / B box width)
int smx_max_active_clusters(int dt, int CL);
cudaError_t launch_smx(const SmxGeom& g, int dt, const CUtensorMap* tmA, const CUtensorMap* tmB, const float* bias,
                       void* out, cudaStream_t st);

// --- split-K reduction: y[m][n] = act(bias[n] + sum_s part[s][m][n]) for n < N, 0 for
// N <= n < write_cols; part fp32 [S][rows][ppitch]; y 16-bit (dt) or fp32 (out_f32) with row
// pitch out_pitch.  The partial sums are added in split order (deterministic).
cudaError_t launch_splitk_reduce(const float* part, int S, int64_t rows, int N, int ppitch, const float* bias, int act,
                                 void* y, int out_pitch, int write_cols, int out_f32, int dt, cudaStream_t st);

// --- LRN across channels (K4), NHWC ----------------------------------------------------------
// Channel c of a pixel is stored at (c/gsz)*gpitch + c%gsz (grouped layouts); pads -> 0.
cudaError_t launch_lrn(const void* x, void* y, int64_t pixels, int C, int Cp, int gsz, int gpitch, int size,
                       float alpha, float beta, float k, int dt, cudaStream_t st);

// --- MAX pooling with a channel-layout change (plain/grouped in, plain/grouped/x-unrolled out), 16-bit,
// kernel <= stride + 1.  obd: zero border of the stored output ((OH+2obd) x (OW+2obd) pixels;
// the border is never written).
// The input is stored on an Hst x Wst grid (>= H x W; pixel (y, x) at y * Wst + x).
cudaError_t launch_pool_remap(const void* x, void* y, int64_t rows, int C, int Cpi, int gsz_i, int gpitch_i, int H,
                              int W, int Hst, int Wst, int OH, int OW, int kernel, int stride, int pad, int Cpo, int gsz_o,
                              int gpitch_o, int xu, int obd, int dt, cudaStream_t st);

// --- LRN + max pooling fused (K4+K5): fp16 NHWC input (pitch Cpi, C channels, pads zero),
// Caffe LRN across channels in fp32, Caffe MAX pooling (kernel 3, stride 2, pad 0) of the LRN
// output; output in type dt with a grouped channel layout (gsz, gpitch, pitch Cpo; pads written
// as 0) and a zero border of obd pixels (never written).  Each LRN value is computed once.
cudaError_t launch_lrn_pool(const void* x, void* y, int64_t rows, int C, int Cpi, int H, int W, int OH, int OW,
                            int kernel, int stride, int pad, int out_gsz, int out_gpitch, int Cpo, int obd, int size,
                            float alpha, float beta, float k, int dt, cudaStream_t st);

// --- pooling (K5), NHWC, Caffe ceil geometry ------------------------------------------------
// Output may be x-unrolled: pixel x stores pooled pixels x..x+out_xu-1 at pitch Cp each
// (out pitch out_xu*Cp); slots past the right edge are zero.
cudaError_t launch_pool(const void* x, void* y, int64_t rows, int C, int Cp, int H, int W, int OH,
                        int OW, int kernel, int stride, int pad, int is_max, int out_xu, int dt, cudaStream_t st);

// --- softmax / argmax / logits copy (K6) ----------------------------------------------------
// logits fp32 [rows][pitch]; mode 0: prob fp32 [rows][N]; 1: argmax int32 [rows]; 2: logits copy.
cudaError_t launch_softmax(const float* logits, int64_t rows, int N, int pitch, void* out, int mode,
                           cudaStream_t st);

}  // namespace djinn
