// Host-side runtime of libdjinn: net-description parser, execution plan, weight arena,
// per-stream workspaces.  The service model is PAPER.md sec 3.1 (L77-84): a pretrained
// model is loaded once and shared read-only by all concurrent requests.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <atomic>
#include <map>
#include <memory>
#include <mutex>
#include <stdexcept>
#include <string>
#include <vector>

#include "kernels.h"

namespace djinn {

struct Error : std::runtime_error {
  int code;
  Error(int c, const std::string& m) : std::runtime_error(m), code(c) {}
};

// ---- parsed description (subset of Caffe prototxt) --------------------------------------
struct PNode {
  std::map<std::string, std::vector<std::string>> scalars;
  std::map<std::string, std::vector<PNode>> blocks;
  const std::string* get(const std::string& k) const;
  const PNode* block(const std::string& k) const;
  int geti(const std::string& k, int def) const;
  double getf(const std::string& k, double def) const;
  std::string gets(const std::string& k, const std::string& def) const;
};
PNode parse_prototxt(const std::string& text);  // throws Error(DJINN_E_PARSE)

struct LayerSpec {
  std::string name, type;
  int num_output = 0, kernel = 0, stride = 1, pad = 0, group = 1;
  bool pool_max = true;
  int lrn_size = 5;
  float alpha = 1.f, beta = 0.75f, lrn_k = 1.f;
  std::vector<int> dims;
  int window = 1;                  // Embedding: words per window, tables' vocabularies and dims
  std::vector<int> vocab, edim;
};

enum OpKind { OP_PACK, OP_GEMM, OP_LRN, OP_POOL, OP_SOFTMAX, OP_LRNPOOL };

// Per-row activation tensor: NHWC, channel pitch Cp.  Channels may be stored in groups of
// gsz at a per-group pitch gpitch (logical channel c lives at (c / gsz) * gpitch + c % gsz),
// so that a grouped convolution's per-group K is 16/32/64-aligned (one TMA row per tap).
struct Shape {
  int C = 0, H = 1, W = 1, Cp = 0;
  int gsz = 1 << 30, gpitch = 1 << 30;
  int xu = 1, P = 0;  // x-unrolled layout: pixel x stores pixels x..x+xu-1, each at pitch P (Cp = xu*P)
  int bdr = 0;        // zero border: stored (H + 2 bdr) x (W + 2 bdr) pixels, pixel (y, x) at (y + bdr, x + bdr)
                      // (the input of a slab convolution: its zero padding is stored)
  int hx = 0, wx = 0; // extra stored rows / columns after the image (never read): the fused first
                      // layer writes its whole virtual Hs x Ws grid (k_stem.cu), pixel (y, x) at (y, x)
  int64_t per_row() const { return (int64_t)(H + 2 * bdr + hx) * (W + 2 * bdr + wx) * Cp; }
  int pos(int c) const { return (c / gsz) * gpitch + c % gsz; }
};

struct Op {
  OpKind kind;
  std::string name;
  Shape in, out;
  int in_buf = 0, out_buf = 0;  // 0/1 ping-pong, 2 logits, 3.. dedicated (bordered), -1 external input
  // gemm
  GemmGeom g{};
  int bn = 0;
  size_t w_off = 0, b_off = 0;  // bytes into the weight arena
  CUtensorMap tmB{};
  int ohw = 1;                  // output pixels per row (conv M = rows * ohw)
  bool fold_half = false;       // bias += 1/2 * rowsum(W): the producer stores sigma - 1/2
  // first-layer input transform (PACK op and the conv it feeds): 0 none, 1 space-to-depth
  // by xf (= conv stride), 2 kx-unroll of a stride-1 kernel of width xf
  int xform = 0, xf = 1, xs = 1;  // xs: kx-unroll x step (packed pixel j starts at input x = j*xs)
  Shape orig_in;                // the layer's input before the transform
  // first-layer kernel with a resident filter bank (k_stem.cu): stem = 2 reads the packed
  // space-to-depth tensor by TMA; stem = 1 reads the fp32 input itself and the pack op before
  // it is not launched (fused = 1)
  int stem = 0, fused = 0;
  int stem_pool = 0;            // stem = 2 with the following MAX pool in its epilogue (the pool op is fused)
  CUtensorMap tmBc{};           // stem: the filter bank as 16-channel SW32 boxes (compact resident B)
  // fused two-layer MLP + softmax (k_mlp.cu): this GEMM op runs the whole net (mlp = 1); the
  // pack, the second GEMM and the softmax ops are not launched (fused = 1)
  int mlp = 0;
  // dense split-K (ksplit > 1): the GEMM writes fp32 partials over ksplit K ranges of kpb
  // K blocks into the workspace's part buffer (pitch npart), a reduction adds bias + act
  int ksplit = 1, kpb = 0, npart = 0;
  MlpGeom mg{};
  CUtensorMap tmW1{}, tmW2{};
  // dense layer + softmax over a thread-block cluster (k_smx.cu): this GEMM op writes the
  // probabilities itself when a forward has >= smx_min_rows rows (the softmax op is then not
  // launched); smx_cl CTAs of smx_ncw columns per 128 rows; tmBs: its own B map (SW64 boxes)
  int smx = 0, smx_cl = 0, smx_ncw = 0;
  int64_t smx_min_rows = 0;
  CUtensorMap tmBs{};
  // SENNA window lookup in place of the pack (embed = 1): see EmbedGeom (kernels.h)
  int embed = 0;
  EmbedGeom eg{};
  int orig_k = 0;               // original kernel size
  // lrn
  int lrn_size = 5;
  float alpha = 0, beta = 0, lrn_k = 1;
  // pool
  int kernel = 0, stride = 1, pad = 0, is_max = 1;
  // algorithmic work (djinn_op_info): per batch row, and once per launch
  double flops_row = 0, bytes_row = 0, weight_bytes = 0;
};

struct ProfRec {  // one timed forward chunk: events[first .. first + n_ops]
  size_t first;
  int n_ops;
  int op;         // -1: every op (n_ops + 1 events); >= 0: only op `op` (events[first], events[first + 1])
};

struct Workspace {
  std::vector<void*> buf;  // 0/1 ping-pong, 2 logits, 3.. dedicated bordered tensors (borders stay zero)
  float* in_stage = nullptr;
  uint16_t* in_stage16 = nullptr;  // djinn_forward16 host rows (two slots like in_stage)
  float* in_wide = nullptr;        // djinn_forward16: one chunk of rows widened to fp32 (read by
                                   // the pack; never shared with the H2D staging slots)
  void* out_stage = nullptr;
  // host-fed mode: H2D on `cin`, D2H on `cout`, compute on the caller's stream; two staging
  // slots, each with a "filled" and a "drained" event (Net::forward)
  cudaStream_t cin = nullptr, cout = nullptr;
  cudaEvent_t in_ready[2] = {}, in_free[2] = {}, out_ready[2] = {}, out_free[2] = {};
  int64_t pipe_cs = 0;  // chunk rows of the last host-fed call (slot offsets depend on it)
  std::vector<CUtensorMap> tmA;  // per op (dense gemm) over its input buffer
  std::vector<CUtensorMap> tmAs;  // per op (smx): the same buffer, 32-K SW64 boxes of 128 / CL rows
  std::vector<CUtensorMap> tmY0, tmY1;  // per op (stem): TMA-store maps over its output buffer
  float* part = nullptr;                 // split-K partial sums (the largest need of any op)
  ~Workspace();
};

struct Net {
  int device = 0;
  int precision = 0;  // DJINN_FP32 / BF16 / FP16
  int dt = DT_F32;
  int64_t max_rows = 0;
  std::string name;
  int rows_per_query = 1;
  std::vector<LayerSpec> layers;
  std::vector<Op> ops;
  int64_t in_elems = 0, out_elems = 0, n_params = 0, n_layers = 0;
  int out_pitch = 0;  // logits pitch
  void* arena = nullptr;
  size_t arena_bytes = 0;
  std::vector<size_t> buf_bytes = std::vector<size_t>(3, 0);
  std::mutex mu;
  std::map<cudaStream_t, std::unique_ptr<Workspace>> ws;
  bool poisoned = false;
  // per-op profiling (djinn_profile)
  bool profile = false;
  int profile_op = -1;  // -1: time every op; k >= 0: time op k only (djinn_profile(net, 2 + k))
  std::vector<cudaEvent_t> prof_events;
  size_t prof_used = 0;
  std::vector<ProfRec> prof_recs;
  cudaEvent_t prof_event();
  void prof_clear();
  ~Net();

  void build(const std::string& desc);                          // parse + plan
  void choose_tiles();                                          // tile widths, CTA pairs, slab smem
  void load_weights(const float* w, size_t n, int mem);         // pack into the arena
  Workspace* workspace(cudaStream_t st);
  void forward(const float* in, int64_t rows, int in_mem, void* out, int out_mem, int mode,
               cudaStream_t st, bool in16 = false);
  std::string plan_string() const;
};

std::atomic<int64_t>& launch_counter();
bool host_prof_on();
void set_last_error(const std::string& msg);  // djinn_last_error() of the calling thread (api.cu)
void host_prof_add(const std::string& key, double us);
void encode_tmap(CUtensorMap* m, int dt, const void* base, int rank, const uint64_t* dims,
                 const uint64_t* strides_bytes, const uint32_t* box, int swizzle_bytes = 128,
                 const uint32_t* elem_strides = nullptr);
void encode_im2col(CUtensorMap* m, int dt, const void* base, const uint64_t* dims, const uint64_t* strides_bytes,
                   const int* lower_wh, const int* upper_wh, int channels, int pixels, const uint32_t* elem_strides);

}  // namespace djinn

// The C ABI's opaque handle (include/djinn.h).
struct djinn_net {
  djinn::Net impl;
};
