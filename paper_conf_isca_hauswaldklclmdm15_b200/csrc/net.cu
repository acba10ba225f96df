// Host runtime of libdjinn: prototxt-subset parser, shape inference, execution plan,
// weight packing into one device arena, per-stream workspaces and the forward driver.
//
// Service model (sec 3.1): DjiNN "loads the pre-trained model associated with
// each application into memory, giving all worker threads read-only access" (L84);
// the DNN library is Caffe's configurable layer framework (L77-78), so the description
// format is a Caffe-prototxt subset.  Batching stacks queries into larger matrices (L185).
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <string.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cctype>
#include <sstream>

#include "../../include/djinn.h"
#include "net.h"

namespace djinn {

// ============================================================================ parser
const std::string* PNode::get(const std::string& k) const {
  auto it = scalars.find(k);
  return (it == scalars.end() || it->second.empty()) ? nullptr : &it->second[0];
}
const PNode* PNode::block(const std::string& k) const {
  auto it = blocks.find(k);
  return (it == blocks.end() || it->second.empty()) ? nullptr : &it->second[0];
}
int PNode::geti(const std::string& k, int def) const {
  const std::string* s = get(k);
  if (!s) return def;
  char* end = nullptr;
  long v = strtol(s->c_str(), &end, 10);
  if (!end || *end) throw Error(DJINN_E_PARSE, "field '" + k + "' is not an integer: " + *s);
  return (int)v;
}
double PNode::getf(const std::string& k, double def) const {
  const std::string* s = get(k);
  if (!s) return def;
  char* end = nullptr;
  double v = strtod(s->c_str(), &end);
  if (!end || *end) throw Error(DJINN_E_PARSE, "field '" + k + "' is not a number: " + *s);
  return v;
}
std::string PNode::gets(const std::string& k, const std::string& def) const {
  const std::string* s = get(k);
  return s ? *s : def;
}

namespace {
struct Lexer {
  const std::string& t;
  size_t i = 0;
  explicit Lexer(const std::string& s) : t(s) {}
  bool next(std::string& tok) {
    for (;;) {
      while (i < t.size() && isspace((unsigned char)t[i])) ++i;
      if (i < t.size() && t[i] == '#') {
        while (i < t.size() && t[i] != '\n') ++i;
        continue;
      }
      break;
    }
    if (i >= t.size()) return false;
    char c = t[i];
    if (c == '{' || c == '}' || c == ':') { tok.assign(1, c); ++i; return true; }
    if (c == '"') {
      size_t j = t.find('"', i + 1);
      if (j == std::string::npos) throw Error(DJINN_E_PARSE, "unterminated string");
      tok = t.substr(i, j - i + 1);
      i = j + 1;
      return true;
    }
    size_t j = i;
    while (j < t.size() && !isspace((unsigned char)t[j]) && t[j] != '{' && t[j] != '}' && t[j] != ':' &&
           t[j] != '"' && t[j] != '#')
      ++j;
    tok = t.substr(i, j - i);
    i = j;
    return true;
  }
};

void parse_block(Lexer& lx, PNode& node, bool top) {
  std::string key, tok;
  while (lx.next(key)) {
    if (key == "}") {
      if (top) throw Error(DJINN_E_PARSE, "unbalanced '}'");
      return;
    }
    if (key == "{" || key == ":") throw Error(DJINN_E_PARSE, "expected a field name, got '" + key + "'");
    if (!lx.next(tok)) throw Error(DJINN_E_PARSE, "unexpected end after '" + key + "'");
    if (tok == ":") {
      if (!lx.next(tok)) throw Error(DJINN_E_PARSE, "missing value for '" + key + "'");
    }
    if (tok == "{") {
      PNode child;
      parse_block(lx, child, false);
      node.blocks[key].push_back(std::move(child));
    } else {
      if (tok == "}" || tok == ":") throw Error(DJINN_E_PARSE, "bad value for '" + key + "'");
      if (tok.size() >= 2 && tok[0] == '"') tok = tok.substr(1, tok.size() - 2);
      node.scalars[key].push_back(tok);
    }
  }
  if (!top) throw Error(DJINN_E_PARSE, "missing '}'");
}
}  // namespace

PNode parse_prototxt(const std::string& text) {
  PNode root;
  Lexer lx(text);
  parse_block(lx, root, true);
  return root;
}

// ============================================================================ helpers
// slab-mode B-loader wait policy (GemmGeom::ldwait), DJINN_LDWAIT=0/1/2 (default spin)
static int ldwait_mode() {
  static const int m = [] {
    const char* e = getenv("DJINN_LDWAIT");
    return e ? atoi(e) : 0;
  }();
  return m;
}

// Epilogue warpgroups per tile stream (GemmGeom::epi_wg): 3 for LRN epilogues (latency-bound:
// IMC conv1+norm1 516 -> 440 us on B200), 2 elsewhere, where a 4th TMEM slot of MMA lookahead
// is worth more (IMC conv5 164 -> 132 us).  DJINN_EPI_WG=2/3 forces one for every GEMM.
static int epi_wg_mode(const GemmGeom& g) {
  static const int m = [] {
    const char* e = getenv("DJINN_EPI_WG");
    return e ? atoi(e) : 0;
  }();
  if (m == 2 || m == 3) return m;
  return g.epi_lrn ? 3 : 2;
}

static int tslots_mode() {
  static const int m = [] {
    const char* e = getenv("DJINN_TSLOTS");
    return e ? atoi(e) : 0;
  }();
  return m;
}

// Which conv+LRN(+pool) triples run LRN + pool as a separate kernel (bit k = k-th LRN); the
// others fuse LRN into the conv epilogue.  Measured on B200.
#ifndef LRN_POOL_DEFAULT
#define LRN_POOL_DEFAULT 2
#endif

bool pdl_enabled() {
  static const bool on = [] {
    const char* e = getenv("DJINN_PDL");
    return !(e && e[0] == '0');
  }();
  return on;
}

// DJINN_HOST_PROF=1: host-side microseconds spent enqueueing each op (printed at exit) -- the
// small services are bound by the host's launch path, not the GPU (tools/host_overhead.py).
bool host_prof_on() {
  static const bool on = [] {
    const char* e = getenv("DJINN_HOST_PROF");
    return e && e[0] == '1';
  }();
  return on;
}
namespace {
struct HostProf {
  std::mutex mu;
  std::map<std::string, std::pair<double, long>> acc;
  ~HostProf() {
    for (auto& kv : acc) fprintf(stderr, "[djinn host] %-28s %9.2f us/call over %ld calls\n", kv.first.c_str(),
                                 kv.second.first / kv.second.second, kv.second.second);
  }
};
HostProf& host_prof() {
  static HostProf h;
  return h;
}
}  // namespace
void host_prof_add(const std::string& key, double us) {
  HostProf& h = host_prof();
  std::lock_guard<std::mutex> lk(h.mu);
  auto& a = h.acc[key];
  a.first += us;
  a.second += 1;
}

cudaError_t ensure_max_smem(const void* kernel, int bytes) {
  static std::mutex mu;
  static std::map<std::pair<int, const void*>, int> done;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  std::lock_guard<std::mutex> lk(mu);
  int& have = done[{dev, kernel}];
  if (have >= bytes) return cudaSuccess;
  e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e == cudaSuccess) have = bytes;
  return e;
}

std::atomic<int64_t>& launch_counter() {
  static std::atomic<int64_t> c{0};
  return c;
}

static void ck(cudaError_t e, const char* what) {
  if (e != cudaSuccess) throw Error(DJINN_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    ck(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q), "cuTensorMapEncodeTiled lookup");
    if (q != cudaDriverEntryPointSuccess || !p) throw Error(DJINN_E_CUDA, "cuTensorMapEncodeTiled unavailable");
    fn = (EncodeTiledFn)p;
  }
  return fn;
}

static CUtensorMapSwizzle swizzle_for(int row_bytes) {
  return row_bytes >= 128 ? CU_TENSOR_MAP_SWIZZLE_128B : row_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
}

void encode_tmap(CUtensorMap* m, int dt, const void* base, int rank, const uint64_t* dims, const uint64_t* strides_bytes,
                 const uint32_t* box, int swizzle_bytes, const uint32_t* elem_strides) {
  cuuint64_t d[5], s[4];
  cuuint32_t b[5], es[5];
  for (int i = 0; i < rank; ++i) { d[i] = dims[i]; b[i] = box[i]; es[i] = elem_strides ? elem_strides[i] : 1; }
  for (int i = 0; i + 1 < rank; ++i) s[i] = strides_bytes[i];
  const CUtensorMapDataType ty = dt == DT_F16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16;
  CUresult r = encode_fn()(m, ty, (cuuint32_t)rank, const_cast<void*>(base), d, s, b, es,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, swizzle_for(swizzle_bytes),
                           CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(DJINN_E_CUDA, "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
}

typedef CUresult (*EncodeIm2colFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const int*, const int*, cuuint32_t, cuuint32_t, const cuuint32_t*,
                                   CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion,
                                   CUtensorMapFloatOOBfill);

void encode_im2col(CUtensorMap* m, int dt, const void* base, const uint64_t* dims, const uint64_t* strides_bytes,
                   const int* lower_wh, const int* upper_wh, int channels, int pixels, const uint32_t* elem_strides) {
  static EncodeIm2colFn fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    ck(cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &p, cudaEnableDefault, &q), "cuTensorMapEncodeIm2col lookup");
    if (q != cudaDriverEntryPointSuccess || !p) throw Error(DJINN_E_CUDA, "cuTensorMapEncodeIm2col unavailable");
    fn = (EncodeIm2colFn)p;
  }
  cuuint64_t d[4], s[3];
  cuuint32_t es[4];
  for (int i = 0; i < 4; ++i) { d[i] = dims[i]; es[i] = elem_strides[i]; }
  for (int i = 0; i < 3; ++i) s[i] = strides_bytes[i];
  const CUtensorMapDataType ty = dt == DT_F16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16;
  CUresult r = fn(m, ty, 4, const_cast<void*>(base), d, s, lower_wh, upper_wh, (cuuint32_t)channels, (cuuint32_t)pixels, es,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, swizzle_for(channels * 2), CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(DJINN_E_CUDA, "cuTensorMapEncodeIm2col failed (" + std::to_string((int)r) + ")");
}

static inline int rup(int v, int m) { return (v + m - 1) / m * m; }
static inline size_t rupz(size_t v, size_t m) { return (v + m - 1) / m * m; }

// ============================================================================ plan
static int act_of(const std::string& t) {
  if (t == "ReLU") return ACT_RELU;
  if (t == "Sigmoid") return ACT_SIGMOID;
  if (t == "TanH") return ACT_TANH;
  if (t == "HardTanh") return ACT_HARDTANH;
  return -1;
}

void Net::build(const std::string& desc) {
  PNode root = parse_prototxt(desc);
  name = root.gets("name", "");
  rows_per_query = root.geti("rows_per_query", 1);
  auto it = root.blocks.find("layer");
  if (it == root.blocks.end() || it->second.empty()) throw Error(DJINN_E_PARSE, "no layers");
  for (const PNode& L : it->second) {
    LayerSpec s;
    s.name = L.gets("name", "");
    s.type = L.gets("type", "");
    if (s.type == "Input") {
      const PNode* ip = L.block("input_param");
      const PNode* sh = ip ? ip->block("shape") : nullptr;
      if (!sh) throw Error(DJINN_E_PARSE, "Input without input_param.shape");
      auto d = sh->scalars.find("dim");
      if (d == sh->scalars.end()) throw Error(DJINN_E_PARSE, "Input shape without dims");
      for (auto& v : d->second) s.dims.push_back(atoi(v.c_str()));
    } else if (s.type == "Convolution" || s.type == "LocallyConnected" || s.type == "InnerProduct") {
      const char* pn = s.type == "Convolution" ? "convolution_param"
                       : s.type == "LocallyConnected" ? "local_param" : "inner_product_param";
      const PNode* p = L.block(pn);
      if (!p) throw Error(DJINN_E_PARSE, s.name + ": missing " + pn);
      s.num_output = p->geti("num_output", 0);
      s.kernel = p->geti("kernel_size", 0);
      s.stride = p->geti("stride", 1);
      s.pad = p->geti("pad", 0);
      s.group = p->geti("group", 1);
    } else if (s.type == "Pooling") {
      const PNode* p = L.block("pooling_param");
      if (!p) throw Error(DJINN_E_PARSE, s.name + ": missing pooling_param");
      std::string m = p->gets("pool", "MAX");
      if (m != "MAX" && m != "AVE") throw Error(DJINN_E_UNSUPPORTED, s.name + ": pool " + m);
      s.pool_max = m == "MAX";
      s.kernel = p->geti("kernel_size", 0);
      s.stride = p->geti("stride", 1);
      s.pad = p->geti("pad", 0);
    } else if (s.type == "LRN") {
      const PNode* p = L.block("lrn_param");
      s.lrn_size = p ? p->geti("local_size", 5) : 5;
      s.alpha = p ? (float)p->getf("alpha", 1.0) : 1.f;
      s.beta = p ? (float)p->getf("beta", 0.75) : 0.75f;
      s.lrn_k = p ? (float)p->getf("k", 1.0) : 1.f;
      if (p && p->gets("norm_region", "ACROSS_CHANNELS") != "ACROSS_CHANNELS")
        throw Error(DJINN_E_UNSUPPORTED, s.name + ": only ACROSS_CHANNELS LRN");
    } else if (s.type == "Embedding") {
      const PNode* p = L.block("embedding_param");
      if (!p) throw Error(DJINN_E_PARSE, s.name + ": missing embedding_param");
      s.window = p->geti("window", 1);
      auto v = p->scalars.find("vocab"), d = p->scalars.find("dim");
      if (v == p->scalars.end() || d == p->scalars.end() || v->second.size() != d->second.size())
        throw Error(DJINN_E_PARSE, s.name + ": embedding_param needs one dim per vocab");
      for (auto& x : v->second) s.vocab.push_back(atoi(x.c_str()));
      for (auto& x : d->second) s.edim.push_back(atoi(x.c_str()));
      if (s.window <= 0 || s.vocab.empty() || (int)s.vocab.size() > EMBED_MAX_TABLES)
        throw Error(DJINN_E_SHAPE, s.name + ": window / number of tables");
      for (size_t t = 0; t < s.vocab.size(); ++t)
        if (s.vocab[t] <= 0 || s.edim[t] <= 0) throw Error(DJINN_E_SHAPE, s.name + ": vocab / dim");
    } else if (act_of(s.type) >= 0 || s.type == "Dropout" || s.type == "Softmax") {
    } else {
      throw Error(DJINN_E_UNSUPPORTED, "layer type '" + s.type + "'");
    }
    layers.push_back(s);
  }
  if (layers[0].type != "Input") throw Error(DJINN_E_SHAPE, "first layer must be Input");
  if (layers.back().type != "Softmax") throw Error(DJINN_E_UNSUPPORTED, "last layer must be Softmax");

  const bool f16 = dt != DT_F32;
  // 16-bit activations: channel pitch a multiple of 16 so every conv's K splits into TMA
  // chunks of 16/32/64 channels (one swizzle atom row of 32/64/128 B)
  // Layout of a tensor with C channels, decided by its next channel-consuming layer (skipping
  // activations, LRN, pooling, dropout, which keep the layout): a conv with G groups wants
  // each group at a pitch of 16/32/64 (<= 64 channels) or a multiple of 64, i.e. one TMA row
  // of 32/64/128 B per tap and chunk.  fp32 path: dense channels.
  auto tap_pitch = [](int c) { return c <= 16 ? 16 : c <= 32 ? 32 : rup(c, 64); };
  // A slab convolution (stride 1, every group's channel pitch a multiple of 64) reads its zero
  // padding from memory: its input is stored with a border of `pad` zero pixels (DESIGN.md
  // sec 4).  DJINN_SLAB=0 turns slab mode off (im2col TMA for every conv).
  const char* slab_env = getenv("DJINN_SLAB");
  const bool slab_on = f16 && !(slab_env && slab_env[0] == '0');
  auto slab_border = [&](const LayerSpec& L, const Shape& sh) {
    const int gp = sh.gsz < sh.C ? sh.gpitch : sh.Cp;
    return (slab_on && L.stride == 1 && L.pad > 0 && gp % 64 == 0) ? L.pad : 0;
  };
  int lrn_ordinal = 0;  // LRN layers after a conv seen so far (DJINN_LRN_POOL bit index)
  auto layout_for = [&](size_t from, Shape sh) {
    sh.Cp = sh.C;
    sh.gsz = sh.gpitch = 1 << 30;
    sh.bdr = 0;
    if (!f16) return sh;
    sh.Cp = rup(sh.C, 16);
    bool border_ok = true;  // only a convolution reading the tensor directly may get a border
    for (size_t j = from; j < layers.size(); ++j) {
      const LayerSpec& L = layers[j];
      // a MAX pool the column kernel handles re-lays the channels itself: its producer
      // writes the plain pitch (no grouped-layout padding read back by the pool)
      if (L.type == "Pooling" && L.pool_max && L.kernel <= L.stride + 1) return sh;
      if (L.type == "Pooling" || L.type == "LRN") border_ok = false;
      if (L.type == "Convolution" && L.group > 1 && sh.C % L.group == 0) {
        const int cg = sh.C / L.group;
        if (cg % 16 == 0) {
          sh.gsz = cg;
          sh.gpitch = tap_pitch(cg);
          sh.Cp = L.group * sh.gpitch;
        }
        if (border_ok) sh.bdr = slab_border(L, sh);
        return sh;
      }
      if (L.type == "Convolution" || L.type == "LocallyConnected") {
        sh.Cp = tap_pitch(sh.C);
        if (border_ok && L.type == "Convolution") sh.bdr = slab_border(L, sh);
        return sh;
      }
      if (L.type == "InnerProduct" || L.type == "Softmax") return sh;
    }
    return sh;
  };
  // output buffer of a new tensor: the free ping-pong buffer, or a dedicated one for a bordered
  // tensor (its border is zeroed once at workspace creation and never written)
  auto pick_buf = [&](const Shape& sh, int cur_buf) {
    if (sh.bdr > 0) {
      buf_bytes.push_back(0);
      return (int)buf_bytes.size() - 1;
    }
    return cur_buf == 0 ? 1 : 0;
  };
  const std::vector<int>& d = layers[0].dims;
  Shape cur;
  if (d.size() == 1) { cur.C = d[0]; }
  else if (d.size() == 3) { cur.C = d[0]; cur.H = d[1]; cur.W = d[2]; }
  else throw Error(DJINN_E_SHAPE, "Input must have 1 or 3 dims");
  if (cur.C <= 0 || cur.H <= 0 || cur.W <= 0) throw Error(DJINN_E_SHAPE, "bad Input dims");
  for (size_t i = 2; i < layers.size(); ++i)
    if (layers[i].type == "Embedding") throw Error(DJINN_E_UNSUPPORTED, layers[i].name + ": Embedding must follow Input");
  const bool emb = layers.size() > 1 && layers[1].type == "Embedding";
  Op pk;
  pk.kind = OP_PACK;
  pk.name = "pack";
  pk.in_buf = -1;
  pk.out_buf = 0;
  n_layers = 0;
  n_params = 0;
  size_t arena_off = 0;
  if (emb) {
    // SENNA window lookup: the pack gathers the window vector from the
    // tables in the arena instead of converting one.  Its output is laid out for layer 2.
    const LayerSpec& E = layers[1];
    const int T = (int)E.vocab.size();
    if (d.size() != 1 || cur.C != E.window * T)
      throw Error(DJINN_E_SHAPE, E.name + ": Input must hold window * tables indices per row");
    pk.embed = 1;
    pk.name = E.name;
    cur.Cp = cur.C;
    pk.in = cur;
    pk.eg.window = E.window;
    pk.eg.T = T;
    pk.eg.D = 0;
    int64_t telems = 0;
    for (int t = 0; t < T; ++t) {
      pk.eg.vocab[t] = E.vocab[t];
      pk.eg.dim[t] = E.edim[t];
      pk.eg.toff[t] = telems;
      pk.eg.D += E.edim[t];
      telems += (int64_t)E.vocab[t] * E.edim[t];
    }
    in_elems = cur.C;
    Shape es;
    es.C = E.window * pk.eg.D;
    cur = layout_for(2, es);
    pk.out = cur;
    pk.w_off = arena_off;
    arena_off += ((size_t)telems * (f16 ? 2 : 4) + 255) & ~(size_t)255;
    n_params += telems;
    ++n_layers;
  } else {
    cur = layout_for(1, cur);
    cur.bdr = 0;  // the pack writes no border (a padded first conv then runs on im2col TMA)
    if (cur.gsz < cur.C) throw Error(DJINN_E_UNSUPPORTED, "grouped first convolution on a 16-bit path");
    in_elems = (int64_t)cur.C * cur.H * cur.W;
    pk.in = cur;
    pk.out = cur;
  }
  ops.push_back(pk);
  int curbuf = 0;

  for (size_t i = emb ? 2 : 1; i < layers.size(); ++i) {
    const LayerSpec& L = layers[i];
    if (L.type != "Softmax") ++n_layers;
    if (L.type == "Dropout") continue;
    if (L.type == "Softmax") {
      if (i + 1 != layers.size()) throw Error(DJINN_E_UNSUPPORTED, "Softmax must be the last layer");
      if (ops.back().kind != OP_GEMM || ops.back().out_buf != 2)
        throw Error(DJINN_E_UNSUPPORTED, "Softmax must follow an InnerProduct");
      Op sm;
      sm.kind = OP_SOFTMAX;
      sm.name = L.name;
      sm.in = cur;
      sm.out = cur;
      sm.in_buf = 2;
      ops.push_back(sm);
      continue;
    }
    if (act_of(L.type) >= 0) throw Error(DJINN_E_UNSUPPORTED, L.name + ": activation must follow a weighted layer");
    if (L.type == "LRN") {
      Op o;
      o.kind = OP_LRN;
      o.name = L.name;
      o.in = o.out = cur;
      if (cur.bdr) throw Error(DJINN_E_UNSUPPORTED, L.name + ": internal: LRN over a bordered tensor");
      o.in_buf = curbuf;
      o.out_buf = curbuf = pick_buf(o.out, curbuf);
      o.lrn_size = L.lrn_size;
      o.alpha = L.alpha;
      o.beta = L.beta;
      o.lrn_k = L.lrn_k;
      if (cur.H * cur.W < 1) throw Error(DJINN_E_SHAPE, L.name);
      ops.push_back(o);
      continue;
    }
    if (L.type == "Pooling") {
      if (L.kernel <= 0 || L.stride <= 0 || L.pad < 0 || L.pad >= L.kernel) throw Error(DJINN_E_SHAPE, L.name + ": bad pooling");
      Op o;
      o.kind = OP_POOL;
      o.name = L.name;
      o.in = cur;
      auto pout = [&](int in) {
        int out = (int)((in + 2 * L.pad - L.kernel + L.stride - 1) / L.stride) + 1;  // ceil
        if (in + 2 * L.pad - L.kernel < 0) out = 1;
        if (L.pad > 0 && (out - 1) * L.stride >= in + L.pad) --out;
        return out;
      };
      o.out = Shape();
      o.out.C = cur.C;
      o.out.H = pout(cur.H);
      o.out.W = pout(cur.W);
      o.out = layout_for(i + 1, o.out);
      if (!(f16 && L.pool_max && L.kernel <= L.stride + 1)) o.out = Shape{cur.C, o.out.H, o.out.W, cur.Cp, cur.gsz, cur.gpitch, 1, 0};
      if (cur.bdr) throw Error(DJINN_E_UNSUPPORTED, L.name + ": internal: pooling over a bordered tensor");
      o.kernel = L.kernel;
      o.stride = L.stride;
      o.pad = L.pad;
      o.is_max = L.pool_max;
      o.in_buf = curbuf;
      o.out_buf = curbuf = pick_buf(o.out, curbuf);
      cur = o.out;
      ops.push_back(o);
      continue;
    }
    // ---- weighted layers: Convolution / LocallyConnected / InnerProduct ----
    bool lrn_pool_next = false;
    int act = ACT_NONE;
    size_t j = i + 1;
    if (j < layers.size() && act_of(layers[j].type) >= 0) {
      act = act_of(layers[j].type);
      ++j;
      ++n_layers;
      i = j - 1;
    }
    size_t nx = i + 1;
    while (nx < layers.size() && layers[nx].type == "Dropout") ++nx;
    const bool last = nx < layers.size() && layers[nx].type == "Softmax";
    Op o;
    o.kind = OP_GEMM;
    o.name = L.name;
    o.in = cur;
    o.in_buf = curbuf;
    GemmGeom& g = o.g;
    memset(&g, 0, sizeof(g));
    g.act = act;
    g.stride = 1;
    g.KH = g.KW = 1;
    if (L.num_output <= 0) throw Error(DJINN_E_SHAPE, L.name + ": num_output");
    int64_t wcount = 0, bcount = 0;
    if (L.type == "Convolution" || L.type == "LocallyConnected") {
      if (L.kernel <= 0 || L.stride <= 0 || L.pad < 0) throw Error(DJINN_E_SHAPE, L.name + ": bad kernel/stride/pad");
      const bool lc = L.type == "LocallyConnected";
      const int grp = lc ? 1 : L.group, pad = lc ? 0 : L.pad;
      if (lc && L.pad != 0) throw Error(DJINN_E_UNSUPPORTED, L.name + ": padded LocallyConnected");
      if (grp <= 0 || cur.C % grp || L.num_output % grp) throw Error(DJINN_E_SHAPE, L.name + ": group does not divide channels");
      const int Cg = cur.C / grp, Cog = L.num_output / grp;
      if (f16 && grp > 1 && (Cg % 16 || Cog % 8))
        throw Error(DJINN_E_UNSUPPORTED, L.name + ": grouped conv needs Cin/group % 16 == 0 and Cout/group % 8 == 0 on 16-bit paths");
      const int OH = (cur.H + 2 * pad - L.kernel) / L.stride + 1, OW = (cur.W + 2 * pad - L.kernel) / L.stride + 1;
      if (cur.H + 2 * pad < L.kernel || cur.W + 2 * pad < L.kernel) throw Error(DJINN_E_SHAPE, L.name + ": kernel larger than input");
      o.orig_in = cur;
      o.orig_k = L.kernel;
      g.mode = lc ? GM_LC : GM_CONV;
      g.N = Cog;
      g.Z = lc ? OH * OW : grp;
      g.H = cur.H; g.W = cur.W; g.Cp_in = cur.Cp;
      g.OH = OH; g.OW = OW;
      g.KH = g.KW = L.kernel;
      g.stride = L.stride;
      g.pad = pad;
      if (f16 && grp > 1 && cur.gsz != Cg)
        throw Error(DJINN_E_UNSUPPORTED, L.name + ": input channel layout does not match the grouping");
      const bool grouped_layout = cur.gsz < cur.C;
      g.Cgp = (grp == 1) ? cur.Cp : (grouped_layout ? cur.gpitch : Cg);
      int creal = (grp == 1) ? cur.C : Cg;  // real (unpadded) channels of a tap
      g.cin_goff = grouped_layout ? cur.gpitch : Cg;
      // First layer with few channels on the tensor-core path: repack the input so that K
      // is dense.  Strided kernels: space-to-depth by the stride (k x k / s  ->  ceil(k/s)^2
      // taps over s*s*C channels, stride 1).  Stride 1: unroll kx into channels (k x k -> k x 1).
      if (f16 && !lc && grp == 1 && ops.size() == 1 && cur.C < 16 && pad == 0) {
        Op& pk = ops[0];
        const int f = L.stride, k = L.kernel;
        if (f > 1) {
          const int Hs = (cur.H + f - 1) / f, Ws = (cur.W + f - 1) / f, ks = (k + f - 1) / f;
          if (Hs - ks + 1 >= OH && Ws - ks + 1 >= OW) {
            pk.xform = o.xform = 1;
            pk.xf = o.xf = f;
            pk.out = Shape();
            pk.out.C = f * f * cur.C; pk.out.H = Hs; pk.out.W = Ws; pk.out.Cp = tap_pitch(f * f * cur.C);
            creal = pk.out.C;
            g.H = Hs; g.W = Ws; g.Cp_in = g.Cgp = pk.out.Cp;
            g.KH = g.KW = ks;
            g.stride = 1;
          }
        } else {
          // kx-unroll, and x-block: each packed pixel holds U = k + XB - 1 horizontal taps so
          // one GEMM row computes XB adjacent output pixels (N = XB * out pitch <= 256); the
          // XB shifted copies of the kernel live in B.  Small-N layers then run full-rate MMAs
          // (N <= 64 costs a 52-cycle floor per MMA on B200) and fetch XB x fewer A rows.
          Shape os;
          os.C = L.num_output; os.H = OH; os.W = OW;
          os = layout_for(i + 1, os);
          int XB = 1;
          static const int kx_xb_env = [] {  // DJINN_KX_XB caps the x-block (experiments)
            const char* e = getenv("DJINN_KX_XB");
            return e ? atoi(e) : 0;
          }();
          const int kx_cap = kx_xb_env > 0 ? kx_xb_env : 8;
          if (os.gsz >= os.C && os.Cp <= 64)
            for (int xbc = 8; xbc >= 2; xbc /= 2)
              if (xbc <= kx_cap && (k + xbc - 1) * cur.C <= 64 && xbc * os.Cp <= 256) { XB = xbc; break; }
          const int U = k + XB - 1, OWb = (OW + XB - 1) / XB;
          creal = U * cur.C;  // real channels of a packed tap (the rest of its 64 are zero)
          // window unroll (xform 3): when the whole k x U window fits one 64-channel pixel (DIG
          // conv1: 5 x 12 x 1 = 60), the packed pixel holds all k rows too and the conv becomes a
          // 1 x 1 conv over the OH x OWb grid -- one 128-byte TMA row per GEMM row instead of k
          // 32-byte ones.  Opt-in (DJINN_WINDOW_UNROLL=1): correct, but measured slower on B200
          // (DIG conv1 41.5 -> 40.0 us, its pack 9.9 -> 15.9 us: conv1 is bound by its epilogue).
          static const bool wu_on = [] {
            const char* e = getenv("DJINN_WINDOW_UNROLL");
            return e && e[0] == '1';
          }();
          const bool wu = wu_on && k > 1 && k * U * cur.C <= 64 && k * U * cur.C > 32;
          pk.xform = o.xform = wu ? 3 : 2;
          pk.xf = o.xf = U;
          pk.xs = o.xs = XB;
          pk.out = Shape();
          pk.out.C = (wu ? k : 1) * U * cur.C; pk.out.H = wu ? OH : cur.H; pk.out.W = OWb;
          pk.out.Cp = tap_pitch(pk.out.C);
          if (wu) creal = pk.out.C;
          g.H = pk.out.H; g.W = pk.out.W; g.Cp_in = g.Cgp = pk.out.Cp;
          g.KH = wu ? 1 : k; g.KW = 1;
          if (XB > 1) {
            g.xb = XB;
            g.OWb = OWb;
            g.N = XB * os.Cp;
            g.xstep = 1;  // packed pixel j already starts at input x = j * XB
          }
        }
        if (pk.xform) { o.in = pk.out; }
      }
      g.kxs = 1;
      // Small-N stride-1 conv fed by a pooling layer: the pool writes an x-unrolled layout
      // (pixel x also carries x+1.. up to 64 channels) and the conv x-blocks XB output pixels
      // per GEMM row (N = XB * out pitch): full-rate MMAs and XB x fewer TMA rows.
      if (f16 && !lc && grp == 1 && ops.size() > 1 && ops.back().kind == OP_POOL && o.xform == 0 && L.stride == 1 &&
          pad == 0 && cur.gsz >= cur.C && cur.xu == 1 && cur.Cp <= 32 && 64 % cur.Cp == 0 &&
          ops.back().in.Cp == cur.Cp && ops.back().in.gsz >= cur.C) {
        Shape os;
        os.C = L.num_output; os.H = OH; os.W = OW;
        os = layout_for(i + 1, os);
        const int xu = 64 / cur.Cp;
        int XB = 1;
        for (int xbc = 8; xbc >= 2; xbc /= 2)
          if (xbc * os.Cp <= 256 && os.gsz >= os.C && os.Cp <= 64) { XB = xbc; break; }
        if (XB > 1) {
          Op& pl = ops.back();
          pl.out.P = pl.out.Cp;
          pl.out.xu = xu;
          pl.out.Cp = xu * pl.out.P;
          cur = pl.out;
          o.in = cur;
          const int KWg = (XB + L.kernel - 1 + xu - 1) / xu;
          g.Cp_in = g.Cgp = cur.Cp;
          g.KW = KWg;
          g.kxs = xu;
          g.xb = XB;
          g.OWb = (OW + XB - 1) / XB;
          g.N = XB * os.Cp;
        }
      }
      g.K = g.KH * g.KW * g.Cgp;
      o.out = Shape();
      o.out.C = L.num_output; o.out.H = OH; o.out.W = OW;
      o.out = layout_for(i + 1, o.out);
      g.out_pitch = o.out.Cp;
      g.cout_goff = Cog;
      g.write_cols = grp == 1 ? o.out.Cp : Cog;
      g.bias_zstride = Cog;
      if (g.xb < 1) { g.xb = 1; g.OWb = OW; }
      if (g.xstep < 1) g.xstep = g.xb > 1 ? g.xb : g.stride;
      g.Co = Cog;
      o.ohw = lc ? 1 : OH * g.OWb;
      g.zf = 1;
      g.cw = g.Cgp >= 64 ? 64 : g.Cgp;
      g.lcg = 1;
      g.kwp = g.KW;
      if (f16 && lc && g.Cgp < 64 && 64 % g.Cgp == 0 && g.KW > 1) {
        // LC A rows are images at one location: put lcg horizontally adjacent taps in one
        // 128-byte TMA row; the padded taps carry zero weights.  x-block XB adjacent
        // locations per GEMM (N = XB * out pitch, each location's filter bank on its own
        // columns, shifted by dx*stride taps): the A row is shared by XB locations, so the
        // N = 16 MMA floor and the A traffic are amortised XB times.
        g.lcg = 64 / g.Cgp;
        g.cw = 64;
        const int P = o.out.Cp;
        int XB = 1;
        // cap on the LC x-block: 8 (N = 128, CTA pairs) pays at a full 256-image batch (FACE L4
        // 79 us vs 101 at 4), 4 below one 128-row tile (FACE 2 / 32 images: 214 -> 192 us, 227 ->
        // 199 us per batch on B200).  DJINN_LC_XB overrides.
        static const int lc_xb_env = [] {
          const char* e = getenv("DJINN_LC_XB");
          return e ? atoi(e) : 0;
        }();
        const int lc_xb_cap = lc_xb_env > 0 ? lc_xb_env : (max_rows <= 128 ? 4 : 8);
        if (o.out.gsz >= o.out.C && P <= 64)
          for (int xbc = 8; xbc >= 2; xbc /= 2)
            if (xbc <= lc_xb_cap && xbc * P <= 256 && (xbc - 1) * g.stride + g.KW <= 32) { XB = xbc; break; }
        g.kwp = rup((XB - 1) * g.stride + g.KW, g.lcg);
        g.K = g.KH * g.kwp * g.Cgp;
        if (XB > 1) {
          g.xb = XB;
          g.OWb = (OW + XB - 1) / XB;
          g.Z = OH * g.OWb;
          g.N = XB * P;
          g.bias_zstride = XB * Cog;
        }
      }
      // M tile = a bx x by x bn block of output pixels (x fastest, product 128): the one with
      // the least padding waste for this layer's OW x OH x batch.
      const char* amode = getenv("DJINN_CONV_A");
      g.a_tiled = (!lc && amode && strcmp(amode, "tiled") == 0) ? 1 : 0;
      // Slab convolution: the input's zero padding is stored (border == pad), so the conv is a
      // pad-0 conv over the stored Hv x Wv grid and every tap of a 128-row tile is a row shift
      // of one contiguous run of input pixels (one TMA slab per tile instead of KH*KW im2col
      // boxes: the operand stream through L2 drops ~KH*KW-fold).  Rows are virtual pixels of
      // the stored grid; the ones outside OH x OWb are computed and discarded.
      if (slab_on && !lc && !g.a_tiled && g.stride == 1 && g.kxs == 1 && g.Cgp % 64 == 0 && o.in.bdr == g.pad) {
        const int Hv = o.in.H + 2 * o.in.bdr, Wv = o.in.W + 2 * o.in.bdr;
        const int R = 128 + (g.KH - 1) * Wv + (g.KW - 1);
        if (R <= 512) {
          g.slab = 1;
          g.Hv = Hv; g.Wv = Wv;
          g.H = Hv; g.W = Wv; g.pad = 0;  // (also valid for an im2col fallback over the stored grid)
          g.slab_parts = (R + 255) / 256;
          g.slab_rows = rup((R + g.slab_parts - 1) / g.slab_parts, 8);
          o.ohw = Hv * Wv;
          // taps of 48 real channels in a 64-channel chunk (IMC conv1 after space-to-depth,
          // conv2's groups): the 4th 16-channel K sub-step multiplies zero weights, so the
          // kernel variant with 3 MMAs per K block skips it (DJINN_KSKIP=0: off)
          const char* ks = getenv("DJINN_KSKIP");
          g.kv16 = (g.Cgp == 64 && creal > 32 && creal <= 48 && g.kxs == 1 && !(ks && ks[0] == '0')) ? 3 : 4;
        }
      }
      if (!g.slab && o.in.bdr > 0) {  // a bordered input read by im2col: pad-0 conv over the stored grid
        if (o.in.bdr > g.pad) throw Error(DJINN_E_SHAPE, L.name + ": internal: input border exceeds the padding");
        g.H = o.in.H + 2 * o.in.bdr; g.W = o.in.W + 2 * o.in.bdr; g.pad -= o.in.bdr;
      }
      if (!lc) {
        double best = 1e30;
        for (int bx = 1; bx <= 128; bx *= 2)
          for (int by = 1; bx * by <= 128; by *= 2) {
            const int bn = 128 / (bx * by);
            if (bx * g.stride > 256 || by * g.stride > 256) continue;
            // padded pixels x (1 + 4/bx): a TMA box streams runs of bx contiguous pixels, short
            // runs cost extra per row (B200 measurement)
            const double cost = (double)rup(OW, bx) * rup(OH, by) * rup((int)max_rows, bn) * (1.0 + 4.0 / bx);
            if (cost < best - 1e-9 || (cost < best + 1e-9 && bx > g.bx)) { best = cost; g.bx = bx; g.by = by; g.bn = bn; }
          }
      }
      if (f16 && (g.Cgp % 16 || (g.Cgp > 64 && g.Cgp % 64) || (g.Cgp < 64 && g.Cgp != 16 && g.Cgp != 32)))
        throw Error(DJINN_E_SHAPE, L.name + ": internal: input channel pitch not TMA-chunkable");
      // Caffe LRN right after (the activation of) this conv: fuse it into the epilogue when one
      // tile holds every channel of a pixel (all groups side by side in TMEM).
      const bool lrn_next = f16 && !lc && i + 1 < layers.size() && layers[i + 1].type == "LRN" &&
                            layers[i + 1].lrn_size == 5;
      // LRN + MAX pool (kernel 3, stride 2, pad 0) as one separate kernel instead of the epilogue
      // fusion: bit k of DJINN_LRN_POOL (default LRN_POOL_DEFAULT) selects it for the k-th LRN.
      const bool pool_next = i + 2 < layers.size() && layers[i + 2].type == "Pooling" && layers[i + 2].pool_max &&
                             layers[i + 2].kernel == 3 && layers[i + 2].stride == 2 && layers[i + 2].pad == 0;
      const int lrn_mask = getenv("DJINN_LRN_POOL") ? atoi(getenv("DJINN_LRN_POOL")) : LRN_POOL_DEFAULT;
      const bool lrn_sep = lrn_next && pool_next && L.num_output % 16 == 0 && ((lrn_mask >> lrn_ordinal) & 1);
      if (lrn_next) ++lrn_ordinal;
      if (lrn_sep) {
        // The conv's epilogue stays bias + ReLU and stores fp16 (only LRN reads it); LRN + the
        // MAX pooling after it run as one kernel (k_misc.cu lrn_pool_kernel).
        lrn_pool_next = true;
        g.out_half = 1;
        o.out.Cp = rup(o.out.C, 16);
        o.out.gsz = o.out.gpitch = 1 << 30;
        g.out_pitch = o.out.Cp;
        g.write_cols = grp == 1 ? o.out.Cp : Cog;
      } else if (lrn_next) {
        const int bn = tc_pick_bn(g);
        if (Cog <= 256 && (grp == 1 || bn == Cog) && grp * bn <= 256) {
          const LayerSpec& R = layers[i + 1];
          g.epi_lrn = 1;
          g.zf = grp;
          g.lrn_size = R.lrn_size;
          g.lrn_alpha_over_n = R.alpha / R.lrn_size;
          g.lrn_beta = R.beta;
          g.lrn_k = R.lrn_k;
          g.write_cols = o.out.Cp;
          o.name += "+" + R.name;
          ++i;
          ++n_layers;
        }
      }
      wcount = lc ? (int64_t)OH * OW * L.num_output * cur.C * L.kernel * L.kernel
                  : (int64_t)L.num_output * Cg * L.kernel * L.kernel;
      bcount = lc ? (int64_t)L.num_output * OH * OW : L.num_output;
    } else {
      g.mode = GM_DENSE;
      g.N = L.num_output;
      g.Z = 1;
      g.K = (int)cur.per_row();
      g.a_pitch = g.K;
      g.zf = 1;
      g.cw = 64;
      o.out = Shape();
      o.out.C = L.num_output; o.out.H = 1; o.out.W = 1;
      o.out = layout_for(i + 1, o.out);
      if (last) o.out.Cp = rup(L.num_output, 8);
      g.out_pitch = o.out.Cp;
      g.write_cols = o.out.Cp;
      g.bias_zstride = 0;
      wcount = (int64_t)L.num_output * cur.C * cur.H * cur.W;
      bcount = L.num_output;
    }
    if (last && g.mode != GM_DENSE) throw Error(DJINN_E_UNSUPPORTED, "the layer before Softmax must be InnerProduct");
    g.out_pitch = o.out.Cp;
    g.out_gsz = o.out.gsz;
    g.out_gpitch = o.out.gpitch;
    if (o.out.gsz < o.out.C) {  // grouped output layout: write real channels, pads zeroed per group
      if (o.out.gsz % 16 || (g.mode == GM_CONV && g.Z > 1 && !g.epi_lrn && g.N % 16))
        throw Error(DJINN_E_UNSUPPORTED, L.name + ": output channel groups must be multiples of 16");
      g.write_cols = (g.mode == GM_CONV && g.Z > 1 && !g.epi_lrn) ? g.N : o.out.C;
    }
    g.Kpad = f16 ? rup(g.K, 64) : g.K;
    g.out_f32 = last ? 1 : 0;
    if (o.out.bdr && g.mode != GM_CONV) throw Error(DJINN_E_UNSUPPORTED, L.name + ": internal: bordered output");
    g.obd = o.out.bdr;
    o.out_buf = last ? 2 : pick_buf(o.out, curbuf);
    if (!last) curbuf = o.out_buf;
    if (last) out_pitch = o.out.Cp;
    o.bn = f16 ? 0 : 64;
    // arena placement
    const size_t wbytes = (size_t)g.Z * g.N * g.Kpad * (f16 ? 2 : 4);
    const size_t bfloats = g.mode == GM_DENSE ? (size_t)g.N : (size_t)g.Z * g.bias_zstride;
    arena_off = rupz(arena_off, 1024);
    o.w_off = arena_off;
    arena_off += wbytes;
    arena_off = rupz(arena_off, 256);
    o.b_off = arena_off;
    arena_off += bfloats * 4;
    n_params += wcount + bcount;
    cur = o.out;
    ops.push_back(o);
    if (lrn_pool_next) {
      const LayerSpec& R = layers[i + 1];
      Op lp;
      lp.kind = OP_LRNPOOL;
      lp.name = R.name;
      lp.in = cur;
      lp.lrn_size = R.lrn_size;
      lp.alpha = R.alpha;
      lp.beta = R.beta;
      lp.lrn_k = R.lrn_k;
      lp.kernel = 1; lp.stride = 1; lp.pad = 0; lp.is_max = 1;
      Shape os = cur;
      ++i;
      ++n_layers;
      if (i + 1 < layers.size() && layers[i + 1].type == "Pooling" && layers[i + 1].pool_max) {
        const LayerSpec& Pl = layers[i + 1];
        auto pout = [&](int in) {
          int out = (int)((in + 2 * Pl.pad - Pl.kernel + Pl.stride - 1) / Pl.stride) + 1;
          if (in + 2 * Pl.pad - Pl.kernel < 0) out = 1;
          if (Pl.pad > 0 && (out - 1) * Pl.stride >= in + Pl.pad) --out;
          return out;
        };
        os.H = pout(cur.H);
        os.W = pout(cur.W);
        lp.kernel = Pl.kernel; lp.stride = Pl.stride; lp.pad = Pl.pad;
        lp.name += "+" + Pl.name;
        ++i;
        ++n_layers;
      }
      os = layout_for(i + 1, os);
      lp.in_buf = o.out_buf;
      lp.out = os;
      lp.out_buf = curbuf = pick_buf(os, o.out_buf);
      cur = os;
      ops.push_back(lp);
    }
  }
  // First-layer kernel (k_stem.cu) for a space-to-depth first conv whose output is a plain NHWC
  // tensor: resident filter bank, TMA-store epilogue, slab of the packed tensor by TMA (default,
  // stem = 2).  DJINN_STEM=1: the kernel gathers the fp32 images itself and the pack op is not
  // launched -- bitwise equal, but measured slower on B200 (its fp32 gather is the bottleneck,
  // DESIGN.md sec 5).  DJINN_STEM=0: the generic slab GEMM.
  {
    const char* se = getenv("DJINN_STEM");
    const int smode = se ? atoi(se) : 3;
    if (f16 && smode > 0 && ops.size() > 1 && ops[0].kind == OP_PACK && ops[0].xform == 1 &&
        ops[1].kind == OP_GEMM && ops[1].xform == 1) {
      Op& c = ops[1];
      const GemmGeom& g = c.g;
      // its output is the whole virtual Hs x Ws grid (one TMA store per 32 pixels); the consumer
      // must be a pool that reads the stored grid (the MAX pool with a layout change)
      const bool pool_next = ops.size() > 2 && ops[2].kind == OP_POOL && ops[2].is_max && ops[2].kernel <= ops[2].stride + 1 &&
                             ops[2].in_buf == c.out_buf;
      if (pool_next && g.mode == GM_CONV && g.Z == 1 && g.zf == 1 && g.stride == 1 && g.pad == 0 && g.xb <= 1 &&
          !g.out_f32 && !g.out_half && c.out.gsz >= c.out.C && c.out.bdr == 0 && c.out.Cp == g.N && g.KH == g.KW &&
          g.H - g.OH >= 0 && g.W - g.OW >= 0 && stem_supported(g.N, c.xf, c.orig_in.C, g.KH, c.out.Cp)) {
        c.stem = smode == 1 ? 1 : 2;
        ops[0].fused = smode == 1 ? 1 : 0;
        c.out.hx = ops[2].in.hx = g.H - g.OH;
        c.out.wx = ops[2].in.wx = g.W - g.OW;
        // DJINN_STEM=3 (default): the MAX pool runs in the first-layer kernel's epilogue (its
        // output goes straight to the pool's output tensor; the conv output never reaches HBM)
        Op& pl = ops[2];
        if (smode == 3 && g.epi_lrn && stem_pool_supported(g.N, g.W, g.OH, g.OW, pl.kernel, pl.stride, pl.pad, pl.out.Cp,
                                                           pl.out.gsz, pl.out.gpitch, pl.out.xu) &&
            pl.out.H == (g.OH - 3) / 2 + 1 && pl.out.W == (g.OW - 3) / 2 + 1 && pl.out.hx == 0 && pl.out.wx == 0) {
          c.stem_pool = 1;
          pl.fused = 1;
          c.name += "+" + pl.name;
          c.out = pl.out;
          c.out_buf = pl.out_buf;
        }
      }
    }
  }
  // Two-layer window MLP nets (pack -> dense -> dense -> softmax: POS / CHK / NER) run as one
  // kernel (k_mlp.cu).  DJINN_MLP=0 keeps the four separate kernels.
  {
    const char* me = getenv("DJINN_MLP");
    if (f16 && !(me && me[0] == '0') && ops.size() == 4 && ops[0].kind == OP_PACK && !ops[0].embed && !ops[0].xform &&
        ops[1].kind == OP_GEMM && ops[1].g.mode == GM_DENSE && ops[2].kind == OP_GEMM && ops[2].g.mode == GM_DENSE &&
        ops[2].g.out_f32 && ops[3].kind == OP_SOFTMAX) {
      MlpGeom m{};
      m.K0 = ops[0].in.C * ops[0].in.H * ops[0].in.W;
      m.K0p = ops[1].g.Kpad;
      m.N1 = ops[1].g.N;
      m.N1p = rup(m.N1, 16);
      m.N1c = m.N1p;
      m.K1p = ops[2].g.Kpad;
      m.N2 = ops[2].g.N;
      m.N2p = rup(m.N2, 16);
      m.act1 = ops[1].g.act;
      if (ops[0].out.Cp == ops[1].g.K && m.K0 <= ops[0].out.Cp && ops[1].out.Cp <= m.K1p && mlp2_supported(m)) {
        ops[1].mlp = 1;
        ops[1].mg = m;
        ops[0].fused = ops[2].fused = ops[3].fused = 1;
      }
    }
    // The same kernel as the tail of a larger net (DIG's ip1 + ReLU + ip2 + softmax): layer 1
    // reads the 16-bit activations of the layer before it by TMA (a_tma).  (After the SENNA
    // token-id lookup it measured mixed -- NER 4096 windows 26.9 -> 24.6 us, POS 65536 155 -> 159
    // us: the TMA-fed kernel keeps 128 rows per CTA -- so the lookup nets keep 3 kernels.)
    const size_t L = ops.size();
    if (f16 && !(me && me[0] == '0') && L >= 4 && !ops[L - 3].mlp && ops[L - 3].kind == OP_GEMM &&
        ops[L - 3].g.mode == GM_DENSE && ops[L - 3].in_buf >= 0 && !ops[L - 3].g.out_f32 && !ops[L - 3].g.out_half &&
        ops[L - 3].g.Z == 1 && ops[L - 2].kind == OP_GEMM && ops[L - 2].g.mode == GM_DENSE && ops[L - 2].g.out_f32 &&
        ops[L - 2].g.Z == 1 && ops[L - 1].kind == OP_SOFTMAX && ops[L - 4].kind != OP_PACK) {
      const Op& a = ops[L - 3];
      const Op& b = ops[L - 2];
      MlpGeom m{};
      m.a_tma = 1;
      m.K0 = a.g.Kpad;
      m.K0p = a.g.Kpad;
      m.N1 = a.g.N;
      m.N1p = rup(m.N1, 16);
      m.K1p = b.g.Kpad;
      m.N2 = b.g.N;
      m.N2p = rup(m.N2, 16);
      m.N1c = m.N1p + m.N2p <= 512 ? m.N1p : 0;
      m.act1 = a.g.act;
      // split layer 1's columns over a cluster (128 per CTA) when it is wide: each CTA then streams
      // 1 / S of W1 (DIG: 512 -> 4 x 128).  DJINN_MLP_SPLIT overrides (1: no split).
      const char* ms = getenv("DJINN_MLP_SPLIT");
      m.nsplit = ms ? atoi(ms) : (m.N1p >= 256 && m.N1p % 128 == 0 ? m.N1p / 128 : 1);
      if (m.nsplit > 1 && !mlp2_supported(m)) m.nsplit = 1;
      if (a.g.a_pitch <= a.g.Kpad && a.g.a_pitch % 8 == 0 && a.out.Cp <= m.K1p && m.N1p <= 512 &&
          mlp2_supported(m)) {
        ops[L - 3].mlp = 1;
        ops[L - 3].mg = m;
        ops[L - 2].fused = ops[L - 1].fused = 1;
      }
    }
  }
  // A wide last dense layer + softmax (ASR's 8000 senones) as one cluster kernel (k_smx.cu) for
  // forwards of >= smx_min_rows rows: opt-in (DJINN_SMX=1), because on B200 it is slower than
  // the persistent tc GEMM + softmax kernel (ASR 8192 frames: 449 vs 311 us).
  // DJINN_SMX_MIN_ROWS overrides the row threshold.
  {
    const char* se = getenv("DJINN_SMX");
    const size_t L = ops.size();
    int cl = 0, ncw = 0;
    if (f16 && se && se[0] == '1' && L >= 2 && ops[L - 1].kind == OP_SOFTMAX && ops[L - 2].kind == OP_GEMM &&
        !ops[L - 2].mlp && ops[L - 2].g.mode == GM_DENSE && ops[L - 2].g.out_f32 && ops[L - 2].g.act == ACT_NONE &&
        ops[L - 2].g.Z == 1 && smx_plan(ops[L - 2].g.N, ops[L - 2].g.Kpad, &cl, &ncw)) {
      Op& o = ops[L - 2];
      o.smx = 1;
      o.smx_cl = cl;
      o.smx_ncw = ncw;
      const char* mr = getenv("DJINN_SMX_MIN_ROWS");
      o.smx_min_rows = mr ? atoll(mr) : 1024;
    }
  }
  out_elems = cur.C;
  arena_bytes = rupz(arena_off, 1024);
  // Centered sigmoid storage on 16-bit paths: a sigmoid layer feeding a dense layer stores
  // sigma(x) - 1/2 and the consumer's bias absorbs 1/2 * rowsum(W) (exact reparametrisation).
  if (f16)
    for (size_t i = 0; i + 1 < ops.size(); ++i)
      if (ops[i].kind == OP_GEMM && ops[i].g.act == ACT_SIGMOID && ops[i + 1].kind == OP_GEMM &&
          ops[i + 1].g.mode == GM_DENSE) {
        ops[i].g.act = ACT_SIGMOID_C;
        ops[i + 1].fold_half = true;
      }
  // algorithmic work per op (real, unpadded dimensions)
  const double es = f16 ? 2.0 : 4.0;
  for (Op& o : ops) {
    const Shape& oin = (o.kind == OP_GEMM && o.g.mode != GM_DENSE) ? o.orig_in : o.in;
    const double in_e = (double)oin.C * oin.H * oin.W, out_e = (double)o.out.C * o.out.H * o.out.W;
    switch (o.kind) {
      case OP_PACK:
        // lookup: indices in, window vector out, one table row read per (word, table)
        o.bytes_row = o.fused ? 0.0 : o.embed ? in_e * 4 + 2.0 * out_e * es : in_e * 4 + in_e * es;
        break;
      case OP_GEMM: {
        const GemmGeom& g = o.g;
        double kreal;
        if (g.mode == GM_DENSE) kreal = in_e;
        else if (g.mode == GM_LC) kreal = (double)o.orig_k * o.orig_k * oin.C;
        else kreal = (double)o.orig_k * o.orig_k * (oin.C / (g.zf > 1 ? g.zf : g.Z));
        // a fused pool (stem_pool) makes o.out the pooled tensor: the GEMM's work is the conv's
        const double gemm_e = o.stem_pool ? (double)g.N * g.OH * g.OW : out_e;
        o.flops_row = 2.0 * gemm_e * kreal;
        o.bytes_row = in_e * (o.stem == 1 ? 4.0 : es) + out_e * (g.out_f32 ? 4.0 : es);  // stem 1 reads the fp32 images
        const double nb = g.mode == GM_DENSE ? g.N : (double)g.Z * g.bias_zstride;
        o.weight_bytes = (g.mode == GM_LC ? (double)g.Z * g.N * kreal
                                          : (g.mode == GM_CONV ? (double)o.out.C * kreal : (double)g.N * kreal)) * es +
                         nb * 4;
        break;
      }
      case OP_LRN: o.bytes_row = 2 * in_e * es; break;
      case OP_LRNPOOL: o.bytes_row = in_e * es + out_e * es; break;
      case OP_POOL: o.bytes_row = o.fused ? 0.0 : in_e * es + out_e * es; break;
      case OP_SOFTMAX:  // in the cluster kernel (smx): no traffic of its own
        o.bytes_row = (&o != &ops[0] && (&o - 1)->smx) ? 0.0 : 2.0 * in_e * 4;
        break;
    }
  }
  for (const Op& o : ops) {
    if (o.kind == OP_SOFTMAX || o.out_buf < 0) continue;
    const size_t es = o.out_buf == 2 ? 4 : (f16 ? 2 : 4);
    buf_bytes[o.out_buf] = std::max(buf_bytes[o.out_buf], (size_t)max_rows * o.out.per_row() * es);
  }
}

// ============================================================================ weights
// Tile width / CTA pairing per GEMM, and slab-mode shared memory (falls back to im2col TMA
// over the stored grid when the slab does not fit).
void Net::choose_tiles() {
  if (dt == DT_F32) return;
  for (Op& o : ops) {
    if (o.kind != OP_GEMM) continue;
    GemmGeom g = o.g;
    g.M = (int)(max_rows * o.ohw);
    o.bn = tc_pick_bn(g);
    o.g.cg = tc_pick_cg(g, o.bn);
    {
      // Dense GEMMs that fill less than one wave of 148 SMs with their default tile get
      // 64-wide tiles if that makes at most two waves (measured on B200: POS l1 16.4 -> 12.4 us,
      // DIG ip1 21.2 -> 16.3, IMC fc8 34.8 -> 22.6, FACE F7 49.3 -> 34.9; IMC fc6/fc7 would
      // become 512 tiles and run 2x slower, so they keep 256-wide pairs; ASR already fills the GPU).
      // DJINN_DENSE_BN=0 disables the rule, =64/128 forces that cap on every dense GEMM.
      static const int env_cap = [] {
        const char* e = getenv("DJINN_DENSE_BN");
        return e ? atoi(e) : -1;
      }();
      int cap = env_cap;
      if (cap < 0) {
        const int64_t mt = (g.M + 128LL * o.g.cg - 1) / (128LL * o.g.cg), nt = (g.N + o.bn - 1) / o.bn;
        const int64_t t64 = ((g.M + 127) / 128) * ((g.N + 63) / 64) * g.Z;  // tiles after the cap (cg = 1)
        cap = (mt * nt * g.Z < 148 && t64 <= 2 * 148) ? 64 : 0;
      }
      // A long-K dense GEMM of at most two row tiles under one wave keeps 128-wide single-CTA tiles
      // and is split over K instead (below): half the K chain per CTA at twice the per-MMA width
      // (N = 64 MMAs run at the 52-cycle floor).  Measured on B200: IMC 16 images 160.8 -> 157.8 us
      // per batch, FACE 2 images 191.0 -> 180.1, FACE F7 at 256 35.2 -> 33.8; IMC fc8 at 1024
      // images was slower (27.1 -> 35.7 us incl. the reduction), hence the row limit.
      // DJINN_SPLITK_WIDE=0 disables.
      static const bool wide_sk = [] {
        const char* e = getenv("DJINN_SPLITK_WIDE");
        return !(e && e[0] == '0');
      }();
      const int64_t t128 = ((g.M + 127) / 128) * ((g.N + 127) / 128) * g.Z;
      const bool wide = env_cap < 0 && wide_sk && g.mode == GM_DENSE && cap == 64 && g.Kpad / 64 >= 32 && t128 <= 74 &&
                        (g.M + 127) / 128 <= 2 && !o.mlp && !o.smx;
      if (wide) {
        o.bn = 128;
        o.g.cg = 1;
      } else if (g.mode == GM_DENSE && cap >= 16 && o.bn > cap) {
        o.bn = cap;
        o.g.cg = tc_pick_cg(g, o.bn);
      }
      // Wave quantisation of large dense GEMMs on CTA pairs: a tile's MMA time grows with its
      // width, so pick the width (192 or 256) with the fewer waves x width over the 74 pairs.
      // Measured on B200 (DJINN_DENSE_BN=192 for all): ASR a1-a5 (8192 x 2048 x 2048, 4 waves
      // of 256 vs 5 of 192) 57.3 -> 54.7 us each; ASR out (N = 8000) and IMC fc6 / fc7 slower at
      // 192, as the model predicts.
      if (env_cap < 0 && g.mode == GM_DENSE && o.g.cg == 2 && o.bn == 256) {
        const int64_t pairs = tc_num_sms() / 2, mt = (g.M + 255) / 256;
        auto cost = [&](int bn) { return ((mt * ((g.N + bn - 1) / bn) + pairs - 1) / pairs) * bn; };
        if (cost(192) < cost(256)) o.bn = 192;
      }
    }
    // Split-K for dense GEMMs that cannot fill the GPU with output tiles but have a long K (FACE
    // F8: 4 tiles of 64 K blocks; the FC layers at the Table 3 batches, e.g. IMC fc6 at 16
    // images): K is cut into S ranges so S x tiles CTAs stream it; the fp32 partials are added
    // in split order by a reduction that applies bias + activation.  DJINN_SPLITK=0 disables.
    {
      static const bool sk_on = [] {
        const char* e = getenv("DJINN_SPLITK");
        return !(e && e[0] == '0');
      }();
      const int nkb = g.Kpad / 64;
      const int64_t tiles = ((g.M + 127) / 128) * ((g.N + o.bn - 1) / o.bn);
      o.ksplit = 1;
      if (sk_on && !o.mlp && !o.smx && g.mode == GM_DENSE && o.g.cg == 1 && nkb >= 32 && tiles <= 74) {
        const int S = (int)std::min<int64_t>(nkb / 8, 148 / tiles);
        if (S >= 2) {
          o.ksplit = S;
          o.kpb = (nkb + S - 1) / S;
          o.npart = rup(g.N, 8);
        }
      }
    }
    if (o.stem) o.g.cg = 2;  // the stem kernel loads B as two boxes of bn / 2 rows per K block
    if (o.g.slab && !tc_slab_config(o.g, o.bn)) {
      o.g.slab = 0;
      o.ohw = o.g.OH * o.g.OWb;
    }
  }
}

void Net::load_weights(const float* w, size_t n, int mem) {
  const bool f16 = dt != DT_F32;
  if (n != (size_t)n_params)
    throw Error(DJINN_E_WEIGHTS, "weight blob has " + std::to_string(n) + " floats, description needs " +
                                     std::to_string(n_params));
  std::vector<float> hostcopy;
  if (mem == DJINN_MEM_DEVICE) {
    hostcopy.resize(n);
    ck(cudaMemcpy(hostcopy.data(), w, n * 4, cudaMemcpyDeviceToHost), "weights D2H");
    w = hostcopy.data();
  }
  std::vector<uint8_t> host(arena_bytes, 0);
  size_t off = 0;  // floats into the canonical blob
  for (Op& o : ops) {
    if (o.kind == OP_PACK && o.embed) {  // lookup tables, converted to the path's type
      int64_t telems = 0;
      for (int t = 0; t < o.eg.T; ++t) telems += (int64_t)o.eg.vocab[t] * o.eg.dim[t];
      uint8_t* dst = host.data() + o.w_off;
      for (int64_t e = 0; e < telems; ++e) {
        const float v = w[off + e];
        if (!f16) { reinterpret_cast<float*>(dst)[e] = v; continue; }
        uint16_t bits;
        if (dt == DT_BF16) { __nv_bfloat16 h = __float2bfloat16_rn(v); memcpy(&bits, &h, 2); }
        else { __half h = __float2half_rn(v); memcpy(&bits, &h, 2); }
        reinterpret_cast<uint16_t*>(dst)[e] = bits;
      }
      off += telems;
      continue;
    }
    if (o.kind != OP_GEMM) continue;
    const GemmGeom& g = o.g;
    uint8_t* wdst = host.data() + o.w_off;
    float* bdst = reinterpret_cast<float*>(host.data() + o.b_off);
    std::vector<double> rowsum(o.fold_half ? g.N : 0, 0.0);
    auto put = [&](int64_t z, int64_t nn, int64_t k, float v) {
      const int64_t idx = (z * g.N + nn) * g.Kpad + k;
      if (!f16) { reinterpret_cast<float*>(wdst)[idx] = v; return; }
      uint16_t bits;
      float r;
      if (dt == DT_BF16) { __nv_bfloat16 h = __float2bfloat16_rn(v); memcpy(&bits, &h, 2); r = __bfloat162float(h); }
      else { __half h = __float2half_rn(v); memcpy(&bits, &h, 2); r = __half2float(h); }
      if (o.fold_half) rowsum[nn] += r;
      reinterpret_cast<uint16_t*>(wdst)[idx] = bits;
    };
    const int C = o.in.C, H = o.in.H, W = o.in.W, Cp = o.in.Cp;
    if (g.mode == GM_CONV) {
      const int grp = g.Z, C0 = o.orig_in.C, Cg = C0 / grp, k = o.orig_k;
      for (int co = 0; co < o.out.C; ++co)
        for (int c = 0; c < Cg; ++c)
          for (int ky = 0; ky < k; ++ky)
            for (int kx = 0; kx < k; ++kx) {
              int64_t kk;
              if (o.xform == 1) {  // space-to-depth: tap (ky/f, kx/f), channel ((ky%f)*f + kx%f)*C0 + c
                const int f = o.xf;
                // the first-layer kernel keeps B dense in K (tap * f*f*C0 + channel, no per-tap pad)
                const int64_t tstride = (o.stem && stem_dense_b()) ? (int64_t)f * f * C0 : g.Cgp;
                kk = (int64_t)((ky / f) * g.KW + kx / f) * tstride + ((ky % f) * f + kx % f) * C0 + c;
              } else if (o.in.xu > 1) {  // x-unrolled input + x-block: tap group j, slot i
                for (int dx = 0; dx < g.xb; ++dx) {
                  const int e = dx + kx, jj = e / g.kxs, ii = e % g.kxs;
                  const int64_t ki = (int64_t)(ky * g.KW + jj) * g.Cgp + ii * o.in.P + c;
                  if (dx > 0) put(0, dx * g.out_pitch + co, ki, w[off]);
                  else kk = ki;
                }
              } else if (o.xform == 3) {  // window unroll: one tap, channel (ky*U + kx)*C0 + c (+ x-block copies)
                const int U = o.xf;
                for (int dx = 1; dx < g.xb; ++dx)
                  put(0, dx * g.out_pitch + co, (int64_t)(ky * U + dx + kx) * C0 + c, w[off]);
                kk = (int64_t)(ky * U + kx) * C0 + c;
              } else if (o.xform == 2) {  // kx-unroll: tap ky, channel kx*C0 + c (+ x-block copies)
                for (int dx = 1; dx < g.xb; ++dx)
                  put(0, dx * g.out_pitch + co, (int64_t)ky * g.Cgp + (dx + kx) * C0 + c, w[off]);
                kk = (int64_t)ky * g.Cgp + kx * C0 + c;
              } else {
                kk = (int64_t)(ky * k + kx) * g.Cgp + c;
              }
              if (g.xb > 1) put(0, co, kk, w[off++]);
              else put(co / g.N, co % g.N, kk, w[off++]);
            }
      for (int co = 0; co < o.out.C; ++co) bdst[co] = w[off++];
    } else if (g.mode == GM_LC) {
      const int k = g.KH;
      const int OH = g.OH, OW = g.OW, Co = g.Co, XB = g.xb;
      for (int loc = 0; loc < OH * OW; ++loc) {
        const int oy = loc / OW, ox = loc % OW;
        const int z = XB > 1 ? oy * g.OWb + ox / XB : loc, dx = XB > 1 ? ox % XB : 0;
        for (int co = 0; co < Co; ++co)
          for (int c = 0; c < C; ++c)
            for (int ky = 0; ky < k; ++ky)
              for (int kx = 0; kx < k; ++kx)
                put(z, dx * (XB > 1 ? g.out_pitch : 0) + co, (int64_t)(ky * g.kwp + dx * g.stride + kx) * g.Cgp + c,
                    w[off++]);
      }
      // bias [Co][OH][OW] -> [z][dx][co] (one row of Co per location, locations padded to XB)
      for (int co = 0; co < Co; ++co)
        for (int loc = 0; loc < OH * OW; ++loc) {
          const int oy = loc / OW, ox = loc % OW;
          const int64_t slot = XB > 1 ? (int64_t)(oy * g.OWb + ox / XB) * XB + ox % XB : loc;
          bdst[slot * Co + co] = w[off++];
        }
    } else {
      // Caffe flattens (c, h, w); our rows are (h, w, c) with channel pitch Cp.
      for (int nn = 0; nn < g.N; ++nn)
        for (int c = 0; c < C; ++c)
          for (int h = 0; h < H; ++h)
            for (int x = 0; x < W; ++x)
              put(0, nn, ((int64_t)h * W + x) * Cp + o.in.pos(c), w[off++]);
      for (int nn = 0; nn < g.N; ++nn) bdst[nn] = (float)(w[off++] + (o.fold_half ? 0.5 * rowsum[nn] : 0.0));
    }
  }
  if (off != n) throw Error(DJINN_E_WEIGHTS, "internal: blob walk mismatch");
  ck(cudaMemcpy(arena, host.data(), arena_bytes, cudaMemcpyHostToDevice), "weights H2D");
}

// ============================================================================ workspace
Workspace::~Workspace() {
  for (void* p : buf) if (p) cudaFree(p);
  if (in_stage) cudaFree(in_stage);
  if (in_stage16) cudaFree(in_stage16);
  if (in_wide) cudaFree(in_wide);
  if (part) cudaFree(part);
  if (out_stage) cudaFree(out_stage);
  for (int s = 0; s < 2; ++s)
    for (cudaEvent_t e : {in_ready[s], in_free[s], out_ready[s], out_free[s]})
      if (e) cudaEventDestroy(e);
  if (cin) cudaStreamDestroy(cin);
  if (cout) cudaStreamDestroy(cout);
}

cudaEvent_t Net::prof_event() {
  if (prof_used == prof_events.size()) {
    cudaEvent_t e;
    ck(cudaEventCreate(&e), "cudaEventCreate");
    prof_events.push_back(e);
  }
  return prof_events[prof_used++];
}

void Net::prof_clear() {
  prof_used = 0;
  prof_recs.clear();
}

Net::~Net() {
  for (cudaEvent_t e : prof_events) cudaEventDestroy(e);
  ws.clear();
  if (arena) cudaFree(arena);
}

Workspace* Net::workspace(cudaStream_t st) {
  std::lock_guard<std::mutex> lk(mu);
  auto it = ws.find(st);
  if (it != ws.end()) return it->second.get();
  std::unique_ptr<Workspace> w(new Workspace);
  w->buf.assign(buf_bytes.size(), nullptr);
  for (size_t b = 0; b < buf_bytes.size(); ++b) {
    if (!buf_bytes[b]) continue;
    if (cudaMalloc(&w->buf[b], buf_bytes[b]) != cudaSuccess) throw Error(DJINN_E_NOMEM, "workspace allocation");
    ck(cudaMemset(w->buf[b], 0, buf_bytes[b]), "workspace memset");
  }
  {
    size_t pb = 0;
    for (const Op& o : ops)
      if (o.ksplit > 1) pb = std::max(pb, (size_t)o.ksplit * max_rows * o.npart * 4);
    if (pb && cudaMalloc(&w->part, pb) != cudaSuccess) throw Error(DJINN_E_NOMEM, "split-K workspace");
  }
  w->tmA.resize(ops.size());
  w->tmAs.resize(ops.size());
  w->tmY0.resize(ops.size());
  w->tmY1.resize(ops.size());
  for (size_t i = 0; i < ops.size(); ++i) {
    const Op& o = ops[i];
    if (!o.stem || o.stem_pool) continue;
    // output: the virtual grid [rows * Hs * Ws][Cp]; boxes of 32 pixels x 64 / 32 channels
    const int Cp = o.out.Cp, odt = o.g.out_half ? DT_F16 : dt;
    uint64_t dims[2] = {(uint64_t)Cp, (uint64_t)max_rows * (o.out.H + o.out.hx) * (o.out.W + o.out.wx)};
    uint64_t strides[1] = {(uint64_t)Cp * 2};
    uint32_t box0[2] = {64, 32}, box1[2] = {32, 32};
    encode_tmap(&w->tmY0[i], odt, w->buf[o.out_buf], 2, dims, strides, box0, 128);
    encode_tmap(&w->tmY1[i], odt, w->buf[o.out_buf], 2, dims, strides, box1, 64);
  }
  if (dt != DT_F32) {
    for (size_t i = 0; i < ops.size(); ++i) {
      const Op& o = ops[i];
      if (o.kind != OP_GEMM) continue;
      const GemmGeom& g = o.g;
      if (g.mode == GM_DENSE) {
        uint64_t dims[2] = {(uint64_t)g.a_pitch, (uint64_t)max_rows};
        uint64_t strides[1] = {(uint64_t)g.a_pitch * 2};
        uint32_t box[2] = {64, 128};
        encode_tmap(&w->tmA[i], dt, w->buf[o.in_buf], 2, dims, strides, box);
        if (o.smx) {
          uint32_t bs[2] = {(uint32_t)smx_bk(), (uint32_t)(128 / o.smx_cl)};
          encode_tmap(&w->tmAs[i], dt, w->buf[o.in_buf], 2, dims, strides, bs, 2 * smx_bk());
        }
        if (o.mlp && o.mg.a_tma) {  // the fused MLP tail: 64-column blocks of 128 rows (SW128)
          uint32_t bs[2] = {(uint32_t)mlp2_wk(1), 128};
          encode_tmap(&w->tmAs[i], dt, w->buf[o.in_buf], 2, dims, strides, bs, 2 * mlp2_wk(1));
        }
        continue;
      }
      // NHWC input [max_rows][H][W][Cp] viewed as a 4D tensor {C, W, H, N}
      uint64_t dims[4] = {(uint64_t)g.Cp_in, (uint64_t)g.W, (uint64_t)g.H, (uint64_t)max_rows};
      uint64_t strides[3] = {(uint64_t)g.Cp_in * 2, (uint64_t)g.W * g.Cp_in * 2, (uint64_t)g.H * g.W * g.Cp_in * 2};
      if (g.mode == GM_CONV && g.slab) {
        // slab: the stored input as [rows * Hv * Wv][Cp] pixels; box {64 channels, slab_rows}
        uint64_t d2[2] = {(uint64_t)g.Cp_in, (uint64_t)max_rows * g.Hv * g.Wv};
        uint64_t s2[1] = {(uint64_t)g.Cp_in * 2};
        uint32_t box[2] = {64, (uint32_t)g.slab_rows};
        encode_tmap(&w->tmA[i], dt, w->buf[o.in_buf], 2, d2, s2, box);
      } else if (g.mode == GM_CONV && g.a_tiled) {
        uint32_t box[4] = {(uint32_t)g.cw, (uint32_t)(g.bx * g.stride), (uint32_t)(g.by * g.stride), (uint32_t)g.bn};
        const uint32_t estr[4] = {1, (uint32_t)g.stride, (uint32_t)g.stride, 1};
        encode_tmap(&w->tmA[i], dt, w->buf[o.in_buf], 4, dims, strides, box, g.cw * 2, estr);
      } else if (g.mode == GM_CONV) {
        // filter-window top-left positions: w = -pad + i*stride, i < OW (same for h)
        const int sx = g.xstep;
        const int lower[2] = {-g.pad, -g.pad};
        const int upper[2] = {-g.pad + (g.OWb - 1) * sx - (g.W - 1), -g.pad + (g.OH - 1) * g.stride - (g.H - 1)};
        if (-g.pad + (g.OWb - 1) * sx + (g.KW - 1) * g.kxs > g.W - 1 + g.pad)
          throw Error(DJINN_E_SHAPE, o.name + ": internal: tap offsets exceed the im2col box");
        const uint32_t estr[4] = {1, (uint32_t)sx, (uint32_t)g.stride, 1};
        encode_im2col(&w->tmA[i], dt, w->buf[o.in_buf], dims, strides, lower, upper, g.cw, 128, estr);
      } else if (g.lcg > 1) {
        // LC with lcg taps per row: view each image row as one dense run {W*C, H, N}; a box
        // {lcg*C, 1, 128} is then lcg adjacent pixels = one 128-byte swizzle row per image.
        uint64_t d3[3] = {(uint64_t)g.W * g.Cp_in, (uint64_t)g.H, (uint64_t)max_rows};
        uint64_t s3[2] = {(uint64_t)g.W * g.Cp_in * 2, (uint64_t)g.H * g.W * g.Cp_in * 2};
        uint32_t box[3] = {(uint32_t)g.cw, 1, 128};
        encode_tmap(&w->tmA[i], dt, w->buf[o.in_buf], 3, d3, s3, box, g.cw * 2);
      } else {
        uint32_t box[4] = {(uint32_t)g.cw, 1, 1, 128};
        encode_tmap(&w->tmA[i], dt, w->buf[o.in_buf], 4, dims, strides, box, g.cw * 2);
      }
    }
  }
  Workspace* r = w.get();
  ws[st] = std::move(w);
  return r;
}

// ============================================================================ forward
// Host-fed pipeline depth: rows of one call are cut into this many chunks when the host
// copies are large, so chunk i+1's H2D, chunk i's kernels and chunk i-1's D2H overlap (PCIe
// is the bound in this mode).  DJINN_PIPE_CHUNKS overrides (1 = no split).
static int pipe_chunks(size_t io_bytes) {
  const char* v = getenv("DJINN_PIPE_CHUNKS");
  if (v && atoi(v) > 0) return atoi(v);
  return io_bytes >= (32u << 20) ? 2 : 1;   // measured on B200 (bench e2e): 2 >= 4 > 1
}

void Net::forward(const float* in, int64_t rows, int in_mem, void* out, int out_mem, int mode, cudaStream_t st,
                  bool in16) {
  if (poisoned) throw Error(DJINN_E_CUDA, "net is poisoned by an earlier CUDA error");
  Workspace* w = workspace(st);
  const bool hin = in_mem == DJINN_MEM_HOST, hout = out_mem == DJINN_MEM_HOST;
  if (hin && !in16 && !w->in_stage)
    if (cudaMalloc(&w->in_stage, (size_t)max_rows * in_elems * 4) != cudaSuccess) throw Error(DJINN_E_NOMEM, "input staging");
  if (in16 && !w->in_wide)
    if (cudaMalloc(&w->in_wide, (size_t)max_rows * in_elems * 4) != cudaSuccess) throw Error(DJINN_E_NOMEM, "input widening");
  if (hin && in16 && !w->in_stage16)
    if (cudaMalloc(&w->in_stage16, (size_t)max_rows * in_elems * 2) != cudaSuccess) throw Error(DJINN_E_NOMEM, "input staging");
  const size_t in_row_bytes = (size_t)in_elems * (in16 ? 2 : 4);
  if (hout && !w->out_stage)
    if (cudaMalloc(&w->out_stage, (size_t)max_rows * out_elems * 4) != cudaSuccess) throw Error(DJINN_E_NOMEM, "output staging");
  if ((hin || hout) && !w->cin) {
    ck(cudaStreamCreateWithFlags(&w->cin, cudaStreamNonBlocking), "copy stream");
    ck(cudaStreamCreateWithFlags(&w->cout, cudaStreamNonBlocking), "copy stream");
    for (int s = 0; s < 2; ++s)
      for (cudaEvent_t* e : {&w->in_ready[s], &w->in_free[s], &w->out_ready[s], &w->out_free[s]})
        ck(cudaEventCreateWithFlags(e, cudaEventDisableTiming), "cudaEventCreate");
  }
  const size_t out_row_bytes = mode == DJINN_OUT_ARGMAX ? 4 : (size_t)out_elems * 4;
  // Chunk size: max_rows for device buffers; with host buffers the batch is split into
  // pipe_chunks() chunks using two staging slots (one slot when two do not fit in max_rows).
  int64_t cs = max_rows;
  int slots = 1;
  if (hin || hout) {
    const int64_t nr = std::min<int64_t>(rows, max_rows);
    const size_t io = (size_t)nr * ((hin ? in_row_bytes : 0) + (hout ? out_row_bytes : 0));
    const int P = pipe_chunks(io);
    cs = std::max<int64_t>(1, (nr + P - 1) / P);
    slots = 2 * cs <= max_rows ? 2 : 1;
    if (slots == 1) cs = max_rows;
    if (cs != w->pipe_cs) {
      // slot boundaries moved: the new slots may overlap either old one, so drain both
      for (int s2 = 0; s2 < 2; ++s2) {
        ck(cudaStreamWaitEvent(w->cin, w->in_free[s2], 0), "event wait");
        ck(cudaStreamWaitEvent(st, w->out_free[s2], 0), "event wait");
      }
      w->pipe_cs = cs;
    }
  }
  std::atomic<int64_t>& launches = launch_counter();
  int last_slot = -1;
  for (int64_t r0 = 0, c = 0; r0 < rows; r0 += cs, ++c) {
    const int64_t n = std::min<int64_t>(cs, rows - r0);
    const int sl = (int)(c % slots);
    const float* src = in16 ? (const float*)((const uint16_t*)in + r0 * in_elems) : in + r0 * in_elems;
    if (hin) {
      // H2D into slot `sl` once the kernels of its previous chunk have consumed it
      void* stage = in16 ? (void*)(w->in_stage16 + (size_t)sl * cs * in_elems) : (void*)(w->in_stage + (size_t)sl * cs * in_elems);
      ck(cudaStreamWaitEvent(w->cin, w->in_free[sl], 0), "event wait");
      ck(cudaMemcpyAsync(stage, src, (size_t)n * in_row_bytes, cudaMemcpyHostToDevice, w->cin), "input H2D");
      ck(cudaEventRecord(w->in_ready[sl], w->cin), "event record");
      ck(cudaStreamWaitEvent(st, w->in_ready[sl], 0), "event wait");
      src = (const float*)stage;
    }
    if (in16) {
      // 16-bit rows -> fp32 (exact) in their own buffer (chunks run in order on `st`, so one
      // chunk's worth is enough); the pack then runs unchanged.  The H2D staging slots are
      // never read by the pack on this path, so an interleaved host-fed djinn_forward cannot
      // overwrite rows a pending pack still reads (its in_free wait covers the widen only).
      float* wide = w->in_wide;
      cudaError_t e = launch_widen16(src, wide, n * in_elems, dt, st);
      ++launch_counter();
      if (e != cudaSuccess) {
        poisoned = true;
        throw Error(DJINN_E_CUDA, std::string("widen16: ") + cudaGetErrorString(e));
      }
      if (hin) ck(cudaEventRecord(w->in_free[sl], st), "event record");  // the 16-bit slot is consumed
      src = wide;
    }
    if (hout) ck(cudaStreamWaitEvent(st, w->out_free[sl], 0), "event wait");  // slot's previous D2H done
    uint8_t* dst = hout ? (uint8_t*)w->out_stage + (size_t)sl * cs * out_row_bytes : (uint8_t*)out + r0 * out_row_bytes;
    // Profiling state is snapshotted under the lock: another thread may toggle it or grow
    // prof_events / prof_recs (reallocating them) while this chunk's kernels are enqueued, so
    // the chunk records into a local copy of its own event handles.
    bool prof = false;
    int pop = -1;  // one timed op, or all (-1)
    std::vector<cudaEvent_t> pev;
    {
      std::lock_guard<std::mutex> lk(mu);
      prof = profile;
      pop = profile_op;
      if (prof) {
        const size_t pbase = prof_used;
        prof_recs.push_back({pbase, pop < 0 ? (int)ops.size() : 1, pop});
        for (size_t i = 0; i <= (pop < 0 ? ops.size() : 1); ++i) pev.push_back(prof_event());
      }
    }
    bool smx_done = false;  // the cluster kernel wrote this chunk's outputs (softmax not launched)
    for (size_t i = 0; i < ops.size(); ++i) {
      const Op& o = ops[i];
      cudaError_t e = cudaSuccess;
      bool skipped = false;
      if (prof && (pop < 0 || pop == (int)i)) ck(cudaEventRecord(pev[pop < 0 ? i : 0], st), "profile event");
      const auto th0 = host_prof_on() ? std::chrono::steady_clock::now() : std::chrono::steady_clock::time_point();
      switch (o.kind) {
        case OP_PACK:
          if (o.fused) { skipped = true; break; }  // the stem GEMM reads the fp32 rows itself
          if (o.embed) {
            e = launch_embed(src, (const uint8_t*)arena + o.w_off, w->buf[0], n, o.eg, o.out.Cp, dt, st);
            break;
          }
          e = launch_pack_input(src, w->buf[0], n, o.in.C, o.in.H, o.in.W, o.xform, o.xf, o.xs, o.out.H, o.out.W, o.out.Cp,
                                dt, st);
          break;
        case OP_GEMM: {
          if (o.fused) { skipped = true; break; }
          if (o.smx && n >= o.smx_min_rows) {
            SmxGeom sg{};
            sg.M = n;
            sg.N = o.g.N;
            sg.Kpad = o.g.Kpad;
            sg.CL = o.smx_cl;
            sg.NCW = o.smx_ncw;
            sg.out_mode = mode;
            e = launch_smx(sg, dt, &w->tmAs[i], &o.tmBs, (const float*)((const uint8_t*)arena + o.b_off), dst, st);
            smx_done = true;
            break;
          }
          if (o.mlp) {
            MlpGeom mg = o.mg;
            mg.rows = n;
            mg.out_mode = mode;
            mg.rpc = mg.a_tma ? 128 : mlp2_rows_per_cta(n);
            const uint8_t* ar = (const uint8_t*)arena;
            e = launch_mlp2(mg, dt, &o.tmW1, &o.tmW2, mg.a_tma ? &w->tmAs[i] : nullptr, src, (const float*)(ar + o.b_off),
                            (const float*)(ar + ops[i + 1].b_off), dst, st);
            break;
          }
          GemmGeom g = o.g;
          g.ldwait = ldwait_mode();
          g.tslots = tslots_mode();
          g.epi_wg = epi_wg_mode(g);
          if (n * o.ohw > (int64_t)INT32_MAX / 2) throw Error(DJINN_E_INVAL, o.name + ": GEMM rows exceed 32 bits");
          g.M = (int)(n * o.ohw);
          g.Nimg = (int)n;
          const void* A = w->buf[o.in_buf];
          void* Y = w->buf[o.out_buf];
          const uint8_t* ar = (const uint8_t*)arena;
          if (o.stem) {
            StemGeom sg{};
            sg.Nimg = (int)n;
            sg.H = o.orig_in.H; sg.W = o.orig_in.W;
            sg.Hs = g.H; sg.Ws = g.W;
            sg.OH = g.OH; sg.OW = g.OW;
            sg.N = g.N;
            sg.act = g.act; sg.epi_lrn = g.epi_lrn; sg.out_half = g.out_half;
            sg.lrn_alpha_over_n = g.lrn_alpha_over_n; sg.lrn_beta = g.lrn_beta; sg.lrn_k = g.lrn_k;
            sg.gather = o.stem == 1;
            sg.slab_rows = g.slab_rows;
            if (o.stem_pool) {
              sg.pool = 1;
              sg.POH = o.out.H; sg.POW = o.out.W;
              sg.bands = stem_pool_bands(sg.Nimg, sg.POH);
              sg.Cpo = o.out.Cp;
              sg.pool_gp = o.out.gsz >= g.N ? g.N / 2 : o.out.gpitch;
              sg.obd = o.out.bdr;
            }
            e = launch_stem_conv(sg, dt, &w->tmA[i], &o.tmB, &o.tmBc, &w->tmY0[i], &w->tmY1[i], src,
                                 (const float*)(ar + o.b_off), Y, st);
          } else if (dt == DT_F32)
            e = launch_simt_gemm(g, (const float*)A, (const float*)(ar + o.w_off), (const float*)(ar + o.b_off),
                                 (float*)Y, st);
          else if (o.ksplit > 1) {
            GemmGeom gp = g;  // fp32 partials over o.ksplit K ranges, no bias / activation
            gp.Z = gp.ksplit = o.ksplit;
            gp.kpb = o.kpb;
            gp.act = ACT_NONE;
            gp.out_f32 = 1;
            gp.out_half = 0;
            gp.out_pitch = gp.write_cols = o.npart;
            gp.out_gsz = gp.out_gpitch = 1 << 30;
            gp.bias_zstride = 0;
            e = launch_tc_gemm(gp, o.bn, dt, &w->tmA[i], &o.tmB, (const float*)(ar + o.b_off), w->part, st);
            if (e == cudaSuccess) {
              ++launches;
              e = launch_splitk_reduce(w->part, o.ksplit, n, g.N, o.npart, (const float*)(ar + o.b_off), g.act, Y,
                                       g.out_pitch, g.write_cols, g.out_f32, dt, st);
            }
          } else
            e = launch_tc_gemm(g, o.bn, dt, &w->tmA[i], &o.tmB, (const float*)(ar + o.b_off), Y, st);
          break;
        }
        case OP_LRN:
          e = launch_lrn(w->buf[o.in_buf], w->buf[o.out_buf], n * o.in.H * o.in.W, o.in.C, o.in.Cp, o.in.gsz,
                         o.in.gpitch, o.lrn_size,
                         o.alpha, o.beta, o.lrn_k, dt, st);
          break;
        case OP_POOL:
          if (o.fused) { skipped = true; break; }  // in the first-layer kernel's epilogue
          if (dt != DT_F32 && o.is_max && o.kernel <= o.stride + 1)
            e = launch_pool_remap(w->buf[o.in_buf], w->buf[o.out_buf], n, o.in.C, o.in.Cp, o.in.gsz, o.in.gpitch,
                                  o.in.H, o.in.W, o.in.H + o.in.hx, o.in.W + o.in.wx, o.out.H, o.out.W, o.kernel,
                                  o.stride, o.pad, o.out.Cp, o.out.gsz, o.out.gpitch, o.out.xu, o.out.bdr, dt, st);
          else
            e = launch_pool(w->buf[o.in_buf], w->buf[o.out_buf], n, o.in.C, o.in.Cp, o.in.H, o.in.W, o.out.H, o.out.W,
                            o.kernel, o.stride, o.pad, o.is_max, o.out.xu, dt, st);
          break;
        case OP_LRNPOOL:
          e = launch_lrn_pool(w->buf[o.in_buf], w->buf[o.out_buf], n, o.in.C, o.in.Cp, o.in.H, o.in.W, o.out.H, o.out.W,
                              o.kernel, o.stride, o.pad, o.out.gsz, o.out.gpitch, o.out.Cp, o.out.bdr, o.lrn_size, o.alpha,
                              o.beta, o.lrn_k, dt, st);
          break;
        case OP_SOFTMAX:
          if (o.fused || smx_done) { skipped = true; break; }
          e = launch_softmax((const float*)w->buf[2], n, (int)out_elems, out_pitch, dst, mode, st);
          break;
      }
      if (host_prof_on())
        host_prof_add(name + "/" + o.name, std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - th0).count());
      if (!skipped) ++launches;
      if (e != cudaSuccess) {
        poisoned = true;
        throw Error(DJINN_E_CUDA, o.name + ": " + cudaGetErrorString(e));
      }
      if (prof && pop == (int)i) ck(cudaEventRecord(pev[1], st), "profile event");
      if (i == (ops[0].fused ? 1u : 0u) && hin && !in16)
        ck(cudaEventRecord(w->in_free[sl], st), "event record");  // the pack (or the stem GEMM) has read the slot
    }
    if (prof && pop < 0) ck(cudaEventRecord(pev[ops.size()], st), "profile event");
    if (hout) {
      ck(cudaEventRecord(w->out_ready[sl], st), "event record");
      ck(cudaStreamWaitEvent(w->cout, w->out_ready[sl], 0), "event wait");
      ck(cudaMemcpyAsync((uint8_t*)out + r0 * out_row_bytes, dst, (size_t)n * out_row_bytes, cudaMemcpyDeviceToHost,
                         w->cout),
         "output D2H");
      ck(cudaEventRecord(w->out_free[sl], w->cout), "event record");
      last_slot = sl;
    }
  }
  // The caller's stream completes only after the last D2H has landed in host memory.
  if (last_slot >= 0) ck(cudaStreamWaitEvent(st, w->out_free[last_slot], 0), "event wait");
}

std::string Net::plan_string() const {
  std::ostringstream s;
  static const char* kinds[] = {"pack", "gemm", "lrn", "pool", "softmax", "lrn+pool"};
  static const char* modes[] = {"dense", "conv", "local"};
  s << "net " << name << " precision " << (dt == DT_F32 ? "fp32" : dt == DT_BF16 ? "bf16" : "fp16") << " max_rows "
    << max_rows << " arena " << arena_bytes << " B params " << n_params << "\n";
  for (const Op& o : ops) {
    s << "  " << kinds[o.kind] << " " << o.name << " in " << o.in.C << "x" << o.in.H << "x" << o.in.W << "/p" << o.in.Cp
      << (o.in.bdr ? "+b" + std::to_string(o.in.bdr) : std::string())
      << " -> " << o.out.C << "x" << o.out.H << "x" << o.out.W << "/p" << o.out.Cp
      << (o.out.bdr ? "+b" + std::to_string(o.out.bdr) : std::string()) << " buf " << o.in_buf << "->"
      << o.out_buf;
    if (o.kind == OP_GEMM)
      s << " [" << modes[o.g.mode] << " N=" << o.g.N << " Z=" << o.g.Z << " K=" << o.g.K << " Kpad=" << o.g.Kpad
        << " act=" << o.g.act << " bn=" << o.bn << " cg=" << o.g.cg << " cw=" << o.g.cw << " zf=" << o.g.zf << " KHxKW=" << o.g.KH << "x"
        << o.g.KW << (o.g.xb > 1 ? " xblock=" + std::to_string(o.g.xb) : std::string())
        << (o.g.slab ? " slab=" + std::to_string(o.g.Hv) + "x" + std::to_string(o.g.Wv) + ":" + std::to_string(o.g.slab_parts) + "x" +
                           std::to_string(o.g.slab_rows) + " stages=" + std::to_string(o.g.stages) + "x" + std::to_string(o.g.kps) +
                           (o.g.kv16 == 3 ? std::string(" mma/kblock=3") : std::string())
                     : std::string())
        << (o.g.kxs > 1 ? " x-unrolled-input=" + std::to_string(o.g.kxs) : std::string())
        << (o.g.lcg > 1 ? " taps/row=" + std::to_string(o.g.lcg) : std::string())
        << (o.g.mode == GM_CONV && o.g.a_tiled ? " block=" + std::to_string(o.g.bx) + "x" + std::to_string(o.g.by) + "x" +
                                                  std::to_string(o.g.bn) : std::string())
        << (o.ksplit > 1 ? " split-K=" + std::to_string(o.ksplit) + "x" + std::to_string(o.kpb) : std::string())
        << (o.stem == 1 ? " stem(fp32 input, fused pack, resident B, TMA-store epilogue)" : "")
        << (o.stem == 2 && !o.stem_pool ? " stem(TMA slab, resident B, TMA-store epilogue)" : "")
        << (o.stem_pool ? " stem(TMA slab, resident B, LRN + 3x3/2 max pool in the epilogue)" : "")
        << (o.g.epi_lrn ? " lrn-epilogue" : "") << (o.g.out_f32 ? " fp32-out" : "") << (o.g.out_half ? " fp16-out" : "") << "]";
    if (o.kind == OP_PACK && o.embed) s << " [embedding window " << o.eg.window << " tables " << o.eg.T << " D " << o.eg.D << "]";
    if (o.kind != OP_GEMM && o.fused) s << " [fused]";
    if (o.kind == OP_GEMM && o.fused) s << " [fused into the MLP kernel]";
    if (o.mlp)
      s << (o.mg.a_tma ? " [MLP tail kernel: this layer + the next + softmax in one launch, A by TMA, N1p="
                       : " [MLP kernel: whole net in one launch, N1p=")
        << o.mg.N1p << " K0p=" << o.mg.K0p << " N2p=" << o.mg.N2p
        << (o.mg.nsplit > 1 ? " split over " + std::to_string(o.mg.nsplit) + "-CTA clusters" : std::string()) << "]";
    if (o.smx)
      s << " [+softmax: cluster kernel, " << o.smx_cl << " CTAs x " << o.smx_ncw << " columns per 128 rows, rows >= "
        << o.smx_min_rows << "]";
    if (o.kind == OP_PACK && o.xform)
      s << " [" << (o.xform == 1 ? "space-to-depth " : o.xform == 3 ? "window-unroll " : "kx-unroll ") << o.xf
        << (o.xs > 1 ? " step " + std::to_string(o.xs) : std::string()) << "]";
    s << "\n";
  }
  return s.str();
}

}  // namespace djinn
