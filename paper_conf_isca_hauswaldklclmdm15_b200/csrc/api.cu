// C ABI of libdjinn (include/djinn.h).  Argument validation, error translation
// (no exception crosses the boundary), device selection, thread-local error message.
#include <string.h>

#include <string>

#include "../../include/djinn.h"
#include "net.h"


namespace {
thread_local std::string g_err;

int fail(int code, const std::string& msg) {
  g_err = msg;
  return code;
}

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

template <typename F>
int guarded(F&& f) {
  try {
    g_err.clear();
    return f();
  } catch (const djinn::Error& e) {
    return fail(e.code, e.what());
  } catch (const std::bad_alloc&) {
    return fail(DJINN_E_NOMEM, "host allocation failed");
  } catch (const std::exception& e) {
    return fail(DJINN_E_INVAL, e.what());
  } catch (...) {
    return fail(DJINN_E_INVAL, "unknown error");
  }
}
}  // namespace

namespace djinn {
void set_last_error(const std::string& msg) { g_err = msg; }
}  // namespace djinn

extern "C" {

int djinn_load_net(const char* desc, size_t desc_len, const float* weights, size_t n_floats, int weights_mem,
                   int device, int precision, int64_t max_rows, djinn_net** out) {
  return guarded([&]() -> int {
    if (!out) return fail(DJINN_E_INVAL, "out is NULL");
    *out = nullptr;
    if (!desc) return fail(DJINN_E_INVAL, "desc is NULL");
    if (precision < DJINN_FP32 || precision > DJINN_FP16) return fail(DJINN_E_INVAL, "bad precision");
    if (weights_mem != DJINN_MEM_HOST && weights_mem != DJINN_MEM_DEVICE) return fail(DJINN_E_INVAL, "bad weights_mem");
    if (max_rows <= 0) return fail(DJINN_E_INVAL, "max_rows must be > 0");
    if (max_rows > (int64_t)1 << 31) return fail(DJINN_E_INVAL, "max_rows too large");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
      cudaGetLastError();
      return fail(DJINN_E_CUDA, "no CUDA device");
    }
    if (device < 0 || device >= ndev) return fail(DJINN_E_INVAL, "bad device ordinal");
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) return fail(DJINN_E_CUDA, "cudaGetDeviceProperties");
    if (prop.major != 10) return fail(DJINN_E_CUDA, "libdjinn is built for sm_100a (B200); device is sm_" +
                                                        std::to_string(prop.major) + std::to_string(prop.minor));
    DeviceGuard dg(device);
    std::unique_ptr<djinn_net> net(new djinn_net);
    djinn::Net& n = net->impl;
    n.device = device;
    n.precision = precision;
    n.dt = precision == DJINN_FP32 ? djinn::DT_F32 : precision == DJINN_BF16 ? djinn::DT_BF16 : djinn::DT_F16;
    n.max_rows = max_rows;
    n.build(std::string(desc, desc_len));
    if (weights && n_floats != (size_t)n.n_params)
      return fail(DJINN_E_WEIGHTS, "weight blob has " + std::to_string(n_floats) + " floats, description needs " +
                                       std::to_string(n.n_params));
    if (cudaMalloc(&n.arena, n.arena_bytes) != cudaSuccess) {
      cudaGetLastError();
      return fail(DJINN_E_NOMEM, "weight arena allocation (" + std::to_string(n.arena_bytes) + " B)");
    }
    // per-layer tile choice and B tensor maps over the arena
    n.choose_tiles();
    // GEMM rows are 32-bit in the kernels (M = rows x output pixels per row): reject a
    // max_rows that would wrap instead of silently skipping the GEMM
    for (const djinn::Op& o : n.ops)
      if (o.kind == djinn::OP_GEMM && (int64_t)max_rows * o.ohw > (int64_t)INT32_MAX / 2)
        return fail(DJINN_E_INVAL, o.name + ": max_rows x output pixels (" + std::to_string(max_rows) + " x " +
                                       std::to_string(o.ohw) + ") exceeds the 32-bit GEMM row range");
    for (djinn::Op& o : n.ops) {
      if (o.kind != djinn::OP_GEMM || n.dt == djinn::DT_F32) continue;
      const djinn::GemmGeom& g = o.g;
      uint64_t dims[3] = {(uint64_t)g.Kpad, (uint64_t)g.N, (uint64_t)g.Z};
      uint64_t strides[2] = {(uint64_t)g.Kpad * 2, (uint64_t)g.N * g.Kpad * 2};
      uint32_t box[3] = {64, (uint32_t)(o.bn / o.g.cg), 1};
      djinn::encode_tmap(&o.tmB, n.dt, (uint8_t*)n.arena + o.w_off, 3, dims, strides, box);
      if (o.stem && djinn::stem_dense_b()) {  // K-dense resident filter bank (kernels.h)
        const int kd = (g.KH * g.KW * o.xf * o.xf * o.orig_in.C + 63) / 64 * 64;
        uint64_t d2[2] = {(uint64_t)kd, (uint64_t)g.N}, s2[1] = {(uint64_t)g.Kpad * 2};
        uint32_t b2[2] = {64, (uint32_t)(g.N / 2)};
        djinn::encode_tmap(&o.tmBc, n.dt, (uint8_t*)n.arena + o.w_off, 2, d2, s2, b2, 128);
      }
    }
    for (djinn::Op& o : n.ops) {  // dense + softmax cluster kernel: its B map, if clusters fit
      if (!o.smx) continue;
      if (djinn::smx_max_active_clusters(n.dt, o.smx_cl) < 1) { o.smx = 0; continue; }
      uint64_t dims[2] = {(uint64_t)o.g.Kpad, (uint64_t)o.g.N}, strides[1] = {(uint64_t)o.g.Kpad * 2};
      uint32_t box[2] = {(uint32_t)djinn::smx_bk(), 256};
      djinn::encode_tmap(&o.tmBs, n.dt, (uint8_t*)n.arena + o.w_off, 2, dims, strides, box, 2 * djinn::smx_bk());
    }
    for (size_t i = 0; i < n.ops.size(); ++i) {  // fused MLP: W1 / W2 maps for its own tiles
      djinn::Op& o = n.ops[i];
      if (!o.mlp) continue;
      const djinn::Op& o2 = n.ops[i + 1];
      uint64_t d1[2] = {(uint64_t)o.g.Kpad, (uint64_t)o.g.N}, s1[1] = {(uint64_t)o.g.Kpad * 2};
      const int wk = djinn::mlp2_wk(o.mg.a_tma);
      uint32_t b1[2] = {(uint32_t)wk, (uint32_t)(o.mg.N1p / (o.mg.nsplit > 1 ? o.mg.nsplit : 1) / 2)};
      djinn::encode_tmap(&o.tmW1, n.dt, (uint8_t*)n.arena + o.w_off, 2, d1, s1, b1, 2 * wk);
      uint64_t d2[2] = {(uint64_t)o2.g.Kpad, (uint64_t)o2.g.N}, s2[1] = {(uint64_t)o2.g.Kpad * 2};
      uint32_t b2[2] = {64, (uint32_t)o.mg.N2p};
      djinn::encode_tmap(&o.tmW2, n.dt, (uint8_t*)n.arena + o2.w_off, 2, d2, s2, b2, 128);
    }
    if (weights) n.load_weights(weights, n_floats, weights_mem);
    *out = net.release();
    return DJINN_OK;
  });
}

int djinn_forward(djinn_net* net, const float* input, int64_t rows, int in_mem, void* output, int out_mem,
                  int out_mode, void* stream) {
  return guarded([&]() -> int {
    if (!net) return fail(DJINN_E_INVAL, "net is NULL");
    if (rows < 0) return fail(DJINN_E_INVAL, "rows < 0");
    if (rows == 0) return DJINN_OK;
    if (!input || !output) return fail(DJINN_E_INVAL, "input/output is NULL");
    if (in_mem != DJINN_MEM_HOST && in_mem != DJINN_MEM_DEVICE) return fail(DJINN_E_INVAL, "bad in_mem");
    if (out_mem != DJINN_MEM_HOST && out_mem != DJINN_MEM_DEVICE) return fail(DJINN_E_INVAL, "bad out_mem");
    if (out_mode < DJINN_OUT_PROB || out_mode > DJINN_OUT_LOGITS) return fail(DJINN_E_INVAL, "bad out_mode");
    DeviceGuard dg(net->impl.device);
    net->impl.forward(input, rows, in_mem, output, out_mem, out_mode, (cudaStream_t)stream);
    return DJINN_OK;
  });
}

int djinn_forward16(djinn_net* net, const void* input, int64_t rows, int in_mem, void* output, int out_mem,
                    int out_mode, void* stream) {
  return guarded([&]() -> int {
    if (!net) return fail(DJINN_E_INVAL, "net is NULL");
    if (rows < 0) return fail(DJINN_E_INVAL, "rows < 0");
    if (net->impl.dt == djinn::DT_F32) return fail(DJINN_E_UNSUPPORTED, "16-bit input on an fp32 net");
    if (rows == 0) return DJINN_OK;
    if (!input || !output) return fail(DJINN_E_INVAL, "input/output is NULL");
    if (in_mem != DJINN_MEM_HOST && in_mem != DJINN_MEM_DEVICE) return fail(DJINN_E_INVAL, "bad in_mem");
    if (out_mem != DJINN_MEM_HOST && out_mem != DJINN_MEM_DEVICE) return fail(DJINN_E_INVAL, "bad out_mem");
    if (out_mode < DJINN_OUT_PROB || out_mode > DJINN_OUT_LOGITS) return fail(DJINN_E_INVAL, "bad out_mode");
    DeviceGuard dg(net->impl.device);
    net->impl.forward((const float*)input, rows, in_mem, output, out_mem, out_mode, (cudaStream_t)stream, true);
    return DJINN_OK;
  });
}

int djinn_sync(djinn_net* net, void* stream) {
  return guarded([&]() -> int {
    if (!net) return fail(DJINN_E_INVAL, "net is NULL");
    DeviceGuard dg(net->impl.device);
    cudaError_t e = cudaStreamSynchronize((cudaStream_t)stream);
    if (e == cudaSuccess) e = cudaGetLastError();
    if (e != cudaSuccess) {
      net->impl.poisoned = true;
      return fail(DJINN_E_CUDA, std::string("asynchronous CUDA error: ") + cudaGetErrorString(e));
    }
    return DJINN_OK;
  });
}

int djinn_free(djinn_net* net) {
  return guarded([&]() -> int {
    if (!net) return DJINN_OK;
    DeviceGuard dg(net->impl.device);
    delete net;
    return DJINN_OK;
  });
}

int djinn_net_info(const djinn_net* net, int64_t* in_elems, int64_t* out_elems, int64_t* n_params,
                   int64_t* n_layers) {
  return guarded([&]() -> int {
    if (!net) return fail(DJINN_E_INVAL, "net is NULL");
    if (in_elems) *in_elems = net->impl.in_elems;
    if (out_elems) *out_elems = net->impl.out_elems;
    if (n_params) *n_params = net->impl.n_params;
    if (n_layers) *n_layers = net->impl.n_layers;
    return DJINN_OK;
  });
}

int djinn_weight_arena(djinn_net* net, void** dev_ptr, size_t* bytes) {
  return guarded([&]() -> int {
    if (!net || !dev_ptr || !bytes) return fail(DJINN_E_INVAL, "NULL argument");
    *dev_ptr = net->impl.arena;
    *bytes = net->impl.arena_bytes;
    return DJINN_OK;
  });
}

int djinn_plan_info(const djinn_net* net, char* buf, size_t cap) {
  return guarded([&]() -> int {
    if (!net) return fail(DJINN_E_INVAL, "net is NULL");
    std::string s = net->impl.plan_string();
    if (buf && cap) {
      size_t k = s.size() < cap - 1 ? s.size() : cap - 1;
      memcpy(buf, s.data(), k);
      buf[k] = 0;
    }
    return (int)s.size();
  });
}

int djinn_profile(djinn_net* net, int enable) {
  return guarded([&]() -> int {
    if (!net) return fail(DJINN_E_INVAL, "net is NULL");
    std::lock_guard<std::mutex> lk(net->impl.mu);
    net->impl.prof_clear();
    if (enable >= 2 && enable - 2 >= (int)net->impl.ops.size()) return fail(DJINN_E_INVAL, "profile op out of range");
    net->impl.profile = enable != 0;
    net->impl.profile_op = enable >= 2 ? enable - 2 : -1;
    return DJINN_OK;
  });
}

int djinn_profile_read(djinn_net* net, double* ms, int64_t* count, int cap, int reset) {
  return guarded([&]() -> int {
    if (!net) return fail(DJINN_E_INVAL, "net is NULL");
    djinn::Net& n = net->impl;
    DeviceGuard dg(n.device);
    std::lock_guard<std::mutex> lk(n.mu);
    const int nops = (int)n.ops.size();
    std::vector<double> acc(nops, 0.0);
    std::vector<int64_t> cnt(nops, 0);
    for (const djinn::ProfRec& r : n.prof_recs) {
      if (cudaEventSynchronize(n.prof_events[r.first + r.n_ops]) != cudaSuccess)
        return fail(DJINN_E_CUDA, "profile event synchronize");
      for (int i = 0; i < r.n_ops && i < nops; ++i) {
        float t = 0.f;
        if (cudaEventElapsedTime(&t, n.prof_events[r.first + i], n.prof_events[r.first + i + 1]) != cudaSuccess)
          return fail(DJINN_E_CUDA, "cudaEventElapsedTime");
        const int op = r.op >= 0 ? r.op : i;
        acc[op] += t;
        cnt[op] += 1;
      }
    }
    for (int i = 0; i < nops && i < cap; ++i) {
      if (ms) ms[i] = acc[i];
      if (count) count[i] = cnt[i];
    }
    if (reset) n.prof_clear();
    return nops;
  });
}

int djinn_op_info(const djinn_net* net, int op, char* name, size_t name_cap, int* kind, double* flops_per_row,
                  double* bytes_per_row, double* weight_bytes) {
  return guarded([&]() -> int {
    if (!net) return fail(DJINN_E_INVAL, "net is NULL");
    const djinn::Net& n = net->impl;
    if (op < 0 || op >= (int)n.ops.size()) return fail(DJINN_E_INVAL, "op index out of range");
    const djinn::Op& o = n.ops[op];
    if (name && name_cap) {
      size_t k = o.name.size() < name_cap - 1 ? o.name.size() : name_cap - 1;
      memcpy(name, o.name.data(), k);
      name[k] = 0;
    }
    if (kind) *kind = (int)o.kind;
    if (flops_per_row) *flops_per_row = o.flops_row;
    if (bytes_per_row) *bytes_per_row = o.bytes_row;
    if (weight_bytes) *weight_bytes = o.weight_bytes;
    return (int)n.ops.size();
  });
}

int djinn_describe(const char* desc, size_t desc_len, int precision, int64_t max_rows, char* buf, size_t cap,
                   int64_t* in_elems, int64_t* out_elems, int64_t* n_params, int64_t* n_layers) {
  return guarded([&]() -> int {
    if (!desc) return fail(DJINN_E_INVAL, "desc is NULL");
    if (precision < DJINN_FP32 || precision > DJINN_FP16) return fail(DJINN_E_INVAL, "bad precision");
    if (max_rows <= 0) return fail(DJINN_E_INVAL, "max_rows must be > 0");
    djinn::Net n;
    n.precision = precision;
    n.dt = precision == DJINN_FP32 ? djinn::DT_F32 : precision == DJINN_BF16 ? djinn::DT_BF16 : djinn::DT_F16;
    n.max_rows = max_rows;
    n.build(std::string(desc, desc_len));
    n.choose_tiles();
    if (in_elems) *in_elems = n.in_elems;
    if (out_elems) *out_elems = n.out_elems;
    if (n_params) *n_params = n.n_params;
    if (n_layers) *n_layers = n.n_layers;
    std::string s = n.plan_string();
    if (buf && cap) {
      size_t k = s.size() < cap - 1 ? s.size() : cap - 1;
      memcpy(buf, s.data(), k);
      buf[k] = 0;
    }
    return (int)s.size();
  });
}

const char* djinn_last_error(void) { return g_err.c_str(); }

int64_t djinn_kernel_launches(void) { return djinn::launch_counter(); }

}  // extern "C"
