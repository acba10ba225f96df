/*
 * djinn.h -- C ABI of the B200-native DjiNN hot path: the batched DNN forward pass
 * (inference) that serves the Tonic Suite networks.
 *
 * The calls follow the paper's statement of the service (sec 3.1):
 *   - "At initialization, DjiNN loads the pre-trained model associated with each
 *     application into memory, giving all worker threads read-only access to this
 *     data" (L84)                                      -> djinn_load_net / djinn_free
 *   - "DjiNN executes the DNN inference pass, which generates a prediction using the
 *     pre-processed input from the application, and returns the prediction result"
 *     (L71); image apps return a classification, ASR/NLP probability vectors
 *     (Table 3)                              -> djinn_forward (out_mode)
 *   - batching "stack[s] multiple inputs into a larger matrix" (L185)
 *                                                      -> `rows` of djinn_forward
 *   - "supporting more applications simply requires providing DjiNN a pretrained
 *     neural network model" (L78)                      -> any net description in the
 *                                                         supported layer subset
 *
 * Conventions (all calls):
 *   - Return 0 (DJINN_OK) on success, a negative DJINN_E_* code on failure; the
 *     message of the last failure on the calling thread is djinn_last_error().
 *     No C++ exception ever crosses this boundary.
 *   - Pointers are borrowed for the duration of the call only; the library copies
 *     what it keeps.  The library owns every device allocation it makes (weight
 *     arena, per-stream workspaces) until djinn_free.
 *   - Everything the network computes runs in this library's sm_100a kernels; there
 *     is no CPU fallback.  A process without a usable sm_100 device gets
 *     DJINN_E_CUDA from djinn_load_net.
 */
#ifndef DJINN_H
#define DJINN_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define DJINN_API __attribute__((visibility("default")))
#else
#define DJINN_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct djinn_net djinn_net;   /* opaque; owned by the library until djinn_free */

enum {
  DJINN_OK = 0,
  DJINN_E_INVAL = -1,        /* bad argument (null pointer, bad enum, rows < 0)            */
  DJINN_E_PARSE = -2,        /* net description does not parse                             */
  DJINN_E_SHAPE = -3,        /* layer shapes inconsistent / unsupported geometry           */
  DJINN_E_WEIGHTS = -4,      /* weight blob length does not match the description          */
  DJINN_E_NOMEM = -5,        /* device or host allocation failed                           */
  DJINN_E_CUDA = -6,         /* CUDA runtime/driver error (also: no sm_100 device)         */
  DJINN_E_UNSUPPORTED = -7   /* layer type / option not supported                          */
};

/* Compute path.  FP32: SIMT FFMA kernels, fp32 storage (exact fp32 accumulation, no TF32).
 * BF16 / FP16: tcgen05 tensor-core kernels, 16-bit operands and activations, fp32
 * accumulation in TMEM, fp32 bias, fp32 logits and probabilities. */
enum { DJINN_FP32 = 0, DJINN_BF16 = 1, DJINN_FP16 = 2 };

/* Memory kind of a caller buffer. */
enum { DJINN_MEM_HOST = 0, DJINN_MEM_DEVICE = 1 };

/* Output of djinn_forward.
 * PROB:   float32 [rows, out_dim] softmax probabilities (default; Table 3 "probability vectors")
 * ARGMAX: int32   [rows] index of the largest logit, ties -> lowest index (Table 3 "classification")
 * LOGITS: float32 [rows, out_dim] pre-softmax scores of the last layer */
enum { DJINN_OUT_PROB = 0, DJINN_OUT_ARGMAX = 1, DJINN_OUT_LOGITS = 2 };

/*
 * djinn_load_net -- parse a net description, pack its weights on `device`, and
 * prepare kernels and workspaces for batches of up to `max_rows` rows.
 *
 *   desc, desc_len : net description text, a subset of Caffe prototxt:
 *                    `name`, `rows_per_query`, and a linear chain of `layer { ... }`
 *                    of types Input (first), Convolution (num_output, kernel_size,
 *                    stride, pad, group), LocallyConnected (num_output, kernel_size,
 *                    stride), InnerProduct (num_output), ReLU, Sigmoid, TanH, HardTanh,
 *                    LRN (local_size, alpha, beta, k; ACROSS_CHANNELS), Pooling
 *                    (pool MAX|AVE, kernel_size, stride, pad; Caffe ceil geometry),
 *                    Dropout (identity at inference), Softmax (last), and Embedding
 *                    (embedding_param: window, then `vocab: V dim: D` per table; only
 *                    directly after an Input of window * tables values): the SENNA
 *                    window lookup the NLP apps run before DjiNN (L104), done in the
 *                    service -- row input = per word the T table indices (word-major,
 *                    exact integers as float32; an index outside [0, V) or not an
 *                    integer selects the zero vector), output = the concatenated
 *                    window vector.  Copied.
 *   weights        : canonical blob, little-endian float32: for each parametrised layer
 *                    in file order its weights then its bias, C-order, shapes
 *                      Convolution      W[Co][Ci/group][k][k],  b[Co]
 *                      LocallyConnected W[OH][OW][Co][Ci][k][k], b[Co][OH][OW]
 *                      InnerProduct     W[No][K] with K in Caffe (c,h,w) order, b[No]
 *                      Embedding        the tables [V_t][D_t] back to back, no bias
 *                    May be NULL: the weight arena is then left uninitialised, to be
 *                    filled through djinn_weight_arena (e.g. an NCCL broadcast from a
 *                    rank that loaded the same description with weights).
 *   n_floats       : number of floats in `weights` (checked: DJINN_E_WEIGHTS).
 *   weights_mem    : DJINN_MEM_HOST or DJINN_MEM_DEVICE (where `weights` lives).
 *   device         : CUDA device ordinal the net lives on.
 *   precision      : DJINN_FP32 | DJINN_BF16 | DJINN_FP16.  16-bit paths round the
 *                    weights to nearest-even at load.
 *   max_rows       : largest batch (rows) processed in one internal pass; larger
 *                    djinn_forward calls are split into chunks of max_rows.  > 0.
 *   out            : receives the net handle.
 */
DJINN_API int djinn_load_net(const char* desc, size_t desc_len, const float* weights, size_t n_floats,
                   int weights_mem, int device, int precision, int64_t max_rows,
                   djinn_net** out);

/*
 * djinn_forward -- run the forward pass of `rows` stacked queries' rows.
 *
 *   input     : float32 [rows, in_elems_per_row] in Caffe NCHW order per row
 *               (Table 3 sizes imply fp32 inputs).  Host or device (in_mem).
 *   rows      : number of rows (>= 0; 0 is a no-op).
 *   output    : per out_mode (see DJINN_OUT_*), host or device (out_mem); must hold
 *               rows * out_elems_per_row floats (PROB/LOGITS) or rows int32 (ARGMAX).
 *   stream    : cudaStream_t to run on (NULL = legacy default stream).  The call is
 *               asynchronous with respect to the host.  With host buffers (the paper's
 *               PCIe-fed service, L231-253) the rows are cut into 2 chunks when the copies
 *               exceed 32 MB
 *               (DJINN_PIPE_CHUNKS env overrides) and the library's own copy streams
 *               overlap chunk i+1's H2D and chunk i-1's D2H with chunk i's kernels on
 *               `stream`; host `input` is read as soon as the call is issued (not
 *               ordered after earlier work on `stream`), and `stream` reaches the end of
 *               this call only after the last D2H has landed.  The caller synchronises
 *               `stream` (djinn_sync) before reading a host `output` or reusing `input`;
 *               page-locked host buffers are needed for the copies to be asynchronous.
 * Thread safety: concurrent calls on one net are safe when they use different streams
 * (weights are read-only; each stream gets its own workspace).  Not concurrent with
 * djinn_free.
 */
DJINN_API int djinn_forward(djinn_net* net, const float* input, int64_t rows, int in_mem,
                  void* output, int out_mem, int out_mode, void* stream);

/*
 * djinn_forward16 -- djinn_forward with the input rows already in the net's 16-bit
 * storage type (bf16 for a DJINN_BF16 net, fp16 for DJINN_FP16): the values the first
 * kernel would round fp32 inputs to, so results are bit-identical to djinn_forward on the
 * widened rows, while a host-fed query moves half the bytes over PCIe (the bottleneck
 * the paper measured for its services, L231-253).
 *   input : uint16 [rows, in_elems_per_row], same row order as djinn_forward; host or
 *           device (in_mem).  Other arguments, asynchrony and threading as djinn_forward.
 * Errors: DJINN_E_UNSUPPORTED on a DJINN_FP32 net.  (Inputs that are not 16-bit floats,
 * e.g. the Embedding layer's token indices, go through djinn_forward.)
 */
DJINN_API int djinn_forward16(djinn_net* net, const void* input, int64_t rows, int in_mem,
                  void* output, int out_mem, int out_mode, void* stream);

/* djinn_sync -- synchronise `stream` and surface asynchronous CUDA errors as
 * DJINN_E_CUDA. */
DJINN_API int djinn_sync(djinn_net* net, void* stream);

/* djinn_free -- release every allocation of the net.  NULL is OK. */
DJINN_API int djinn_free(djinn_net* net);

/* djinn_net_info -- any pointer may be NULL.
 *   in_elems_per_row : product of the Input shape (e.g. 3*227*227)
 *   out_elems_per_row: classes of the last layer
 *   n_params         : number of floats in the canonical weight blob
 *   n_layers         : layers excluding Input and Softmax */
DJINN_API int djinn_net_info(const djinn_net* net, int64_t* in_elems_per_row, int64_t* out_elems_per_row,
                   int64_t* n_params, int64_t* n_layers);

/* djinn_weight_arena -- device pointer and size of the packed weight arena (one
 * allocation), for the one-time weight broadcast of the multi-GPU harness
 * (SURVEY.md sec 8(e)).  Nets loaded from the same description, precision and
 * max_rows have byte-identical arena layouts. */
DJINN_API int djinn_weight_arena(djinn_net* net, void** dev_ptr, size_t* bytes);

/* djinn_plan_info -- human-readable description of the execution plan (kernels, tile
 * shapes, buffer sizes); `buf` receives a NUL-terminated string, truncated to `cap`.
 * Returns the full length (excluding NUL) or a negative error. */
DJINN_API int djinn_plan_info(const djinn_net* net, char* buf, size_t cap);

/* djinn_profile -- enable (1) / disable (0) per-op device timing of subsequent
 * djinn_forward calls on this net: a CUDA event is recorded on the forward's stream
 * before each kernel and after the last one (PAPER.md L151-173 profiles per kernel,
 * weighted by kernel time).  enable = 2 + k times plan op k only (one event before and
 * one after its kernel; the rest of the forward keeps its programmatic-launch overlap).
 * Enabling clears earlier records.  k out of range: DJINN_E_INVAL. */
DJINN_API int djinn_profile(djinn_net* net, int enable);

/* djinn_profile_read -- synchronise the recorded events and return, per op of the plan
 * (index 0..n_ops-1), the summed device milliseconds and the number of timed launches.
 * ms / count may be NULL; at most `cap` entries are written.  reset != 0 clears the
 * records.  Returns n_ops or a negative error. */
DJINN_API int djinn_profile_read(djinn_net* net, double* ms, int64_t* count, int cap, int reset);

/* djinn_op_info -- static description of plan op `op` (0 <= op < n_ops):
 *   name (NUL-terminated, truncated to name_cap), kind (0 pack, 1 gemm, 2 lrn, 3 pool,
 *   4 softmax), and its ALGORITHMIC work per row of the batch: flops (2 per
 *   multiply-add, real unpadded dimensions), activation bytes read + written at the
 *   path's storage width, and the bytes of weights + bias it must read once per launch.
 * Any output pointer may be NULL.  Returns n_ops or a negative error. */
DJINN_API int djinn_op_info(const djinn_net* net, int op, char* name, size_t name_cap, int* kind,
                            double* flops_per_row, double* bytes_per_row, double* weight_bytes);

/* djinn_describe -- parse and plan `desc` for `precision` / `max_rows` WITHOUT touching a
 * device or weights (host-side planner only): writes the plan text (as djinn_plan_info)
 * into buf (truncated to cap) and the net's in/out elements per row, parameter and layer
 * counts (any pointer may be NULL).  Returns the full plan length or a negative error
 * (DJINN_E_PARSE / _SHAPE / _UNSUPPORTED / _INVAL). */
DJINN_API int djinn_describe(const char* desc, size_t desc_len, int precision, int64_t max_rows, char* buf,
                             size_t cap, int64_t* in_elems_per_row, int64_t* out_elems_per_row, int64_t* n_params,
                             int64_t* n_layers);

/* djinn_last_error -- thread-local message of the last failure ("" if none). */
DJINN_API const char* djinn_last_error(void);

/* djinn_kernel_launches -- number of kernels the library launched on this process
 * since load (for the bench's gpu_launches claim). */
DJINN_API int64_t djinn_kernel_launches(void);

/* ------------------------------------------------------------------ query batcher
 * The service's batching (sec 5.1: "stacking multiple inputs into a larger
 * matrix ... increases the dimensions of the matrix multiplication"; Table 3 L153-161 batches
 * queries of an application): a per-net queue in front of djinn_forward.  Clients submit whole
 * queries (any number of rows) from any thread; a worker thread stacks pending queries into one
 * batch of at most max_batch_rows rows and runs it as one djinn_forward (pinned host staging,
 * the library's own stream) when the batch is full or its oldest query has waited max_wait_us,
 * then copies each query's output rows back.  While one batch runs on the GPU the next one
 * fills (two staging buffers).
 *
 * Ownership: `input` is copied at submit; `output` (host memory of rows x the out_mode's row
 * size, see djinn_forward) must stay valid until the query's djinn_batcher_wait returned.  The
 * net must outlive the batcher; the batcher uses its own CUDA stream of the net's device.
 * Tickets are positive and complete in submission order.  A forward error fails every query
 * of that batch (their wait returns the error) and the batcher stays usable. */
typedef struct djinn_batcher djinn_batcher;

/* max_batch_rows in [1, the net's max_rows]; max_wait_us >= 0 (0: run whatever is pending as
 * soon as the worker is free). */
DJINN_API int djinn_batcher_create(djinn_net* net, int64_t max_batch_rows, int64_t max_wait_us, int out_mode,
                                   djinn_batcher** out);
/* Queue one query of `rows` rows (1 <= rows <= max_batch_rows) of fp32 host input; blocks only
 * while both staging buffers are busy.  *ticket receives the query's ticket. */
DJINN_API int djinn_batcher_submit(djinn_batcher* b, const float* input, int64_t rows, void* output, int64_t* ticket);
/* Wait until the query `ticket` has its output (timeout_us < 0: no limit).  Returns DJINN_OK,
 * DJINN_E_INVAL on timeout / unknown ticket, or the error of its batch's forward. */
DJINN_API int djinn_batcher_wait(djinn_batcher* b, int64_t ticket, int64_t timeout_us);
/* Statistics since create: batches run, rows run, queries completed, and query latency
 * (submit -> output written) percentiles p50 / p99 in microseconds (any pointer may be NULL). */
DJINN_API int djinn_batcher_stats(djinn_batcher* b, int64_t* batches, int64_t* rows, int64_t* queries, double* p50_us,
                                  double* p99_us);
/* Closed-loop load generator for the serving measurements: `clients` native threads, each
 * repeatedly submitting the next query of `queries` (n_queries x rows_per_query fp32 rows, used
 * round robin) and waiting for it, for `seconds`.  Reports completed queries per second and the
 * p50 / p99 latency of the queries of that run. */
DJINN_API int djinn_batcher_drive(djinn_batcher* b, const float* queries, int64_t n_queries, int64_t rows_per_query,
                                  int clients, double seconds, double* queries_per_s, double* p50_us, double* p99_us);
/* Drain pending queries, stop the worker, free the staging buffers. */
DJINN_API int djinn_batcher_destroy(djinn_batcher* b);

#ifdef __cplusplus
}
#endif
#endif /* DJINN_H */
