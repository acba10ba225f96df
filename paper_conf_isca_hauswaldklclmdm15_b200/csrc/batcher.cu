// Query batcher of the DjiNN service (include/djinn.h "query batcher"): a per-net queue that
// stacks whole queries into one batch -- PAPER.md sec 5.1: batching "stack[s] multiple
// inputs into a larger matrix" and "increases the dimensions of the matrix multiplication" --
// and a worker thread that runs each batch as one djinn_forward on its own CUDA stream.
//
// Host-side runtime only (no kernels): two pinned staging buffers alternate between "filling"
// (clients memcpy their query rows in under the lock) and "running" (the worker's forward:
// pipelined H2D / kernels / D2H, then the per-query output rows are copied to each client's
// buffer).  A batch closes when it is full or its oldest query has waited max_wait_us.
// Tickets are issued and completed in submission order, so completion is one counter.
#include <cuda_runtime.h>
#include <string.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "../../include/djinn.h"
#include "net.h"

namespace {
using Clock = std::chrono::steady_clock;

struct Query {
  int64_t ticket, row0, rows;
  void* out;
  Clock::time_point t0;
};

struct Buffer {
  float* in = nullptr;    // pinned [max_rows][in_elems]
  uint8_t* out = nullptr; // pinned [max_rows][out row bytes]
  std::vector<Query> q;
  int64_t rows = 0;
  int copying = 0;        // submitters still copying their rows in (outside the lock)
};

int bfail(int code, const std::string& m) {
  djinn::set_last_error(m);  // djinn_last_error() of this thread
  return code;
}
}  // namespace

struct djinn_batcher {
  djinn_net* net = nullptr;
  int device = 0, mode = 0;
  int64_t max_rows = 0, max_wait_us = 0, in_elems = 0;
  size_t out_row = 0;
  cudaStream_t st = nullptr;
  Buffer buf[2];
  int fill = 0;                 // buffer clients fill
  bool running[2] = {false, false};
  std::mutex mu;
  std::condition_variable cv_work, cv_space, cv_done;
  int64_t next_ticket = 1, done_upto = 1;  // tickets < done_upto are complete
  struct Failed {
    int64_t first, last;
    int err;
  };
  std::vector<Failed> failed;  // tickets of batches whose forward failed
  bool stop = false;
  bool flush_req = false;  // a submitter's query does not fit the filling buffer: close it now
  std::thread worker;
  // statistics
  int64_t n_batches = 0, n_rows = 0, n_queries = 0;
  std::vector<float> lat_us;  // query latencies (bounded reservoir)

  void run();
  int wait(int64_t ticket, int64_t timeout_us);
};

void djinn_batcher::run() {
  cudaSetDevice(device);
  std::unique_lock<std::mutex> lk(mu);
  for (;;) {
    // a batch is ready when full, when its oldest query is max_wait_us old, or on stop
    for (;;) {
      Buffer& f = buf[fill];
      if (f.rows > 0 && f.copying > 0) {  // rows reserved but not yet copied in
        cv_work.wait(lk);
        continue;
      }
      if (f.rows > 0 && (f.rows >= max_rows || stop || flush_req)) break;
      if (f.rows > 0) {
        const auto due = f.q.front().t0 + std::chrono::microseconds(max_wait_us);
        if (Clock::now() >= due) break;
        cv_work.wait_until(lk, due);
        continue;
      }
      if (stop) return;
      cv_work.wait(lk);
    }
    const int b = fill;
    Buffer& B = buf[b];
    running[b] = true;
    flush_req = false;
    fill ^= 1;  // clients now fill the other buffer (free: the worker runs one batch at a time)
    cv_space.notify_all();
    lk.unlock();
    int err = DJINN_OK;
    std::string msg;
    try {
      net->impl.forward(B.in, B.rows, DJINN_MEM_HOST, B.out, DJINN_MEM_HOST, mode, st);
      const cudaError_t e = cudaStreamSynchronize(st);
      if (e != cudaSuccess) {
        err = DJINN_E_CUDA;
        msg = cudaGetErrorString(e);
      }
    } catch (const djinn::Error& e) {
      err = e.code;
      msg = e.what();
    } catch (const std::exception& e) {
      err = DJINN_E_INVAL;
      msg = e.what();
    }
    const auto t1 = Clock::now();
    if (err == DJINN_OK)
      for (const Query& q : B.q) memcpy(q.out, B.out + q.row0 * out_row, (size_t)q.rows * out_row);
    lk.lock();
    const int64_t last = B.q.back().ticket;
    if (err != DJINN_OK) failed.push_back({B.q.front().ticket, last, err});
    ++n_batches;
    n_rows += B.rows;
    n_queries += (int64_t)B.q.size();
    for (const Query& q : B.q) {
      const float us = (float)std::chrono::duration<double, std::micro>(t1 - q.t0).count();
      if (lat_us.size() < (1u << 20)) lat_us.push_back(us);
      else lat_us[(size_t)(q.ticket % (1 << 20))] = us;
    }
    done_upto = last + 1;
    B.q.clear();
    B.rows = 0;
    running[b] = false;
    cv_done.notify_all();
    cv_space.notify_all();
  }
}

int djinn_batcher::wait(int64_t ticket, int64_t timeout_us) {
  std::unique_lock<std::mutex> lk(mu);
  if (ticket <= 0 || ticket >= next_ticket) return bfail(DJINN_E_INVAL, "unknown ticket");
  auto ready = [&] { return done_upto > ticket; };
  if (timeout_us < 0) cv_done.wait(lk, ready);
  else if (!cv_done.wait_for(lk, std::chrono::microseconds(timeout_us), ready))
    return bfail(DJINN_E_INVAL, "timeout");
  for (const Failed& f : failed)
    if (f.first <= ticket && ticket <= f.last) return bfail(f.err, "the query's batch failed in djinn_forward");
  return DJINN_OK;
}

extern "C" {

int djinn_batcher_create(djinn_net* net, int64_t max_batch_rows, int64_t max_wait_us, int out_mode,
                         djinn_batcher** out) {
  try {
    if (!out) return bfail(DJINN_E_INVAL, "out is NULL");
    *out = nullptr;
    if (!net) return bfail(DJINN_E_INVAL, "net is NULL");
    if (max_batch_rows < 1 || max_batch_rows > net->impl.max_rows) return bfail(DJINN_E_INVAL, "max_batch_rows");
    if (max_wait_us < 0) return bfail(DJINN_E_INVAL, "max_wait_us < 0");
    if (out_mode < DJINN_OUT_PROB || out_mode > DJINN_OUT_LOGITS) return bfail(DJINN_E_INVAL, "out_mode");
    std::unique_ptr<djinn_batcher> b(new djinn_batcher);
    b->net = net;
    b->device = net->impl.device;
    b->mode = out_mode;
    b->max_rows = max_batch_rows;
    b->max_wait_us = max_wait_us;
    b->in_elems = net->impl.in_elems;
    b->out_row = out_mode == DJINN_OUT_ARGMAX ? 4 : (size_t)net->impl.out_elems * 4;
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(b->device);
    bool ok = cudaStreamCreateWithFlags(&b->st, cudaStreamNonBlocking) == cudaSuccess;
    for (int i = 0; i < 2 && ok; ++i) {
      ok = cudaMallocHost(&b->buf[i].in, (size_t)max_batch_rows * b->in_elems * 4) == cudaSuccess &&
           cudaMallocHost(&b->buf[i].out, (size_t)max_batch_rows * b->out_row) == cudaSuccess;
    }
    cudaSetDevice(prev);
    if (!ok) {
      cudaGetLastError();
      for (auto& bb : b->buf) {
        if (bb.in) cudaFreeHost(bb.in);
        if (bb.out) cudaFreeHost(bb.out);
      }
      if (b->st) cudaStreamDestroy(b->st);
      return bfail(DJINN_E_NOMEM, "batcher staging buffers");
    }
    djinn_batcher* p = b.release();
    p->worker = std::thread([p] { p->run(); });
    *out = p;
    return DJINN_OK;
  } catch (const std::exception& e) {
    return bfail(DJINN_E_INVAL, e.what());
  }
}

int djinn_batcher_submit(djinn_batcher* b, const float* input, int64_t rows, void* output, int64_t* ticket) {
  if (!b || !input || !output) return bfail(DJINN_E_INVAL, "NULL argument");
  if (rows < 1 || rows > b->max_rows) return bfail(DJINN_E_INVAL, "rows must be in [1, max_batch_rows]");
  std::unique_lock<std::mutex> lk(b->mu);
  if (b->stop) return bfail(DJINN_E_INVAL, "batcher is stopping");
  // room in the filling buffer, or wait for the worker to swap buffers
  while (b->buf[b->fill].rows + rows > b->max_rows || b->running[b->fill]) {
    b->flush_req = true;  // the filling buffer cannot take this query: run it now
    b->cv_work.notify_one();
    b->cv_space.wait(lk);
  }
  // reserve the rows under the lock, copy them in outside it (concurrent submitters copy in
  // parallel; the worker closes a batch only once every reserved copy has landed)
  Buffer& f = b->buf[b->fill];
  Query q{b->next_ticket++, f.rows, rows, output, Clock::now()};
  float* dst = f.in + f.rows * b->in_elems;
  f.q.push_back(q);
  f.rows += rows;
  ++f.copying;
  if (ticket) *ticket = q.ticket;
  lk.unlock();
  memcpy(dst, input, (size_t)rows * b->in_elems * 4);
  lk.lock();
  --f.copying;
  b->cv_work.notify_one();
  return DJINN_OK;
}

int djinn_batcher_wait(djinn_batcher* b, int64_t ticket, int64_t timeout_us) {
  if (!b) return bfail(DJINN_E_INVAL, "batcher is NULL");
  return b->wait(ticket, timeout_us);
}

int djinn_batcher_stats(djinn_batcher* b, int64_t* batches, int64_t* rows, int64_t* queries, double* p50_us,
                        double* p99_us) {
  if (!b) return bfail(DJINN_E_INVAL, "batcher is NULL");
  std::vector<float> l;
  {
    std::lock_guard<std::mutex> lk(b->mu);
    if (batches) *batches = b->n_batches;
    if (rows) *rows = b->n_rows;
    if (queries) *queries = b->n_queries;
    l = b->lat_us;
  }
  std::sort(l.begin(), l.end());
  auto pct = [&](double p) { return l.empty() ? 0.0 : (double)l[std::min(l.size() - 1, (size_t)(p * l.size()))]; };
  if (p50_us) *p50_us = pct(0.50);
  if (p99_us) *p99_us = pct(0.99);
  return DJINN_OK;
}

int djinn_batcher_drive(djinn_batcher* b, const float* queries, int64_t n_queries, int64_t rows_per_query, int clients,
                        double seconds, double* queries_per_s, double* p50_us, double* p99_us) {
  if (!b || !queries || n_queries < 1 || rows_per_query < 1 || clients < 1 || seconds <= 0)
    return bfail(DJINN_E_INVAL, "bad argument");
  if (rows_per_query > b->max_rows) return bfail(DJINN_E_INVAL, "rows_per_query > max_batch_rows");
  std::atomic<bool> go{true};
  std::atomic<int> err{DJINN_OK};
  std::vector<std::vector<float>> lat(clients);
  std::vector<int64_t> done(clients, 0);
  const size_t out_bytes = (size_t)rows_per_query * b->out_row;
  const auto t0 = Clock::now();
  std::vector<std::thread> th;
  for (int c = 0; c < clients; ++c)
    th.emplace_back([&, c] {
      std::vector<uint8_t> out(out_bytes);
      int64_t i = c;
      while (go.load(std::memory_order_relaxed)) {
        const float* q = queries + (i % n_queries) * rows_per_query * b->in_elems;
        int64_t t = 0;
        const auto s0 = Clock::now();
        int rc = djinn_batcher_submit(b, q, rows_per_query, out.data(), &t);
        if (rc == DJINN_OK) rc = djinn_batcher_wait(b, t, -1);
        if (rc != DJINN_OK) {
          err.store(rc);
          break;
        }
        lat[c].push_back((float)std::chrono::duration<double, std::micro>(Clock::now() - s0).count());
        ++done[c];
        i += clients;
      }
    });
  std::this_thread::sleep_for(std::chrono::duration<double>(seconds));
  go.store(false);
  for (auto& t : th) t.join();
  const double el = std::chrono::duration<double>(Clock::now() - t0).count();
  if (err.load() != DJINN_OK) return bfail(err.load(), "a query failed during the drive");
  std::vector<float> all;
  int64_t n = 0;
  for (int c = 0; c < clients; ++c) {
    n += done[c];
    all.insert(all.end(), lat[c].begin(), lat[c].end());
  }
  std::sort(all.begin(), all.end());
  auto pct = [&](double p) { return all.empty() ? 0.0 : (double)all[std::min(all.size() - 1, (size_t)(p * all.size()))]; };
  if (queries_per_s) *queries_per_s = n / el;
  if (p50_us) *p50_us = pct(0.50);
  if (p99_us) *p99_us = pct(0.99);
  return DJINN_OK;
}

int djinn_batcher_destroy(djinn_batcher* b) {
  if (!b) return DJINN_OK;
  {
    std::lock_guard<std::mutex> lk(b->mu);
    b->stop = true;
  }
  b->cv_work.notify_all();
  if (b->worker.joinable()) b->worker.join();
  for (auto& bb : b->buf) {
    if (bb.in) cudaFreeHost(bb.in);
    if (bb.out) cudaFreeHost(bb.out);
  }
  if (b->st) cudaStreamDestroy(b->st);
  delete b;
  return DJINN_OK;
}

}  // extern "C"
