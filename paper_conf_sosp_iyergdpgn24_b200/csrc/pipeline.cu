// Constant-batch split pipeline on one GPU (e3.h).
//
// E3 runs every split on full batches and fuses the survivors of several
// upstream runs into the next split's batch ("we execute the first split
// twice ... combine the two outputs to obtain a batch size of 16",
// PAPER.md:761-766; "multiple batches are fused"; each
// split "immediately moves on to the next" batch).
//
// Host stage loop:
//   * one device ring per split s >= 1 holding its queued input rows; the
//     compaction kernel of split s-1 writes survivors straight into the ring
//     tail, so a full pop is a zero-copy pointer into the ring (a copy only
//     when the B rows wrap around the ring end, or for a padded flush);
//   * the host mirrors head (pops are host decisions) and a lower bound of
//     tail (survivor counts arrive through a host-mapped mailbox, read after
//     the run's event completes);
//   * decision for run t uses the counts of runs <= t-1-lag (lag = 1: the GPU
//     always has the previous run queued while the host decides): deepest
//     split with >= B known rows first; else wait for the outstanding run;
//     else flush the shallowest non-empty queue padded to B;
//   * every split batch has exactly B rows (padding rows never exit).
// The decision sequence is a deterministic function of the exit outcomes,
// replayed exactly by oracle/pipeline_sim.py (tests compare the traces).
#include <chrono>
#include <cstring>
#include <deque>
#include <new>
#include <vector>

#include "common.cuh"
#include "prof.h"
#include "split.h"

namespace {

constexpr int kSlots = 8;        // in-flight run bookkeeping (>= lag + 2)
constexpr int kInSlots = 4;      // host-input staging batches

struct DevQueue {
  uint8_t *rows = nullptr;
  int64_t *ids = nullptr;
  int64_t cap = 0;
  int64_t *tails = nullptr;   // device [2]: the tail alternates between two slots per push
  int64_t pushes = 0;         // pushes issued (host): push j reads slot j&1, writes slot (j+1)&1
  int64_t head = 0;    // rows popped (host decision, exact)
  int64_t known = 0;   // rows pushed by completed runs (lower bound of tail)
};

}  // namespace

struct e3_pipeline {
  e3_plan plan;
  int device = 0;
  int sms = 148;
  bool poisoned = false;
  int B = 0;
  int64_t row_bytes = 0;
  std::shared_ptr<e3::Workspace> ws;
  std::vector<e3_split *> splits;
  std::vector<DevQueue> q;            // q[s] feeds split s (q[0] unused)
  int64_t *tails = nullptr;           // device [2 * n_splits]
  int *overflow = nullptr;            // device flag
  uint8_t *staging = nullptr;         // [B, row] wrapped / flush pops
  int64_t *staging_ids = nullptr;
  uint8_t *sink = nullptr;            // [B, row] output of the last split (empty)
  int64_t *out_tails = nullptr;       // device [2]: tail slots of the caller's output buffer
  int64_t *sink_ids = nullptr;
  volatile int *mailbox = nullptr;    // host-mapped [kSlots]
  int *mailbox_dev = nullptr;
  cudaEvent_t ev[kSlots] = {};
  // host-input staging
  uint8_t *in_rows = nullptr;         // [kInSlots, B, row]
  int64_t *in_ids = nullptr;
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t in_ready[kInSlots] = {};
  cudaEvent_t in_free[kInSlots] = {};
  // trace
  std::vector<int32_t> tr_split, tr_nvalid;
  std::vector<int64_t> tr_ids;

  ~e3_pipeline() {
    cudaSetDevice(device);
    for (auto *s : splits) e3_split_destroy(s);
    for (auto &Q : q) {
      cudaFree(Q.rows);
      cudaFree(Q.ids);
    }
    cudaFree(tails);
    cudaFree(overflow);
    cudaFree(staging);
    cudaFree(staging_ids);
    cudaFree(sink);
    cudaFree(out_tails);
    cudaFree(sink_ids);
    cudaFree(in_rows);
    cudaFree(in_ids);
    if (mailbox) cudaFreeHost(const_cast<int *>(mailbox));
    for (auto &e : ev)
      if (e) cudaEventDestroy(e);
    for (int i = 0; i < kInSlots; ++i) {
      if (in_ready[i]) cudaEventDestroy(in_ready[i]);
      if (in_free[i]) cudaEventDestroy(in_free[i]);
    }
    if (copy_stream) cudaStreamDestroy(copy_stream);
  }
};

using namespace e3;

namespace {

bool is_device_ptr(const void *p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

struct Runner {
  e3_pipeline *pl;
  cudaStream_t st;
  const e3_exits *ex;
  e3_stats *stats;
  // input stream
  const uint8_t *x;
  const int64_t *ids;
  int64_t n;
  // survivors of a non-final last split (stage pipeline): caller's buffer
  uint8_t *out_rows = nullptr;
  int64_t *out_ids = nullptr;
  int64_t out_cap = 0;
  int64_t out_pushes = 0;
  int64_t out_known = 0;
  bool host_in;
  int64_t cursor = 0;      // inputs dispatched
  int64_t staged = 0;      // host inputs issued to the copy stream (batches)
  struct Pend {
    int split, slot;
  };
  std::deque<Pend> pending;
  int64_t run_no = 0;

  int64_t count(int s) const {
    if (s == 0) return n - cursor;
    return pl->q[s].known - pl->q[s].head;
  }

  e3_status apply_oldest() {
    Pend p = pending.front();
    pending.pop_front();
    const auto t0 = std::chrono::steady_clock::now();
    E3_CUDA_TRY(cudaEventSynchronize(pl->ev[p.slot]));
    if (stats) stats->host_sync_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    const int c = pl->mailbox[p.slot];
    if (c < 0) {
      set_error("survivor queue overflow (increase queue_cap_batches)");
      return E3_ECAPACITY;
    }
    if (p.split + 1 < pl->plan.n_splits) pl->q[p.split + 1].known += c;
    else out_known += c;
    prof_add_bytes(PK_COMPACT, 2.0 * c * pl->row_bytes);   // read + write of the survivors
    if (stats) stats->rows_out[p.split] += c;
    return E3_OK;
  }

  // host inputs: batch j of the input stream -> staging slot j % kInSlots
  e3_status stage_host_batch(int64_t j) {
    const int slot = (int)(j % kInSlots);
    const int64_t first = j * pl->B;
    const int64_t rows = (n - first) < pl->B ? (n - first) : pl->B;
    E3_CUDA_TRY(cudaStreamWaitEvent(pl->copy_stream, pl->in_free[slot], 0));
    uint8_t *dst = pl->in_rows + (size_t)slot * pl->B * pl->row_bytes;
    E3_CUDA_TRY(cudaMemcpyAsync(dst, x + first * pl->row_bytes, rows * pl->row_bytes, cudaMemcpyHostToDevice,
                                pl->copy_stream));
    E3_CUDA_TRY(cudaMemcpyAsync(pl->in_ids + (size_t)slot * pl->B, ids + first, rows * 8, cudaMemcpyHostToDevice,
                                pl->copy_stream));
    E3_CUDA_TRY(cudaEventRecord(pl->in_ready[slot], pl->copy_stream));
    return E3_OK;
  }

  e3_status launch(int s, int nv) {
    const int B = pl->B;
    const int64_t rb = pl->row_bytes;
    const uint8_t *xin;
    const int64_t *idin;
    int in_slot = -1;
    e3_status r;
    if (s == 0) {
      if (host_in) {
        const int64_t j = cursor / B;   // cursor is always a multiple of B here
        while (staged <= j + 1 && staged * B < n) {   // keep one batch of look-ahead in flight
          r = stage_host_batch(staged);
          if (r != E3_OK) return r;
          ++staged;
        }
        in_slot = (int)(j % kInSlots);
        E3_CUDA_TRY(cudaStreamWaitEvent(st, pl->in_ready[in_slot], 0));
        const uint8_t *src = pl->in_rows + (size_t)in_slot * B * rb;
        const int64_t *sid = pl->in_ids + (size_t)in_slot * B;
        if (nv == B) {
          xin = src;
          idin = sid;
        } else {
          ProfScope ps(PK_COPY, st, 0, 2.0 * B * rb);
          r = ring_pop_copy(src, sid, (int64_t)1 << 40, 0, nv, B, rb, pl->staging, pl->staging_ids, pl->sms, st);
          if (r != E3_OK) return r;
          xin = pl->staging;
          idin = pl->staging_ids;
        }
      } else if (nv == B) {
        xin = x + cursor * rb;
        idin = ids + cursor;
      } else {
        ProfScope ps(PK_COPY, st, 0, 2.0 * B * rb);
        r = ring_pop_copy(x + cursor * rb, ids + cursor, (int64_t)1 << 40, 0, nv, B, rb, pl->staging,
                          pl->staging_ids, pl->sms, st);
        if (r != E3_OK) return r;
        xin = pl->staging;
        idin = pl->staging_ids;
      }
      cursor += nv;
    } else {
      DevQueue &Q = pl->q[s];
      const int64_t pos = Q.head % Q.cap;
      if (nv == B && pos + B <= Q.cap) {
        xin = Q.rows + pos * rb;   // zero-copy pop
        idin = Q.ids + pos;
      } else {
        ProfScope ps(PK_COPY, st, 0, 2.0 * B * rb);
        r = ring_pop_copy(Q.rows, Q.ids, Q.cap, Q.head, nv, B, rb, pl->staging, pl->staging_ids, pl->sms, st);
        if (r != E3_OK) return r;
        xin = pl->staging;
        idin = pl->staging_ids;
      }
      Q.head += nv;
    }
    const int slot = (int)(run_no % kSlots);
    RingDst dst{};
    if (s + 1 < pl->plan.n_splits) {
      DevQueue &N = pl->q[s + 1];
      dst.rows = N.rows;
      dst.ids = N.ids;
      dst.cap = N.cap;
      dst.tail_dev = N.tails + (N.pushes & 1);
      dst.tail_out = N.tails + ((N.pushes + 1) & 1);
      ++N.pushes;
      dst.head = N.head;
    } else if (out_rows) {
      dst.rows = out_rows;
      dst.ids = out_ids;
      dst.cap = out_cap;
      dst.tail_dev = pl->out_tails + (out_pushes & 1);
      dst.tail_out = pl->out_tails + ((out_pushes + 1) & 1);
      ++out_pushes;
    } else {
      dst.rows = pl->sink;
      dst.ids = pl->sink_ids;
      dst.cap = B;
    }
    dst.overflow_dev = pl->overflow;
    dst.mailbox = pl->mailbox_dev ? reinterpret_cast<volatile int *>(pl->mailbox_dev + slot) : nullptr;
    r = split_run_to(pl->splits[s], st, xin, idin, nullptr, nv, dst, nullptr, ex);
    if (r != E3_OK) return r;
    if (in_slot >= 0) E3_CUDA_TRY(cudaEventRecord(pl->in_free[in_slot], st));
    E3_CUDA_TRY(cudaEventRecord(pl->ev[slot], st));
    if (pl->plan.trace) {
      pl->tr_split.push_back(s);
      pl->tr_nvalid.push_back(nv);
      const size_t off = pl->tr_ids.size();
      pl->tr_ids.resize(off + B);
      E3_CUDA_TRY(cudaMemcpyAsync(pl->tr_ids.data() + off, idin, (size_t)B * 8, cudaMemcpyDeviceToHost, st));
      E3_CUDA_TRY(cudaStreamSynchronize(st));
    }
    pending.push_back({s, slot});
    ++run_no;
    if (stats) {
      stats->runs++;
      stats->batches[s]++;
      stats->valid_rows[s] += nv;
      stats->padded_rows[s] += B - nv;
    }
    return E3_OK;
  }

  e3_status run() {
    const int k = pl->plan.n_splits;
    const int B = pl->B;
    const int lag = pl->plan.lag;
    e3_status r;
    for (;;) {
      while ((int)pending.size() > lag) {
        r = apply_oldest();
        if (r != E3_OK) return r;
      }
      int pick = -1;
      for (int s = k - 1; s >= 0; --s)
        if (count(s) >= B) {
          pick = s;
          break;
        }
      if (pick < 0) {
        if (!pending.empty()) {
          if (stats) stats->host_waits++;
          r = apply_oldest();
          if (r != E3_OK) return r;
          continue;
        }
        for (int s = 0; s < k; ++s)
          if (count(s) > 0) {
            pick = s;   // flush: shallowest non-empty queue, padded to B
            break;
          }
        if (pick < 0) break;   // every input has exited
      }
      const int64_t c = count(pick);
      const int nv = (int)(c >= B ? B : c);
      const auto t0 = std::chrono::steady_clock::now();
      r = launch(pick, nv);
      if (stats) stats->host_launch_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
      if (r != E3_OK) return r;
    }
    while (!pending.empty()) {
      r = apply_oldest();
      if (r != E3_OK) return r;
    }
    return E3_OK;
  }
};

}  // namespace

extern "C" {

e3_status e3_pipeline_create(const e3_plan *p, const e3_weights *w, int device, e3_pipeline **out) {
  E3_CHECK_ARG(p && w && out, "null argument");
  E3_CHECK_ARG(p->n_splits >= 1 && p->n_splits <= E3_MAX_SPLITS, "n_splits outside 1..64");
  E3_CHECK_ARG(p->lag >= 0 && p->lag <= kSlots - 2, "lag outside 0..6");
  const e3_split_desc &d0 = p->split[0];
  for (int s = 0; s < p->n_splits; ++s) {
    const e3_split_desc &d = p->split[s];
    E3_CHECK_ARG(d.hidden == d0.hidden && d.seq_len == d0.seq_len && d.ffn == d0.ffn && d.batch == d0.batch &&
                     d.heads == d0.heads && d.arch == d0.arch && d.dtype == d0.dtype,
                 "splits differ in model dims or batch");
    E3_CHECK_ARG(s == 0 || d.layer_begin == p->split[s - 1].layer_end, "splits not contiguous");
    E3_CHECK_ARG(s == p->n_splits - 1 || d.final_ramp == 0, "only the last split may hold the final ramp");
  }
  for (int s = 0; s < p->n_splits; ++s) {
    e3_status r = split_validate(&p->split[s], w);
    if (r != E3_OK) return r;
  }
  E3_CUDA_TRY(cudaSetDevice(device));
  e3_pipeline *pl = new (std::nothrow) e3_pipeline();
  if (!pl) return E3_ECUDA;
  pl->plan = *p;
  // split s is launched while queue s+1 holds < B known rows; up to `lag`
  // pending runs plus this one may each still push up to B rows
  const int min_cap = p->lag + 2 > 4 ? p->lag + 2 : 4;
  if (pl->plan.queue_cap_batches < min_cap) pl->plan.queue_cap_batches = min_cap;
  pl->device = device;
  pl->sms = num_sms(device);
  pl->B = d0.batch;
  const int elem = d0.dtype == E3_DTYPE_FP32 ? 4 : 2;
  pl->row_bytes = (int64_t)d0.seq_len * d0.hidden * elem;
  e3_status r = Workspace::create(device, d0.batch, d0.seq_len, d0.hidden, d0.ffn, elem, &pl->ws);
  for (int s = 0; s < p->n_splits && r == E3_OK; ++s) {
    e3_split *sp = nullptr;
    r = split_create_shared(&p->split[s], w, device, pl->ws, &sp);
    if (r == E3_OK) pl->splits.push_back(sp);
  }
  auto fail = [&](cudaError_t e, const char *what) {
    delete pl;
    return cuda_fail(e, what);
  };
  if (r != E3_OK) {
    delete pl;
    return r;
  }
  const int64_t cap = (int64_t)pl->plan.queue_cap_batches * pl->B;
  cudaError_t e = cudaMalloc(&pl->tails, 2 * sizeof(int64_t) * p->n_splits);
  if (e == cudaSuccess) e = cudaMemset(pl->tails, 0, 2 * sizeof(int64_t) * p->n_splits);
  if (e != cudaSuccess) return fail(e, "alloc tails");
  pl->q.resize(p->n_splits);
  for (int s = 1; s < p->n_splits; ++s) {
    DevQueue &Q = pl->q[s];
    Q.cap = cap;
    Q.tails = pl->tails + 2 * s;
    e = cudaMalloc(&Q.rows, (size_t)cap * pl->row_bytes);
    if (e == cudaSuccess) e = cudaMalloc(&Q.ids, (size_t)cap * 8);
    if (e != cudaSuccess) return fail(e, "alloc queue ring");
  }
  e = cudaMalloc(&pl->overflow, sizeof(int));
  if (e == cudaSuccess) e = cudaMemset(pl->overflow, 0, sizeof(int));
  if (e == cudaSuccess) e = cudaMalloc(&pl->staging, (size_t)pl->B * pl->row_bytes);
  if (e == cudaSuccess) e = cudaMalloc(&pl->staging_ids, (size_t)pl->B * 8);
  if (e == cudaSuccess) e = cudaMalloc(&pl->sink, (size_t)pl->B * pl->row_bytes);
  if (e == cudaSuccess) e = cudaMalloc(&pl->out_tails, 2 * sizeof(int64_t));
  if (e == cudaSuccess) e = cudaMalloc(&pl->sink_ids, (size_t)pl->B * 8);
  if (e == cudaSuccess) e = cudaMalloc(&pl->in_rows, (size_t)kInSlots * pl->B * pl->row_bytes);
  if (e == cudaSuccess) e = cudaMalloc(&pl->in_ids, (size_t)kInSlots * pl->B * 8);
  int *mb = nullptr;
  if (e == cudaSuccess) e = cudaHostAlloc(reinterpret_cast<void **>(&mb), kSlots * sizeof(int), cudaHostAllocMapped);
  if (e == cudaSuccess) {
    pl->mailbox = mb;
    e = cudaHostGetDevicePointer(reinterpret_cast<void **>(&pl->mailbox_dev), mb, 0);
  }
  for (int i = 0; i < kSlots && e == cudaSuccess; ++i) e = cudaEventCreateWithFlags(&pl->ev[i], cudaEventDisableTiming);
  for (int i = 0; i < kInSlots && e == cudaSuccess; ++i) {
    e = cudaEventCreateWithFlags(&pl->in_ready[i], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&pl->in_free[i], cudaEventDisableTiming);
  }
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&pl->copy_stream, cudaStreamNonBlocking);
  if (e != cudaSuccess) return fail(e, "e3_pipeline_create");
  *out = pl;
  return E3_OK;
}

e3_status e3_pipeline_destroy(e3_pipeline *pl) {
  delete pl;
  return E3_OK;
}

static e3_status pipeline_run_impl(e3_pipeline *pl, void *stream, const void *x, const int64_t *ids, int64_t n,
                                   const e3_exits *ex, e3_stats *st, void *x_out, int64_t *id_out, int64_t out_cap,
                                   int64_t *n_out) {
  E3_CHECK_ARG(pl, "null pipeline");
  if (pl->poisoned) {
    set_error("pipeline poisoned by an earlier failure");
    return E3_ESTATE;
  }
  E3_CHECK_ARG(n >= 0, "negative n");
  E3_CHECK_ARG(n == 0 || (x && ids), "null inputs");
  int prev = 0;
  E3_CUDA_TRY(cudaGetDevice(&prev));
  E3_CUDA_TRY(cudaSetDevice(pl->device));
  if (st) std::memset(st, 0, sizeof(*st));
  Runner R{};
  R.pl = pl;
  R.st = reinterpret_cast<cudaStream_t>(stream);
  R.ex = ex;
  R.stats = st;
  R.x = reinterpret_cast<const uint8_t *>(x);
  R.ids = ids;
  R.n = n;
  const bool xd = n > 0 && is_device_ptr(x), idd = n > 0 && is_device_ptr(ids);
  if (n > 0 && xd != idd) {
    set_error("x and ids must both be device or both be host memory");
    return E3_EINVAL;
  }
  R.host_in = n > 0 && !xd;
  const bool final_last = pl->plan.split[pl->plan.n_splits - 1].final_ramp != 0;
  if (!final_last && !x_out) {
    set_error("the plan's last split is not final: use e3_pipeline_run_out");
    return E3_EINVAL;
  }
  if (!final_last) {
    R.out_rows = reinterpret_cast<uint8_t *>(x_out);
    R.out_ids = id_out;
    R.out_cap = out_cap;
    E3_CUDA_TRY(cudaMemsetAsync(pl->out_tails, 0, 2 * sizeof(int64_t), R.st));
  }
  pl->tr_split.clear();
  pl->tr_nvalid.clear();
  pl->tr_ids.clear();
  // fresh queues for this job
  for (int s = 1; s < pl->plan.n_splits; ++s) {
    pl->q[s].head = 0;
    pl->q[s].known = 0;
    pl->q[s].pushes = 0;
  }
  E3_CUDA_TRY(cudaMemsetAsync(pl->tails, 0, 2 * sizeof(int64_t) * pl->plan.n_splits, R.st));
  if (R.host_in) {
    // the copy stream must not overwrite staging slots still read by earlier work
    for (int i = 0; i < kInSlots; ++i) E3_CUDA_TRY(cudaEventRecord(pl->in_free[i], R.st));
  }
  e3_status r = R.run();
  if (r == E3_OK) {
    int ovf = 0, derr = 0;
    E3_CUDA_TRY(cudaMemcpyAsync(&ovf, pl->overflow, sizeof(int), cudaMemcpyDeviceToHost, R.st));
    E3_CUDA_TRY(cudaMemcpyAsync(&derr, pl->ws->err, sizeof(int), cudaMemcpyDeviceToHost, R.st));
    E3_CUDA_TRY(cudaStreamSynchronize(R.st));
    if (ovf) {
      set_error("survivor queue overflow");
      r = E3_ECAPACITY;
    } else if (derr) {
      // rows whose KV slot / position lies outside the cache were skipped
      E3_CUDA_TRY(cudaMemsetAsync(pl->ws->err, 0, sizeof(int), R.st));
      set_error("a token's KV slot or position lies outside the cache (rows skipped)");
      r = E3_EINVAL;
    }
  }
  if (r == E3_ECUDA || r == E3_ECAPACITY) pl->poisoned = true;
  if (n_out) *n_out = R.out_known;
  cudaSetDevice(prev);
  return r;
}

e3_status e3_pipeline_run(e3_pipeline *pl, void *stream, const void *x, const int64_t *ids, int64_t n,
                          const e3_exits *ex, e3_stats *st) {
  return pipeline_run_impl(pl, stream, x, ids, n, ex, st, nullptr, nullptr, 0, nullptr);
}

e3_status e3_pipeline_run_out(e3_pipeline *pl, void *stream, const void *x, const int64_t *ids, int64_t n,
                              const e3_exits *ex, e3_stats *st, void *x_out, int64_t *id_out, int64_t out_cap,
                              int64_t *n_out) {
  E3_CHECK_ARG(pl && x_out && id_out && n_out && out_cap >= 0, "bad output buffer");
  E3_CHECK_ARG(pl->plan.split[pl->plan.n_splits - 1].final_ramp == 0,
               "e3_pipeline_run_out needs a plan whose last split is not final");
  E3_CHECK_ARG(((reinterpret_cast<uintptr_t>(x_out)) & 15) == 0, "x_out must be 16-byte aligned");
  return pipeline_run_impl(pl, stream, x, ids, n, ex, st, x_out, id_out, out_cap, n_out);
}



e3_status e3_pipeline_trace(e3_pipeline *pl, int32_t *split, int32_t *n_valid, int64_t *ids_out, int64_t max_runs,
                            int64_t *n_runs) {
  E3_CHECK_ARG(pl && n_runs, "null argument");
  const int64_t n = (int64_t)pl->tr_split.size();
  *n_runs = n;
  const int64_t m = n < max_runs ? n : max_runs;
  for (int64_t i = 0; i < m; ++i) {
    if (split) split[i] = pl->tr_split[i];
    if (n_valid) n_valid[i] = pl->tr_nvalid[i];
    if (ids_out) std::memcpy(ids_out + i * pl->B, pl->tr_ids.data() + i * pl->B, (size_t)pl->B * 8);
  }
  return E3_OK;
}

}  // extern "C"
