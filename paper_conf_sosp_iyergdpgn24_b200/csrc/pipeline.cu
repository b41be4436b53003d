// Constant-batch split pipeline (e3.h).
//
// E3 runs every split on full batches and fuses the survivors of several
// upstream runs into the next split's batch ("we execute the first split
// twice ... combine the two outputs to obtain a batch size of 16",
// PAPER.md:761-766; "multiple batches are fused"; each
// split "immediately moves on to the next" batch).
//
// Host stage loop of one rank:
//   * one device ring per local split s >= 1 holding its queued input rows;
//     the compaction kernel of split s-1 writes survivors straight into the
//     ring tail, so a full pop is a zero-copy pointer into the ring (a copy
//     only when the B rows wrap around the ring end, or for a padded flush);
//   * the host mirrors head (pops are host decisions) and a lower bound of
//     tail (survivor counts arrive through a host-mapped mailbox, read after
//     the run's event completes);
//   * decision for run t uses the counts of runs <= t-1-lag (lag = 1: the GPU
//     always has the previous run queued while the host decides): deepest
//     split with >= B known rows first; else wait for the outstanding run;
//     else flush the shallowest non-empty queue padded to B -- but only once
//     nothing upstream can still deliver rows;
//   * every split batch has exactly B rows (padding rows never exit).
// Multi-rank plans (e3_plan.replicas / device_of): the rank runs its STAGE
// (a contiguous range of splits).  The survivors of the stage's last split go
// to the next stage as fixed-size messages (header {n, flag} | B ids | B rows,
// written in place by the compaction kernel) over the link to receiver
// (i + k) mod r; the first split of a stage receives messages into inbox
// buffers and an append kernel (on the rank's append stream) moves the valid
// rows into its queue ring.  End of stream: an EOS message (flag 1) and
// kInbox - 1 pad messages (flag 2) per link, matching the receives the peer
// keeps posted ahead.  The host never blocks on a transfer while it has a
// run to issue; link buffers are reused only after their transfer completed.
// On one rank the decision sequence is a deterministic function of the exit
// outcomes, replayed exactly by oracle/pipeline_sim.py (tests compare traces).
#include <chrono>
#include <cstring>
#include <deque>
#include <new>
#include <thread>
#include <vector>

#include "comm.h"
#include "common.cuh"
#include "prof.h"
#include "split.h"

namespace {

constexpr int kSlots = 8;        // in-flight run bookkeeping (>= lag + 2)
constexpr int kInSlots = 4;      // host-input staging batches
constexpr int kOutSlots = 4;     // message buffers per send link
constexpr int kInbox = 2;        // message buffers (= receives posted ahead) per receive link

struct DevQueue {
  uint8_t *rows = nullptr;
  int64_t *ids = nullptr;
  int64_t cap = 0;
  int64_t *tails = nullptr;   // device [2]: the tail alternates between two slots per push
  int64_t pushes = 0;         // pushes issued (host): push j reads slot j&1, writes slot (j+1)&1
  int64_t head = 0;    // rows popped (host decision, exact)
  int64_t head_done = 0;   // rows popped by runs that have completed (ring space reusable)
  int64_t known = 0;   // rows pushed by completed runs / applied appends (lower bound of tail)
  int64_t inflight = 0;    // appends enqueued, not yet applied (<= B rows each)
};

// message = header {int32 n, int32 flag, int64 reserved} | ids [B] | rows [B]
struct MsgLayout {
  int64_t ids_off = 16, rows_off = 0, bytes = 0;
};

struct SendLink {
  std::unique_ptr<e3::Link> link;
  uint8_t *buf[kOutSlots] = {};
  cudaEvent_t ready[kOutSlots] = {};
  int64_t msg_of[kOutSlots] = {-1, -1, -1, -1};   // message in flight from the slot (-1: free)
};

struct RecvLink {
  std::unique_ptr<e3::Link> link;
  uint8_t *buf[kInbox] = {};
  cudaEvent_t appended_ev[kInbox] = {};
  // message numbers are the link's (they continue across jobs): this job's
  // first message is `base`, its inbox slot (no - base) % kInbox
  int64_t base = 0;
  int64_t appended = 0;   // appends enqueued (messages base .. appended-1)
  int64_t applied = 0;    // appends whose outcome the host has read
  int64_t eos_at = -1;    // message number of the end-of-stream message (-1: not yet)
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
  std::vector<e3_split *> splits;     // indexed by split; NULL where another rank hosts it
  int s_lo = 0, s_hi = 0;             // this rank's splits [s_lo, s_hi)
  std::vector<DevQueue> q;            // q[s] feeds split s (q[0] unused)
  int64_t *tails = nullptr;           // device [2 * n_splits]
  int *overflow = nullptr;            // device flag
  uint8_t *staging = nullptr;         // [B, row] wrapped / flush pops
  int64_t *staging_ids = nullptr;     // [2, B]: by run parity (read by the run's tail)
  uint8_t *sink = nullptr;            // [B, row] output of the last split (empty)
  int64_t *out_tails = nullptr;       // device [2]: tail slots of the caller's output buffer
  int64_t *sink_ids = nullptr;
  volatile int *mailbox = nullptr;    // host-mapped [kSlots]
  int *mailbox_dev = nullptr;
  cudaEvent_t ev[kSlots] = {};        // run done (recorded on tail_stream)
  // the last ramp + compaction of a run overlap the next run's layers
  // (split_run_to's tail stream; higher priority, so its few CTAs are placed
  // first as the layer kernels' CTAs retire)
  cudaStream_t tail_stream = nullptr;
  cudaEvent_t fork[kSlots] = {};
  cudaEvent_t joined = nullptr;
  // host-input staging
  uint8_t *in_rows = nullptr;         // [kInSlots, B, row]
  int64_t *in_ids = nullptr;
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t in_ready[kInSlots] = {};
  cudaEvent_t in_free[kInSlots] = {};
  // multi-rank
  e3_comm *comm = nullptr;            // borrowed
  int rank = 0, my_index = 0;         // replica index of this rank in its stage
  MsgLayout msg;
  std::vector<SendLink> out;          // to the next stage's replicas, in rank-list order
  std::vector<RecvLink> in;           // from the previous stage's replicas
  cudaStream_t append_stream = nullptr;
  volatile int2 *amail = nullptr;     // host-mapped [in links][kInbox] (n or -1, flag)
  int2 *amail_dev = nullptr;
  int64_t sent_data = 0;              // data messages sent (routing counter)
  // trace
  std::vector<int32_t> tr_split, tr_nvalid;
  std::vector<int64_t> tr_ids;

  ~e3_pipeline() {
    cudaSetDevice(device);
    cudaDeviceSynchronize();
    for (auto *s : splits)
      if (s) e3_split_destroy(s);
    for (auto &Q : q) {
      cudaFree(Q.rows);
      cudaFree(Q.ids);
    }
    for (auto &L : out)
      for (int i = 0; i < kOutSlots; ++i) {
        cudaFree(L.buf[i]);
        if (L.ready[i]) cudaEventDestroy(L.ready[i]);
      }
    for (auto &L : in)
      for (int i = 0; i < kInbox; ++i) {
        cudaFree(L.buf[i]);
        if (L.appended_ev[i]) cudaEventDestroy(L.appended_ev[i]);
      }
    out.clear();
    in.clear();
    if (amail) cudaFreeHost(const_cast<int2 *>(amail));
    if (append_stream) cudaStreamDestroy(append_stream);
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
    for (auto &e : fork)
      if (e) cudaEventDestroy(e);
    if (joined) cudaEventDestroy(joined);
    if (tail_stream) cudaStreamDestroy(tail_stream);
  }
};

namespace e3 {
// ---- inbox -> queue ring (append stream) ---------------------------------
__global__ void inbox_copy_kernel(const uint8_t *__restrict__ msg, int64_t ids_off, int64_t rows_off, int64_t vpr,
                                  RingDst dst) {
  const int n = *reinterpret_cast<const int *>(msg);
  const int flag = *reinterpret_cast<const int *>(msg + 4);
  if (flag != 0 || n <= 0) return;
  const int64_t tail = *dst.tail_dev;
  if ((tail - dst.head) + n > dst.cap) return;   // overflow: reported by the finish kernel
  const uint4 *src = reinterpret_cast<const uint4 *>(msg + rows_off);
  uint4 *ring = reinterpret_cast<uint4 *>(dst.rows);
  const int64_t total = (int64_t)n * vpr;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < total; v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t k = v / vpr, off = v - k * vpr;
    ring[((tail + k) % dst.cap) * vpr + off] = src[v];
  }
  if (blockIdx.x == 0) {
    const int64_t *ids = reinterpret_cast<const int64_t *>(msg + ids_off);
    for (int k = threadIdx.x; k < n; k += blockDim.x) dst.ids[(tail + k) % dst.cap] = ids[k];
  }
}

__global__ void inbox_finish_kernel(const uint8_t *__restrict__ msg, RingDst dst, int2 *mail) {
  const int n = *reinterpret_cast<const int *>(msg);
  const int flag = *reinterpret_cast<const int *>(msg + 4);
  const int64_t tail = *dst.tail_dev;
  const bool data = flag == 0 && n > 0;
  const bool fits = !data || (tail - dst.head) + n <= dst.cap;
  *dst.tail_out = (data && fits) ? tail + n : tail;
  if (!fits && dst.overflow_dev) *dst.overflow_dev = 1;
  int2 m;
  m.x = !fits ? -1 : (flag == 0 ? n : 0);
  m.y = flag;
  reinterpret_cast<volatile int *>(mail)[1] = m.y;
  reinterpret_cast<volatile int *>(mail)[0] = m.x;
  __threadfence_system();
}

}  // namespace e3

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

double comm_timeout_s() {
  static const double t = [] {
    const char *e = getenv("E3_COMM_TIMEOUT_S");
    return e ? atof(e) : 600.0;
  }();
  return t;
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
  // survivors of a non-final last split (single rank): caller's buffer
  uint8_t *out_rows = nullptr;
  int64_t *out_ids = nullptr;
  int64_t out_cap = 0;
  int64_t out_pushes = 0;
  int64_t out_known = 0;
  bool host_in;
  int64_t cursor = 0;      // inputs dispatched
  int64_t staged = 0;      // host inputs issued to the copy stream (batches)
  struct Pend {
    int split, slot, nv;
  };
  std::deque<Pend> pending;
  int64_t run_no = 0;
  int rr = 0;              // deterministic mode: the receive link whose message is appended next
  std::chrono::steady_clock::time_point last_progress = std::chrono::steady_clock::now();

  int64_t count(int s) const {
    if (s == 0) return n - cursor;
    return pl->q[s].known - pl->q[s].head;
  }

  bool upstream_done() const {   // nothing can still arrive from another rank
    for (const auto &R : pl->in)
      if (R.eos_at < 0) return false;
    return true;
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
    if (p.split > 0) pl->q[p.split].head_done += p.nv;
    if (p.split + 1 < pl->s_hi) pl->q[p.split + 1].known += c;
    else out_known += c;
    prof_add_bytes(PK_COMPACT, 2.0 * c * pl->row_bytes);   // read + write of the survivors
    if (stats) stats->rows_out[p.split] += c;
    last_progress = std::chrono::steady_clock::now();
    return E3_OK;
  }

  // ---- receive links: apply finished appends, enqueue new ones, re-post
  // receives.  Non-blocking; *progress = something changed.
  e3_status service_in(bool *progress) {
    const int s = pl->s_lo;
    DevQueue &Q = pl->q[s];
    const int nl = (int)pl->in.size();
    const bool det = pl->plan.deterministic != 0;
    for (int i = 0; i < nl; ++i) {
      RecvLink &R = pl->in[i];
      while (R.applied < R.appended) {
        const int slot = (int)((R.applied - R.base) % kInbox);
        const cudaError_t qe = cudaEventQuery(R.appended_ev[slot]);
        if (qe == cudaErrorNotReady) {
          cudaGetLastError();
          break;
        }
        E3_CUDA_TRY(qe);
        const volatile int *mp = reinterpret_cast<const volatile int *>(pl->amail + i * kInbox + slot);
        const int2 m = make_int2(mp[0], mp[1]);
        const int64_t no = R.applied++;
        --Q.inflight;
        *progress = true;
        if (m.x < 0) {
          set_error("survivor queue overflow on a received batch (increase queue_cap_batches)");
          return E3_ECAPACITY;
        }
        if (m.y == 0) {
          Q.known += m.x;
          if (stats) stats->msgs_recv++;
          if (R.eos_at < 0 && R.link->posted == no + kInbox) {   // keep kInbox receives ahead
            e3_status r = R.link->post(R.buf[slot], (size_t)pl->msg.bytes, nullptr);
            if (r != E3_OK) return r;
          }
          if (det && i == rr) rr = next_rr(rr);
        } else if (m.y == 1) {
          R.eos_at = no;
          if (det && i == rr) rr = next_rr(rr);
        }
      }
      if (R.eos_at >= 0) continue;
      if (det && i != rr) continue;
      while (R.appended < R.link->posted && R.appended - R.applied < (det ? 1 : kInbox)) {
        if ((Q.known + (Q.inflight + 1) * pl->B) - Q.head_done > Q.cap) break;   // ring room for one batch
        bool done = false;
        cudaEvent_t rev = nullptr;
        e3_status r = R.link->query(R.appended, &done, &rev);
        if (r != E3_OK) return r;
        if (!done) break;
        const int slot = (int)((R.appended - R.base) % kInbox);
        E3_CUDA_TRY(cudaStreamWaitEvent(pl->append_stream, rev, 0));
        RingDst dst{};
        dst.rows = Q.rows;
        dst.ids = Q.ids;
        dst.cap = Q.cap;
        dst.tail_dev = Q.tails + (Q.pushes & 1);
        dst.tail_out = Q.tails + ((Q.pushes + 1) & 1);
        ++Q.pushes;
        dst.head = Q.head_done;
        dst.overflow_dev = pl->overflow;
        const int64_t vpr = pl->row_bytes / 16;
        const int grid = (int)std::min<int64_t>(2 * pl->sms, (pl->B * vpr + 255) / 256);
        inbox_copy_kernel<<<grid > 0 ? grid : 1, 256, 0, pl->append_stream>>>(R.buf[slot], pl->msg.ids_off,
                                                                                pl->msg.rows_off, vpr, dst);
        E3_CUDA_TRY(cudaGetLastError());
        inbox_finish_kernel<<<1, 1, 0, pl->append_stream>>>(R.buf[slot], dst, pl->amail_dev + i * kInbox + slot);
        E3_CUDA_TRY(cudaGetLastError());
        count_launch();
        count_launch();
        E3_CUDA_TRY(cudaEventRecord(R.appended_ev[slot], pl->append_stream));
        ++R.appended;
        ++Q.inflight;
        *progress = true;
      }
    }
    if (*progress) last_progress = std::chrono::steady_clock::now();
    return E3_OK;
  }

  int next_rr(int cur) const {
    const int nl = (int)pl->in.size();
    for (int k = 1; k <= nl; ++k) {
      const int j = (cur + k) % nl;
      if (pl->in[j].eos_at < 0) return j;
    }
    return cur;
  }

  e3_status service(bool *progress) {
    *progress = false;
    if (pl->in.empty()) return E3_OK;
    return service_in(progress);
  }

  // nothing to issue: poll the links until something changes (watchdog)
  e3_status wait_progress() {
    for (;;) {
      bool p = false;
      e3_status r = service(&p);
      if (r != E3_OK) return r;
      if (p) return E3_OK;
      r = check_links();
      if (r != E3_OK) return r;
      std::this_thread::yield();
    }
  }

  e3_status check_links() {
    for (auto &L : pl->out) {
      e3_status r = L.link->check_async();
      if (r != E3_OK) return r;
    }
    for (auto &R : pl->in) {
      e3_status r = R.link->check_async();
      if (r != E3_OK) return r;
    }
    const double idle = std::chrono::duration<double>(std::chrono::steady_clock::now() - last_progress).count();
    if (idle > comm_timeout_s()) {
      std::string m = "inter-stage transfer made no progress for E3_COMM_TIMEOUT_S seconds (rank " +
                      std::to_string(pl->rank) + ", splits [" + std::to_string(pl->s_lo) + "," +
                      std::to_string(pl->s_hi) + "), pending runs " + std::to_string(pending.size());
      for (size_t i = 0; i < pl->in.size(); ++i) {
        const RecvLink &R = pl->in[i];
        m += "; in[" + std::to_string(i) + "] posted " + std::to_string(R.link->posted) + " appended " +
             std::to_string(R.appended) + " applied " + std::to_string(R.applied) + " eos " + std::to_string(R.eos_at);
      }
      for (size_t i = 0; i < pl->out.size(); ++i) {
        m += "; out[" + std::to_string(i) + "] posted " + std::to_string(pl->out[i].link->posted) + " in flight";
        for (int k = 0; k < kOutSlots; ++k) m += " " + std::to_string(pl->out[i].msg_of[k]);
      }
      if (pl->s_lo > 0 && pl->s_lo < (int)pl->q.size()) {
        const DevQueue &Q = pl->q[pl->s_lo];
        m += "; q[s_lo] known " + std::to_string(Q.known) + " head " + std::to_string(Q.head) + " head_done " +
             std::to_string(Q.head_done) + " inflight " + std::to_string(Q.inflight) + " cap " + std::to_string(Q.cap);
      }
      set_error(m + ")");
      return E3_ENCCL;
    }
    return E3_OK;
  }

  // a free message buffer on send link L (waits, servicing receives, while
  // every buffer's transfer is still in flight)
  e3_status acquire_slot(SendLink &L, int *slot) {
    for (;;) {
      for (int i = 0; i < kOutSlots; ++i) {
        if (L.msg_of[i] < 0) {
          *slot = i;
          return E3_OK;
        }
        bool done = false;
        e3_status r = L.link->query(L.msg_of[i], &done, nullptr);
        if (r != E3_OK) return r;
        if (done) {
          L.msg_of[i] = -1;
          *slot = i;
          last_progress = std::chrono::steady_clock::now();
          return E3_OK;
        }
      }
      bool p = false;
      e3_status r = service(&p);
      if (r == E3_OK) r = check_links();
      if (r != E3_OK) return r;
      std::this_thread::yield();
    }
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
    const int par = (int)(run_no & 1);
    const int slot = (int)(run_no % kSlots);
    int64_t *const stg_ids = pl->staging_ids + (size_t)par * B;   // read until the run's tail ends
    cudaStream_t tst = prof_enabled() ? st : pl->tail_stream;   // profiled step: serial, clean intervals
    if (run_no >= 2)   // run_no - 2's tail still reads the parity buffers this run writes
      E3_CUDA_TRY(cudaStreamWaitEvent(st, pl->ev[(run_no - 2) % kSlots], 0));
    // destination of the survivors first (a send link may have to free a buffer)
    RingDst dst{};
    SendLink *SL = nullptr;
    int out_slot = -1;
    if (s + 1 < pl->s_hi) {
      DevQueue &N = pl->q[s + 1];
      dst.rows = N.rows;
      dst.ids = N.ids;
      dst.cap = N.cap;
      dst.tail_dev = N.tails + (N.pushes & 1);
      dst.tail_out = N.tails + ((N.pushes + 1) & 1);
      ++N.pushes;
      dst.head = N.head_done;
    } else if (!pl->out.empty()) {
      SL = &pl->out[(size_t)((pl->my_index + pl->sent_data) % (int64_t)pl->out.size())];
      r = acquire_slot(*SL, &out_slot);
      if (r != E3_OK) return r;
      uint8_t *m = SL->buf[out_slot];
      E3_CUDA_TRY(cudaMemsetAsync(m, 0, 16, st));   // n (written by the compaction), flag 0
      dst.rows = m + pl->msg.rows_off;
      dst.ids = reinterpret_cast<int64_t *>(m + pl->msg.ids_off);
      dst.cap = B;
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
          r = ring_pop_copy(src, sid, (int64_t)1 << 40, 0, nv, B, rb, pl->staging, stg_ids, pl->sms, st);
          if (r != E3_OK) return r;
          xin = pl->staging;
          idin = stg_ids;
        }
      } else if (nv == B) {
        xin = x + cursor * rb;
        idin = ids + cursor;
      } else {
        ProfScope ps(PK_COPY, st, 0, 2.0 * B * rb);
        r = ring_pop_copy(x + cursor * rb, ids + cursor, (int64_t)1 << 40, 0, nv, B, rb, pl->staging,
                          stg_ids, pl->sms, st);
        if (r != E3_OK) return r;
        xin = pl->staging;
        idin = stg_ids;
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
        r = ring_pop_copy(Q.rows, Q.ids, Q.cap, Q.head, nv, B, rb, pl->staging, stg_ids, pl->sms, st);
        if (r != E3_OK) return r;
        xin = pl->staging;
        idin = stg_ids;
      }
      Q.head += nv;
    }
    dst.overflow_dev = pl->overflow;
    dst.mailbox = pl->mailbox_dev ? reinterpret_cast<volatile int *>(pl->mailbox_dev + slot) : nullptr;
    int32_t *n_surv_dev = SL ? reinterpret_cast<int32_t *>(SL->buf[out_slot]) : nullptr;
    r = split_run_to(pl->splits[s], st, xin, idin, nullptr, nv, dst, n_surv_dev, ex, tst, par, pl->fork[slot]);
    if (r != E3_OK) return r;
    // the run ends on the tail stream (its ids are read there)
    if (in_slot >= 0) E3_CUDA_TRY(cudaEventRecord(pl->in_free[in_slot], tst));
    E3_CUDA_TRY(cudaEventRecord(pl->ev[slot], tst));
    if (SL) {   // ship the message once the run has written it
      E3_CUDA_TRY(cudaEventRecord(SL->ready[out_slot], tst));
      r = SL->link->post(SL->buf[out_slot], (size_t)pl->msg.bytes, SL->ready[out_slot]);
      if (r != E3_OK) return r;
      SL->msg_of[out_slot] = SL->link->posted - 1;
      ++pl->sent_data;
      if (stats) stats->msgs_sent++;
    }
    if (pl->plan.trace) {
      pl->tr_split.push_back(s);
      pl->tr_nvalid.push_back(nv);
      const size_t off = pl->tr_ids.size();
      pl->tr_ids.resize(off + B);
      E3_CUDA_TRY(cudaMemcpyAsync(pl->tr_ids.data() + off, idin, (size_t)B * 8, cudaMemcpyDeviceToHost, st));
      E3_CUDA_TRY(cudaStreamSynchronize(st));
    }
    pending.push_back({s, slot, nv});
    ++run_no;
    if (stats) {
      stats->runs++;
      stats->batches[s]++;
      stats->valid_rows[s] += nv;
      stats->padded_rows[s] += B - nv;
      if (nv < B) stats->flushes[s]++;
    }
    return E3_OK;
  }

  // end of stream on every send link: EOS, then kInbox - 1 pads (the
  // receives the peer keeps posted beyond its last data message)
  e3_status finish_out() {
    for (auto &L : pl->out) {
      for (int k = 0; k < kInbox; ++k) {
        int slot = -1;
        e3_status r = acquire_slot(L, &slot);
        if (r != E3_OK) return r;
        const int hdr[4] = {0, k == 0 ? 1 : 2, 0, 0};
        E3_CUDA_TRY(cudaMemcpyAsync(L.buf[slot], hdr, sizeof hdr, cudaMemcpyHostToDevice, st));
        E3_CUDA_TRY(cudaEventRecord(L.ready[slot], st));
        r = L.link->post(L.buf[slot], (size_t)pl->msg.bytes, L.ready[slot]);
        if (r != E3_OK) return r;
        L.msg_of[slot] = L.link->posted - 1;
      }
    }
    for (auto &L : pl->out)   // every transfer of this rank completed
      for (int i = 0; i < kOutSlots; ++i)
        while (L.msg_of[i] >= 0) {
          bool done = false;
          e3_status r = L.link->query(L.msg_of[i], &done, nullptr);
          if (r == E3_OK && !done) r = check_links();
          if (r != E3_OK) return r;
          if (done) L.msg_of[i] = -1;
          else std::this_thread::yield();
        }
    return E3_OK;
  }

  // the receives posted beyond each EOS (the pads) must land before return
  e3_status finish_in() {
    for (auto &R : pl->in)
      for (int64_t m = R.applied; m < R.link->posted; ++m)
        for (;;) {
          bool done = false;
          e3_status r = R.link->query(m, &done, nullptr);
          if (r == E3_OK && !done) r = check_links();
          if (r != E3_OK) return r;
          if (done) break;
          std::this_thread::yield();
        }
    if (pl->append_stream) E3_CUDA_TRY(cudaStreamSynchronize(pl->append_stream));
    return E3_OK;
  }

  e3_status run() {
    const int lo = pl->s_lo, hi = pl->s_hi;
    const int B = pl->B;
    const int lag = pl->plan.lag;
    e3_status r;
    for (auto &R : pl->in)   // kInbox receives ahead on every link
      for (int k = 0; k < kInbox; ++k) {
        r = R.link->post(R.buf[k], (size_t)pl->msg.bytes, nullptr);
        if (r != E3_OK) return r;
      }
    for (;;) {
      bool p = false;
      r = service(&p);
      if (r != E3_OK) return r;
      while ((int)pending.size() > lag) {
        r = apply_oldest();
        if (r != E3_OK) return r;
      }
      int pick = -1;
      for (int s = hi - 1; s >= lo; --s)
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
        if (!upstream_done()) {   // rows may still arrive from the previous stage
          r = wait_progress();
          if (r != E3_OK) return r;
          continue;
        }
        for (int s = lo; s < hi; ++s)
          if (count(s) > 0) {
            pick = s;   // flush: shallowest non-empty queue, padded to B
            break;
          }
        if (pick < 0) break;   // every input has exited or left this stage
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
    r = finish_out();
    if (r == E3_OK) r = finish_in();
    return r;
  }
};

// Stages of a multi-rank plan: maximal runs of consecutive splits with the
// same replica rank list.
struct Stage {
  int lo, hi;
  std::vector<int> ranks;
};

e3_status plan_stages(const e3_plan *p, int world, std::vector<Stage> *stages) {
  int off = 0;
  std::vector<std::vector<int>> ranks(p->n_splits);
  for (int s = 0; s < p->n_splits; ++s) {
    const int r = p->replicas[s];
    E3_CHECK_ARG(r >= 1 && off + r <= E3_MAX_REPLICA_SLOTS, "replicas[s] must be >= 1 (sum <= 256)");
    for (int j = 0; j < r; ++j) {
      const int d = p->device_of[off + j];
      E3_CHECK_ARG(d >= 0 && d < world, "device_of outside the communicator");
      for (int k : ranks[s]) E3_CHECK_ARG(k != d, "a split has two replicas on one rank");
      ranks[s].push_back(d);
    }
    off += r;
  }
  stages->clear();
  for (int s = 0; s < p->n_splits; ++s) {
    if (!stages->empty() && stages->back().ranks == ranks[s]) {
      stages->back().hi = s + 1;
      continue;
    }
    stages->push_back({s, s + 1, ranks[s]});
  }
  for (size_t g = 0; g < stages->size(); ++g)
    for (size_t h = 0; h < g; ++h)
      for (int a : (*stages)[g].ranks)
        for (int b : (*stages)[h].ranks)
          E3_CHECK_ARG(a != b, "a rank hosts two non-adjacent split ranges (stages must use disjoint ranks)");
  return E3_OK;
}

}  // namespace

extern "C" {

e3_status e3_pipeline_create(const e3_plan *p, const e3_weights *w, int device, e3_comm *comm,
                             e3_pipeline **out) {
  E3_CHECK_ARG(p && w && out, "null argument");
  E3_CHECK_ARG(p->n_splits >= 1 && p->n_splits <= E3_MAX_SPLITS, "n_splits outside 1..64");
  E3_CHECK_ARG(p->lag >= 0 && p->lag <= kSlots - 2, "lag outside 0..6");
  const e3_split_desc &d0 = p->split[0];
  for (int s = 0; s < p->n_splits; ++s) {
    const e3_split_desc &d = p->split[s];
    E3_CHECK_ARG(d.hidden == d0.hidden && d.seq_len == d0.seq_len && d.ffn == d0.ffn && d.batch == d0.batch &&
                     d.heads == d0.heads && d.arch == d0.arch && d.dtype == d0.dtype,
                 "splits differ in model dims, batch or dtype");
    E3_CHECK_ARG(s == 0 || d.layer_begin == p->split[s - 1].layer_end, "splits not contiguous");
    E3_CHECK_ARG(s == p->n_splits - 1 || d.final_ramp == 0, "only the last split may hold the final ramp");
  }
  bool multi = false;
  for (int s = 0; s < p->n_splits; ++s) multi = multi || p->replicas[s] != 0;
  const int world = comm ? comm_world(comm) : 1, rank = comm ? comm_rank(comm) : 0;
  std::vector<Stage> stages;
  int my_stage = 0;
  if (multi) {
    E3_CHECK_ARG(comm, "a plan with replicas / device_of needs a communicator");
    E3_CHECK_ARG(comm_device(comm) == device, "device differs from the communicator's device");
    E3_CHECK_ARG(p->split[p->n_splits - 1].final_ramp == 1, "a multi-rank plan must end in the model's final ramp");
    E3_CHECK_ARG(p->transport == E3_TRANSPORT_NCCL || p->transport == E3_TRANSPORT_LOOPBACK ||
                     p->transport == E3_TRANSPORT_P2P,
                 "bad transport");
    if (p->transport == E3_TRANSPORT_P2P) {
      set_error("e3_pipeline_create: transport P2P is not implemented (use NCCL or LOOPBACK)");
      return E3_EUNSUPPORTED;
    }
    E3_CHECK_ARG(p->transport == comm_transport(comm), "plan transport differs from the communicator's");
    for (int s = 0; s < p->n_splits; ++s)
      if (p->split[s].test == E3_TEST_PATIENCE) {
        set_error("e3_pipeline_create: dependent exits (E3_TEST_PATIENCE) keep per-input state in the caller's "
                  "e3_exits.state: single-rank plans only");
        return E3_EUNSUPPORTED;
      }
    e3_status r = plan_stages(p, world, &stages);
    if (r != E3_OK) return r;
    my_stage = -1;
    for (size_t g = 0; g < stages.size(); ++g)
      for (int k : stages[g].ranks)
        if (k == rank) my_stage = (int)g;
  } else {
    stages.push_back({0, p->n_splits, {rank}});
  }
  const bool idle = my_stage < 0;
  const int lo = idle ? 0 : stages[my_stage].lo, hi = idle ? 0 : stages[my_stage].hi;
  for (int s = lo; s < hi; ++s) {
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
  pl->comm = comm;
  pl->rank = rank;
  pl->s_lo = lo;
  pl->s_hi = hi;
  pl->splits.assign(p->n_splits, nullptr);
  const int elem = d0.dtype == E3_DTYPE_FP32 ? 4 : 2;
  pl->row_bytes = (int64_t)d0.seq_len * d0.hidden * elem;
  auto fail = [&](cudaError_t e, const char *what) {
    delete pl;
    return cuda_fail(e, what);
  };
  auto fail_r = [&](e3_status r) {
    delete pl;
    return r;
  };
  // links first: NCCL link communicators are collective over the world
  if (multi) {
    const int64_t idb = ((int64_t)pl->B * 8 + 15) / 16 * 16;
    pl->msg.ids_off = 16;
    pl->msg.rows_off = 16 + idb;
    pl->msg.bytes = pl->msg.rows_off + (int64_t)pl->B * pl->row_bytes;
    int color = 0;
    for (size_t g = 0; g + 1 < stages.size(); ++g)
      for (size_t i = 0; i < stages[g].ranks.size(); ++i)
        for (size_t j = 0; j < stages[g + 1].ranks.size(); ++j, ++color) {
          const int a = stages[g].ranks[i], b = stages[g + 1].ranks[j];
          const bool member = rank == a || rank == b;
          std::unique_ptr<Link> L;
          e3_status r = comm_make_link(comm, color, member, rank == a, rank == a ? b : a, &L);
          if (r != E3_OK) return fail_r(r);
          if (!member) continue;
          if (rank == a) {
            pl->out.emplace_back();
            pl->out.back().link = std::move(L);
          } else {
            pl->in.emplace_back();
            pl->in.back().link = std::move(L);
          }
        }
    if (!idle)
      for (size_t i = 0; i < stages[my_stage].ranks.size(); ++i)
        if (stages[my_stage].ranks[i] == rank) pl->my_index = (int)i;
  }
  if (idle) {
    *out = pl;
    return E3_OK;
  }
  e3_status r = Workspace::create(device, d0.batch, d0.seq_len, d0.hidden, d0.ffn, elem, &pl->ws);
  for (int s = lo; s < hi && r == E3_OK; ++s) {
    e3_split *sp = nullptr;
    r = split_create_shared(&p->split[s], w, device, pl->ws, &sp);
    if (r == E3_OK) pl->splits[s] = sp;
  }
  if (r != E3_OK) return fail_r(r);
  cudaError_t e = cudaMalloc(&pl->tails, 2 * sizeof(int64_t) * p->n_splits);
  if (e == cudaSuccess) e = cudaMemset(pl->tails, 0, 2 * sizeof(int64_t) * p->n_splits);
  if (e != cudaSuccess) return fail(e, "alloc tails");
  pl->q.resize(p->n_splits);
  for (int s = (lo > 0 ? lo : 1); s < hi; ++s) {
    DevQueue &Q = pl->q[s];
    int64_t batches = pl->plan.queue_cap_batches;
    if (s == lo) batches += (int64_t)kInbox * (int64_t)pl->in.size() + 2;   // appends in flight
    Q.cap = batches * pl->B;
    Q.tails = pl->tails + 2 * s;
    e = cudaMalloc(&Q.rows, (size_t)Q.cap * pl->row_bytes);
    if (e == cudaSuccess) e = cudaMalloc(&Q.ids, (size_t)Q.cap * 8);
    if (e != cudaSuccess) return fail(e, "alloc queue ring");
  }
  for (auto &L : pl->out)
    for (int i = 0; i < kOutSlots && e == cudaSuccess; ++i) {
      e = cudaMalloc(&L.buf[i], (size_t)pl->msg.bytes);
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(&L.ready[i], cudaEventDisableTiming);
    }
  for (auto &R : pl->in)
    for (int i = 0; i < kInbox && e == cudaSuccess; ++i) {
      e = cudaMalloc(&R.buf[i], (size_t)pl->msg.bytes);
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(&R.appended_ev[i], cudaEventDisableTiming);
    }
  if (e == cudaSuccess && !pl->in.empty()) {
    e = cudaStreamCreateWithFlags(&pl->append_stream, cudaStreamNonBlocking);
    int2 *am = nullptr;
    if (e == cudaSuccess)
      e = cudaHostAlloc(reinterpret_cast<void **>(&am), pl->in.size() * kInbox * sizeof(int2), cudaHostAllocMapped);
    if (e == cudaSuccess) {
      pl->amail = am;
      e = cudaHostGetDevicePointer(reinterpret_cast<void **>(&pl->amail_dev), am, 0);
    }
  }
  if (e != cudaSuccess) return fail(e, "alloc link buffers");
  e = cudaMalloc(&pl->overflow, sizeof(int));
  if (e == cudaSuccess) e = cudaMemset(pl->overflow, 0, sizeof(int));
  if (e == cudaSuccess) e = cudaMalloc(&pl->staging, (size_t)pl->B * pl->row_bytes);
  if (e == cudaSuccess) e = cudaMalloc(&pl->staging_ids, 2 * (size_t)pl->B * 8);
  if (e == cudaSuccess) e = cudaMalloc(&pl->sink, (size_t)pl->B * pl->row_bytes);
  if (e == cudaSuccess) e = cudaMalloc(&pl->out_tails, 2 * sizeof(int64_t));
  if (e == cudaSuccess) e = cudaMalloc(&pl->sink_ids, (size_t)pl->B * 8);
  if (lo == 0) {
    if (e == cudaSuccess) e = cudaMalloc(&pl->in_rows, (size_t)kInSlots * pl->B * pl->row_bytes);
    if (e == cudaSuccess) e = cudaMalloc(&pl->in_ids, (size_t)kInSlots * pl->B * 8);
  }
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
  int prio_lo = 0, prio_hi = 0;
  if (e == cudaSuccess) e = cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
  static const bool tail_lo = getenv("E3_TAIL_PRIO_LOW") != nullptr;   // diagnostics: tail at the main stream's priority
  if (e == cudaSuccess)
    e = cudaStreamCreateWithPriority(&pl->tail_stream, cudaStreamNonBlocking, tail_lo ? prio_lo : prio_hi);
  for (int i = 0; i < kSlots && e == cudaSuccess; ++i)
    e = cudaEventCreateWithFlags(&pl->fork[i], cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&pl->joined, cudaEventDisableTiming);
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
  E3_CHECK_ARG(n == 0 || pl->s_lo == 0, "only ranks hosting split 0 take inputs");
  if (st) std::memset(st, 0, sizeof(*st));
  if (pl->s_hi == 0) {   // this rank hosts no split of the plan
    if (n_out) *n_out = 0;
    return E3_OK;
  }
  int prev = 0;
  E3_CUDA_TRY(cudaGetDevice(&prev));
  E3_CUDA_TRY(cudaSetDevice(pl->device));
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
  const bool final_last = pl->plan.split[pl->s_hi - 1].final_ramp != 0 || !pl->out.empty();
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
  // fresh queues and links for this job (a job is one stream of inputs)
  for (auto &Q : pl->q) {
    Q.head = Q.head_done = Q.known = Q.pushes = Q.inflight = 0;
  }
  for (auto &L : pl->out)
    for (auto &m : L.msg_of) m = -1;
  for (auto &Rl : pl->in) {
    Rl.base = Rl.appended = Rl.applied = Rl.link->posted;
    Rl.eos_at = -1;
  }
  pl->sent_data = 0;
  E3_CUDA_TRY(cudaStreamWaitEvent(R.st, pl->joined, 0));   // the previous job's tails (any stream)
  E3_CUDA_TRY(cudaMemsetAsync(pl->tails, 0, 2 * sizeof(int64_t) * pl->plan.n_splits, R.st));
  E3_CUDA_TRY(cudaStreamSynchronize(R.st));   // tails reset before any append-stream work
  if (R.host_in) {
    // the copy stream must not overwrite staging slots still read by earlier work
    for (int i = 0; i < kInSlots; ++i) E3_CUDA_TRY(cudaEventRecord(pl->in_free[i], R.st));
  }
  e3_status r = R.run();
  {   // join: the caller's stream waits for the last tails
    const cudaError_t je = cudaEventRecord(pl->joined, pl->tail_stream);
    if (je == cudaSuccess) cudaStreamWaitEvent(R.st, pl->joined, 0);
    if (je != cudaSuccess && r == E3_OK) {
      set_error("join of the tail stream failed");
      r = E3_ECUDA;
    }
  }
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
  if (r == E3_ECUDA || r == E3_ECAPACITY || r == E3_ENCCL) pl->poisoned = true;
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
  E3_CHECK_ARG(pl->out.empty() && pl->in.empty(), "e3_pipeline_run_out is for single-rank plans");
  E3_CHECK_ARG(pl->plan.split[pl->plan.n_splits - 1].final_ramp == 0,
               "e3_pipeline_run_out needs a plan whose last split is not final");
  E3_CHECK_ARG(((reinterpret_cast<uintptr_t>(x_out)) & 15) == 0, "x_out must be 16-byte aligned");
  return pipeline_run_impl(pl, stream, x, ids, n, ex, st, x_out, id_out, out_cap, n_out);
}

e3_status e3_decode_run(e3_pipeline *pl, void *stream, void *x, const int64_t *ids, int64_t n, int32_t steps,
                        const void *embed, int32_t *tokens_out, const e3_exits *ex, e3_stats *st) {
  E3_CHECK_ARG(pl && ex && x && ids && embed && n > 0 && steps >= 0, "bad arguments");
  if (pl->poisoned) {
    set_error("pipeline poisoned by an earlier failure");
    return E3_ESTATE;
  }
  const e3_split_desc &d0 = pl->plan.split[0];
  E3_CHECK_ARG(d0.arch == E3_ARCH_LLAMA_DECODE, "e3_decode_run needs a LLAMA_DECODE plan");
  E3_CHECK_ARG(pl->s_lo == 0 && pl->s_hi == pl->plan.n_splits && pl->in.empty() && pl->out.empty(),
               "e3_decode_run: every split on this rank (the fill needs every layer)");
  E3_CHECK_ARG(pl->plan.split[pl->plan.n_splits - 1].final_ramp, "the plan must end in the model's final ramp");
  E3_CHECK_ARG(ex->hidden && ex->exit_layer && ex->label, "e3_decode_run needs ex->hidden, exit_layer and label");
  E3_CHECK_ARG(is_device_ptr(x) && is_device_ptr(ids) && is_device_ptr(embed), "x, ids, embed must be device memory");
  cudaStream_t cs = reinterpret_cast<cudaStream_t>(stream);
  const e3_split *s0 = pl->splits[0];
  if (st) std::memset(st, 0, sizeof(*st));
  const int elem = d0.dtype == E3_DTYPE_FP32 ? 4 : 2;
  for (int step = 0; step < steps; ++step) {
    e3_stats sst;
    e3_status r = e3_pipeline_run(pl, stream, x, ids, n, ex, &sst);
    if (r != E3_OK) return r;
    if (st) {
      st->runs += sst.runs;
      for (int s = 0; s < pl->plan.n_splits; ++s) {
        st->batches[s] += sst.batches[s];
        st->valid_rows[s] += sst.valid_rows[s];
        st->padded_rows[s] += sst.padded_rows[s];
        st->rows_out[s] += sst.rows_out[s];
        st->flushes[s] += sst.flushes[s];
      }
      st->host_waits += sst.host_waits;
      st->host_launch_ms += sst.host_launch_ms;
      st->host_sync_ms += sst.host_sync_ms;
    }
    E3_CUDA_TRY(cudaSetDevice(pl->device));
    // K/V of the skipped layers, chunk by chunk of B tokens (layer 0 is never skipped)
    for (int64_t c0 = 0; c0 < n; c0 += pl->B) {
      const int nv = (int)std::min<int64_t>(pl->B, n - c0);
      for (int s = 0; s < pl->plan.n_splits; ++s) {
        const e3_split_desc &d = pl->plan.split[s];
        for (int l = std::max(1, d.layer_begin); l < d.layer_end; ++l) {
          r = llama_fill_layer(pl->splits[s], l, cs, ids + c0, nv, *ex, pl->staging_ids);
          if (r != E3_OK) {
            if (r == E3_ECUDA) pl->poisoned = true;
            return r;
          }
        }
      }
    }
    r = decode_advance_run(ids, n, ex->label, ex->capacity, tokens_out ? tokens_out + (int64_t)step * n : nullptr,
                           embed, d0.num_labels, (int64_t)d0.hidden * elem, x, s0->kv.slot_of_id,
                           const_cast<int32_t *>(s0->kv.pos_of_slot), s0->kv.n_slots, pl->ws->err, cs);
    if (r != E3_OK) return r;
    int derr = 0;
    E3_CUDA_TRY(cudaMemcpyAsync(&derr, pl->ws->err, sizeof(int), cudaMemcpyDeviceToHost, cs));
    E3_CUDA_TRY(cudaStreamSynchronize(cs));
    if (derr) {
      E3_CUDA_TRY(cudaMemsetAsync(pl->ws->err, 0, sizeof(int), cs));
      set_error("e3_decode_run: a token's slot, position or label lies outside the cache / vocabulary");
      return E3_EINVAL;
    }
  }
  return E3_OK;
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
