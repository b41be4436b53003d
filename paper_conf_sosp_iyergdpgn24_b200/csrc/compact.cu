// Stable survivor compaction and the queue ring
// copies of the re-batching engine (a5, K6).
//
// Compaction: pos = exclusive_scan(alive), x_out[pos[i]] = x[i] for alive i,
// order preserved ("the overhead associated with reforming a batch after
// certain samples exit").  Every CTA recomputes the scan of
// the B flags itself (B <= 4096: warp __ballot_sync + __popc per 32 flags, a
// serial scan over <= 128 words), so no grid-wide sync is needed; the CTAs
// then split the n_surv * row_bytes gather into equal contiguous ranges of
// 16-byte vectors with 4 independent loads in flight per thread.  Output goes
// either to a contiguous buffer or straight into the next split's queue ring
// (wrapping at row granularity), which makes the later pop zero-copy.  The CTA
// that retires last publishes n_surv (device + host-mapped mailbox) and
// advances the ring tail.
#include "common.cuh"
#include "kernels.h"
#include "ln_row.cuh"
#include "prof.h"

namespace e3 {

namespace {

constexpr int kMaxB = 4096;
constexpr int kThreads = 256;
constexpr int kUnroll = 4;

__device__ __forceinline__ int block_scan_flags(const uint8_t *alive, int B, int16_t *src_of, int *word_cnt,
                                                int16_t *pos_of = nullptr) {
  // word_cnt: [kMaxB/32 + 1] smem
  const int warp = warp_id(), lane = lane_id();
  const int nwords = (B + 31) / 32;
  for (int w = warp; w < nwords; w += kThreads / 32) {
    const int i = w * 32 + lane;
    const unsigned bal = __ballot_sync(0xffffffffu, i < B && alive[i] != 0);
    if (lane == 0) word_cnt[w] = __popc(bal);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int run = 0;
    for (int w = 0; w < nwords; ++w) {
      const int c = word_cnt[w];
      word_cnt[w] = run;
      run += c;
    }
    word_cnt[nwords] = run;
  }
  __syncthreads();
  for (int w = warp; w < nwords; w += kThreads / 32) {
    const int i = w * 32 + lane;
    const bool f = i < B && alive[i] != 0;
    const unsigned bal = __ballot_sync(0xffffffffu, f);
    const int pos = word_cnt[w] + __popc(bal & ((1u << lane) - 1u));
    if (f) src_of[pos] = (int16_t)i;
    if (pos_of && i < B) pos_of[i] = f ? (int16_t)pos : (int16_t)-1;
  }
  __syncthreads();
  return word_cnt[nwords];
}

__global__ void __launch_bounds__(kThreads)
    compact_kernel(const uint8_t *__restrict__ x, const int64_t *__restrict__ id, const uint8_t *__restrict__ alive,
                   int B, int64_t row_bytes, RingDst dst, int32_t *n_surv_dev, unsigned *done_ctr) {
  __shared__ int16_t src_of[kMaxB];
  __shared__ int word_cnt[kMaxB / 32 + 1];
  __shared__ bool is_last;
  const int n = block_scan_flags(alive, B, src_of, word_cnt);
  const int64_t tail = dst.tail_dev ? *(volatile int64_t *)dst.tail_dev : 0;
  const bool fits = (tail - dst.head) + n <= dst.cap;

  if (fits && n > 0) {
    const int64_t vpr = row_bytes / 16;                     // vectors per row
    const int64_t total = (int64_t)n * vpr;
    const int64_t per = (total + gridDim.x - 1) / gridDim.x;
    const int64_t beg = (int64_t)blockIdx.x * per;
    const int64_t end = beg + per < total ? beg + per : total;
    const uint4 *src = reinterpret_cast<const uint4 *>(x);
    uint4 *ring = reinterpret_cast<uint4 *>(dst.rows);
    // walk the CTA's range row segment by row segment (no per-vector division)
    for (int64_t v = beg; v < end;) {
      const int64_t k = v / vpr;
      const int64_t off0 = v - k * vpr;
      const int64_t seg_end = (k + 1) * vpr < end ? (k + 1) * vpr : end;
      const int len = (int)(seg_end - v);
      const uint4 *s_row = src + (int64_t)src_of[k] * vpr + off0;
      uint4 *d_row = ring + ((tail + k) % dst.cap) * vpr + off0;
      for (int i0 = threadIdx.x; i0 < len; i0 += kThreads * kUnroll) {
        uint4 buf[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          const int i = i0 + u * kThreads;
          if (i < len) buf[u] = __ldcs(s_row + i);
        }
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          const int i = i0 + u * kThreads;
          if (i < len) d_row[i] = buf[u];
        }
      }
      v = seg_end;
    }
    if (blockIdx.x == 0)
      for (int k = threadIdx.x; k < n; k += kThreads) dst.ids[(tail + k) % dst.cap] = id[src_of[k]];
  }

  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned t = atomicAdd(done_ctr, 1u);
    is_last = (t == gridDim.x - 1);
  }
  __syncthreads();
  if (is_last && threadIdx.x == 0) {
    *done_ctr = 0;
    const int out = fits ? n : 0;
    if (!fits && dst.overflow_dev) *dst.overflow_dev = 1;
    if (dst.tail_dev) {   // next tail into the queue's other slot when given (as ln_compact)
      if (dst.tail_out) *(volatile int64_t *)dst.tail_out = fits ? tail + n : tail;
      else if (fits) *(volatile int64_t *)dst.tail_dev = tail + n;
    }
    if (n_surv_dev) *n_surv_dev = out;
    if (dst.mailbox) {
      *dst.mailbox = fits ? out : -1;
      __threadfence_system();
    }
  }
}

// rows [head, head+n) of the ring -> dst rows [0, n); rows [n, B) zero, ids -1.
// grid (chunks of a row, B rows)
__global__ void __launch_bounds__(kThreads)
    ring_pop_kernel(const uint4 *__restrict__ ring, const int64_t *__restrict__ ring_ids, int64_t cap, int64_t head,
                    int n, int B, int64_t vpr, uint4 *__restrict__ out, int64_t *__restrict__ out_ids) {
  const int k = blockIdx.y;
  const int64_t i0 = (int64_t)blockIdx.x * kThreads * kUnroll + threadIdx.x;
  const uint4 *s_row = ring + ((head + k) % cap) * vpr;
  uint4 *d_row = out + (int64_t)k * vpr;
#pragma unroll
  for (int u = 0; u < kUnroll; ++u) {
    const int64_t i = i0 + u * kThreads;
    if (i < vpr) d_row[i] = (k < n) ? s_row[i] : make_uint4(0, 0, 0, 0);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) out_ids[k] = (k < n) ? ring_ids[(head + k) % cap] : -1;
}

// device-count push: rows [0, *n_dev) appended at *tail_dev; grid (chunks, max_rows)
__global__ void __launch_bounds__(kThreads)
    ring_push_kernel(const uint4 *__restrict__ rows, const int64_t *__restrict__ ids, const int32_t *n_dev,
                     uint4 *__restrict__ ring, int64_t *__restrict__ ring_ids, int64_t cap, const int64_t *tail_dev,
                     const int64_t *head_dev, int64_t vpr) {
  const int n = *n_dev;
  const int k = blockIdx.y;
  if (k >= n) return;
  const int64_t tail = *tail_dev, head = *head_dev;
  if ((tail - head) + n > cap) return;   // flagged by ring_push_finish
  const int64_t i0 = (int64_t)blockIdx.x * kThreads * kUnroll + threadIdx.x;
  const uint4 *s_row = rows + (int64_t)k * vpr;
  uint4 *d_row = ring + ((tail + k) % cap) * vpr;
#pragma unroll
  for (int u = 0; u < kUnroll; ++u) {
    const int64_t i = i0 + u * kThreads;
    if (i < vpr) d_row[i] = s_row[i];
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) ring_ids[(tail + k) % cap] = ids[k];
}

__global__ void ring_push_finish(const int32_t *n_dev, int64_t *tail_dev, const int64_t *head_dev, int64_t cap,
                                 int *overflow_dev) {
  const int n = *n_dev;
  if ((*tail_dev - *head_dev) + n > cap) {
    *overflow_dev = 1;
  } else {
    *tail_dev += n;
  }
}

__global__ void fill_kernel(int32_t *dst, int v) { *dst = v; }

// Fused LN2 + compaction of a split's last layer: survivors' token rows are
// read PRE-LayerNorm (y = residual sum), normalised (ln_row.cuh, bit-identical
// to layernorm_kernel and to the ramp's CLS rows) and written straight into
// the destination (next split's queue ring or a contiguous buffer).  Rows that
// exited are never normalised or written.  One warp per token row, kRowsInFlight
// rows' loads in flight per warp.  No grid-wide ticket: every CTA derives the
// same survivor count from the flags, CTA 0 publishes it (n_surv, host
// mailbox, overflow flag) and writes the queue's NEXT tail slot (dst.tail_out)
// while everyone reads the current one (dst.tail_dev) -- the two slots
// alternate per push, chosen by the host.
constexpr int kRowsInFlight = 4;

// two CTAs per SM where the row fits in <= 3 vectors per lane: with one
// (160 registers) only 8 warps x 4 rows were in flight per SM and the gather
// was latency-bound (r01 timeline: ~7 us for 22 MB of L2-resident rows)
template <int VPL, bool kLn>
__global__ void __launch_bounds__(kThreads, VPL <= 3 ? 2 : 1)
    ln_compact_kernel(const __nv_bfloat16 *__restrict__ y, const int64_t *__restrict__ id,
                      const uint8_t *__restrict__ alive, int B, int S, int H, const __nv_bfloat16 *__restrict__ g,
                      const __nv_bfloat16 *__restrict__ bb, float eps, RingDst dst, int32_t *n_surv_dev) {
  __shared__ int16_t src_of[kMaxB];
  __shared__ int16_t pos_of[kMaxB];
  __shared__ int word_cnt[kMaxB / 32 + 1];
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  const int warp = warp_id(), lane = lane_id();
  LnParams<VPL> p;
  if (kLn) ln_load_params<VPL>(p, g, bb, H, lane);   // weights: before the dependency wait
  pdl_wait();
  pdl_trigger();
  const unsigned long long tl1 = tl_now();
  const int stride = gridDim.x * (kThreads / 32);
  const int all_units = B * S;
  // One pass over the SOURCE rows when every row has a slot (BB: 8192 rows,
  // 2 x 148 CTAs x 8 warps x 4): the row loads are issued before the scan of
  // the alive flags, LayerNorm runs on them, and only survivors are stored at
  // their compacted position -- the load latency overlaps the scan instead of
  // following it (exiting rows are read and normalised for nothing, <= B S H 2
  // bytes of L2 traffic).  Otherwise survivors are gathered by destination.
  const bool spec = all_units <= kRowsInFlight * stride;
  uint4 v[kRowsInFlight][VPL];
  if (spec) {
#pragma unroll
    for (int j = 0; j < kRowsInFlight; ++j) {
      const int u = blockIdx.x * (kThreads / 32) + warp + j * stride;
      if (u < all_units) ln_load_row<VPL>(v[j], y + (size_t)u * H, H, lane);
    }
  }
  const int64_t tail = dst.tail_dev ? *dst.tail_dev : 0;
  const int n = block_scan_flags(alive, B, src_of, word_cnt, pos_of);
  if (threadIdx.x == 0) tl_rec(tlb, 60, tl1, tl1);   // scan done
  const bool fits = (tail - dst.head) + n <= dst.cap;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    const int out = fits ? n : 0;
    if (!fits && dst.overflow_dev) *dst.overflow_dev = 1;
    if (dst.tail_out) *dst.tail_out = fits ? tail + n : tail;
    if (n_surv_dev) *n_surv_dev = out;
    if (dst.mailbox) *dst.mailbox = fits ? out : -1;   // read by the host after the run's event
  }
  if (!fits || n == 0) {
    if (threadIdx.x == 0) tl_rec(tlb, 6, tl0, tl1);
    return;
  }

  const int units = n * S;
  __nv_bfloat16 *ring = reinterpret_cast<__nv_bfloat16 *>(dst.rows);
  const size_t row_elems = (size_t)S * H;
  if (spec) {
#pragma unroll
    for (int j = 0; j < kRowsInFlight; ++j) {
      const int u = blockIdx.x * (kThreads / 32) + warp + j * stride;
      if (u < all_units) {
        const int b = u / S, t = u - b * S;
        const int k = pos_of[b];
        if (k >= 0) {
          if (kLn) ln_apply<VPL>(v[j], p, H, eps, lane);
          ln_store_row<VPL>(v[j], ring + ((tail + k) % dst.cap) * row_elems + (size_t)t * H, H, lane);
        }
      }
    }
  }
  // gather by destination, software-pipelined: the rows are walked in
  // batches of kRowsInFlight / 2 and the next batch's loads are issued before
  // the current batch is normalised and stored, so every warp always has
  // loads in flight (VT, 50 k token rows per run: the load -> store -> load
  // rhythm of whole batches left the HBM idle between them)
  if (!spec && kLn) {   // LayerNorm-ing gathers: batches of kRowsInFlight (the pipelined form spills here)
    for (int u0 = blockIdx.x * (kThreads / 32) + warp; u0 < units; u0 += kRowsInFlight * stride) {
#pragma unroll
      for (int j = 0; j < kRowsInFlight; ++j) {
        const int u = u0 + j * stride;
        if (u < units) {
          const int k = u / S, t = u - k * S;
          ln_load_row<VPL>(v[j], y + (size_t)src_of[k] * row_elems + (size_t)t * H, H, lane);
        }
      }
#pragma unroll
      for (int j = 0; j < kRowsInFlight; ++j) {
        const int u = u0 + j * stride;
        if (u < units) {
          const int k = u / S, t = u - k * S;
          ln_apply<VPL>(v[j], p, H, eps, lane);
          ln_store_row<VPL>(v[j], ring + ((tail + k) % dst.cap) * row_elems + (size_t)t * H, H, lane);
        }
      }
    }
  } else if (!spec) {
    constexpr int HB = kRowsInFlight / 2;
    auto load_batch = [&](int u0, int half) {
#pragma unroll
      for (int j = 0; j < HB; ++j) {
        const int u = u0 + j * stride;
        if (u < units) {
          const int k = u / S, t = u - k * S;
          ln_load_row<VPL>(v[half * HB + j], y + (size_t)src_of[k] * row_elems + (size_t)t * H, H, lane);
        }
      }
    };
    auto store_batch = [&](int u0, int half) {
#pragma unroll
      for (int j = 0; j < HB; ++j) {
        const int u = u0 + j * stride;
        if (u < units) {
          const int k = u / S, t = u - k * S;
          if (kLn) ln_apply<VPL>(v[half * HB + j], p, H, eps, lane);
          ln_store_row<VPL>(v[half * HB + j], ring + ((tail + k) % dst.cap) * row_elems + (size_t)t * H, H, lane);
        }
      }
    };
    int u0 = blockIdx.x * (kThreads / 32) + warp;
    if (u0 < units) load_batch(u0, 0);
    while (u0 < units) {   // two batches per trip: the register halves stay compile-time indices
      if (u0 + HB * stride < units) load_batch(u0 + HB * stride, 1);
      store_batch(u0, 0);
      u0 += HB * stride;
      if (u0 >= units) break;
      if (u0 + HB * stride < units) load_batch(u0 + HB * stride, 0);
      store_batch(u0, 1);
      u0 += HB * stride;
    }
  }
  if (blockIdx.x == 0)
    for (int k = threadIdx.x; k < n; k += kThreads) dst.ids[(tail + k) % dst.cap] = id[src_of[k]];
  if (threadIdx.x == 0) tl_rec(tlb, 6, tl0, tl1);
}

}  // namespace

E3_TL_SETTER(tl_set_compact)

e3_status ln_compact_run(const void *y, const int64_t *id, const uint8_t *alive, int B, int S, int H, const void *g,
                         const void *b, float eps, const RingDst &dst, int32_t *n_surv_dev, int sms,
                         cudaStream_t st) {
  if (B > kMaxB || H % 8 || H > 4096) {
    set_error("ln_compact: need B <= 4096, H % 8 == 0, H <= 4096");
    return E3_EUNSUPPORTED;
  }
  // kRowsInFlight token rows per warp on a full batch, but never more CTAs
  // than are resident at once: a second wave would repeat the whole latency
  // chain (scan, loads, stores) -- 4 waves cost 12.8 us at BB (r01 ncu)
  int64_t grid = ((int64_t)B * S + 8 * kRowsInFlight - 1) / (8 * kRowsInFlight);
  auto *yp = reinterpret_cast<const __nv_bfloat16 *>(y);
  auto *gp = reinterpret_cast<const __nv_bfloat16 *>(g);
  auto *bp = reinterpret_cast<const __nv_bfloat16 *>(b);
  const int vpl = (H / 8 + 31) / 32;
  static const int cap_env = [] {   // diagnostics: E3_COMPACT_GRID caps the CTAs
    const char *e = getenv("E3_COMPACT_GRID");
    return e ? atoi(e) : 0;
  }();
#define E3_LNC(V)                                                                                          \
  do {                                                                                                     \
    auto kern = gp ? ln_compact_kernel<V, true> : ln_compact_kernel<V, false>;                             \
    static int occ_[2] = {0, 0};                                                                           \
    int &occ = occ_[gp ? 1 : 0];                                                                           \
    if (!occ) E3_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kThreads, 0));        \
    if (occ < 1) occ = 1;                                                                                  \
    if (grid > (int64_t)occ * sms) grid = (int64_t)occ * sms;                                              \
    if (cap_env > 0 && grid > cap_env) grid = cap_env;                                                     \
    if (grid < 1) grid = 1;                                                                                \
    E3_CUDA_TRY(launch_k(kern, dim3((unsigned)grid), dim3(kThreads), 0, st, yp, id, alive, B, S, H, gp, bp, \
                         eps, dst, n_surv_dev));                                                           \
  } while (0)
  if (vpl <= 1) E3_LNC(1);
  else if (vpl <= 3) E3_LNC(3);
  else if (vpl <= 4) E3_LNC(4);
  else if (vpl <= 8) E3_LNC(8);
  else E3_LNC(16);
#undef E3_LNC
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status compact_run(const void *x, const int64_t *id, const uint8_t *alive, int B, int64_t row_bytes,
                      const RingDst &dst, int32_t *n_surv_dev, unsigned *done_ctr, int sms, cudaStream_t st) {
  if (B > kMaxB || row_bytes % 16) {
    set_error("compact: need B <= 4096 and row_bytes % 16 == 0");
    return E3_EUNSUPPORTED;
  }
  // enough CTAs to keep >= ~32 KB in flight per SM on a full batch
  const int64_t bytes = (int64_t)B * row_bytes;
  int64_t grid = bytes / (32 * 1024);
  if (grid > 2 * sms) grid = 2 * sms;
  if (grid < 1) grid = 1;
  compact_kernel<<<(int)grid, kThreads, 0, st>>>(reinterpret_cast<const uint8_t *>(x), id, alive, B, row_bytes, dst,
                                                 n_surv_dev, done_ctr);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status ring_pop_copy(const uint8_t *ring, const int64_t *ring_ids, int64_t cap, int64_t head, int n, int B,
                        int64_t row_bytes, void *dst, int64_t *dst_ids, int sms, cudaStream_t st) {
  (void)sms;
  const int64_t vpr = row_bytes / 16;
  dim3 grid((unsigned)((vpr + kThreads * kUnroll - 1) / (kThreads * kUnroll)), (unsigned)B);
  ring_pop_kernel<<<grid, kThreads, 0, st>>>(reinterpret_cast<const uint4 *>(ring), ring_ids, cap, head, n, B, vpr,
                                             reinterpret_cast<uint4 *>(dst), dst_ids);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status ring_push_copy(const void *rows, const int64_t *ids, const int32_t *n_dev, int max_rows, uint8_t *ring,
                         int64_t *ring_ids, int64_t cap, int64_t *tail_dev, const int64_t *head_dev,
                         int *overflow_dev, int64_t row_bytes, cudaStream_t st) {
  const int64_t vpr = row_bytes / 16;
  if (max_rows > 0) {
    dim3 grid((unsigned)((vpr + kThreads * kUnroll - 1) / (kThreads * kUnroll)), (unsigned)max_rows);
    ring_push_kernel<<<grid, kThreads, 0, st>>>(reinterpret_cast<const uint4 *>(rows), ids, n_dev,
                                                reinterpret_cast<uint4 *>(ring), ring_ids, cap, tail_dev, head_dev,
                                                vpr);
    E3_CUDA_TRY(cudaGetLastError());
    count_launch();
  }
  ring_push_finish<<<1, 1, 0, st>>>(n_dev, tail_dev, head_dev, cap, overflow_dev);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status fill_valid(int32_t *dst, int value, cudaStream_t st) {
  fill_kernel<<<1, 1, 0, st>>>(dst, value);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace e3
