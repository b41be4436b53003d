// LLaMA decode helpers of the split path (DESIGN.md §6
// K8): RMSNorm, single-query attention over the KV cache, and the LM-head
// ramp's decision.  The GEMMs of the decode layer are gemm_dec.cu.
//
//   rmsnorm_kernel   warp per token row: y = bf16(x / sqrt(mean x^2 + eps) * g)
//   attn_dec_kernel  one CTA per (head, token), 8 warps: q from the QKV
//                    epilogue (RoPE applied), keys/values of the token's slot
//                    at positions 0..pos (the new one written by the same
//                    epilogue); every key / value row is one coalesced
//                    256-byte warp load, 8 keys per warp step reduced with 9
//                    shuffles;
//                    scores fp32, p = exp(s - max) unrounded, out = bf16(p V / l)
//                    -- HBM-bound on the cache stream (537 MB per Llama-7B
//                    layer at 64 tokens x 513 positions)
//   lm_decide_kernel warp per row: merges the LM-head tiles' softmax
//                    statistics in tile order (softstat.cuh), max-prob /
//                    entropy, strict threshold, exit record, alive flag --
//                    the same semantics as the encoder ramps (the logits
//                    were written to the records by the LM-head epilogue).
#include "common.cuh"
#include "exitrule.cuh"
#include "kernels.h"
#include "prof.h"
#include "softstat.cuh"

namespace e3 {

namespace {

template <int VPL>
__global__ void __launch_bounds__(256) rmsnorm_kernel(const __nv_bfloat16 *__restrict__ x,
                                                      const __nv_bfloat16 *__restrict__ g,
                                                      __nv_bfloat16 *__restrict__ y, int rows, int H, float eps) {
  const int warp = warp_id(), lane = lane_id();
  const int row = blockIdx.x * 8 + warp;
  const int nvec = H / 8;
  uint4 gv[VPL];
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int k = lane + 32 * i;
    gv[i] = (k < nvec) ? __ldg(reinterpret_cast<const uint4 *>(g) + k) : make_uint4(0, 0, 0, 0);
  }
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  pdl_wait();
  pdl_trigger();
  const unsigned long long tl1 = tl_now();
  if (row >= rows) return;
  const uint4 *xr = reinterpret_cast<const uint4 *>(x + (size_t)row * H);
  uint4 v[VPL];
  float ss = 0.f;
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int k = lane + 32 * i;
    v[i] = (k < nvec) ? xr[k] : make_uint4(0, 0, 0, 0);
    const uint32_t w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
#pragma unroll
    for (int e = 0; e < 4; ++e) ss += bf_lo(w[e]) * bf_lo(w[e]) + bf_hi(w[e]) * bf_hi(w[e]);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) ss += __shfl_xor_sync(0xffffffffu, ss, o);
  const float rinv = 1.0f / sqrtf(ss / (float)H + eps);
  uint4 *yr = reinterpret_cast<uint4 *>(y + (size_t)row * H);
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int k = lane + 32 * i;
    if (k >= nvec) continue;
    const uint32_t w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
    const uint32_t gw[4] = {gv[i].x, gv[i].y, gv[i].z, gv[i].w};
    uint32_t o[4];
#pragma unroll
    for (int e = 0; e < 4; ++e)
      o[e] = pack_bf16(bf_lo(w[e]) * rinv * bf_lo(gw[e]), bf_hi(w[e]) * rinv * bf_hi(gw[e]));
    yr[k] = make_uint4(o[0], o[1], o[2], o[3]);
  }
  if (threadIdx.x == 0) tl_rec(tlb, 8700, tl0, tl1);
}

constexpr int kAttnThreads = 256;
constexpr int kAW = kAttnThreads / 32;   // warps
constexpr int kHd = 128;                 // head_dim
constexpr int kKeysPerStep = 8;          // keys per warp per step (one 256-B row each)

__device__ __forceinline__ float block_reduce(float v, float *red, bool is_max) {
  const int warp = warp_id(), lane = lane_id();
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    const float w = __shfl_xor_sync(0xffffffffu, v, o);
    v = is_max ? fmaxf(v, w) : v + w;
  }
  __syncthreads();   // red[] free
  if (lane == 0) red[warp] = v;
  __syncthreads();
  float r = red[0];
#pragma unroll
  for (int w = 1; w < kAW; ++w) r = is_max ? fmaxf(r, red[w]) : r + red[w];
  return r;
}

// 8 per-lane partial dot products -> lane L holds the full sum of key
// ((L>>4)&1)*4 + ((L>>3)&1)*2 + ((L>>2)&1)  (9 shuffles for 8 keys)
__device__ __forceinline__ float reduce8(float (&v)[8], int lane) {
  const bool b16 = lane & 16, b8 = lane & 8, b4 = lane & 4;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const float send = b16 ? v[i] : v[i + 4], keep = b16 ? v[i + 4] : v[i];
    v[i] = keep + __shfl_xor_sync(0xffffffffu, send, 16);
  }
#pragma unroll
  for (int i = 0; i < 2; ++i) {
    const float send = b8 ? v[i] : v[i + 2], keep = b8 ? v[i + 2] : v[i];
    v[i] = keep + __shfl_xor_sync(0xffffffffu, send, 8);
  }
  {
    const float send = b4 ? v[0] : v[1], keep = b4 ? v[1] : v[0];
    v[0] = keep + __shfl_xor_sync(0xffffffffu, send, 4);
  }
  v[0] += __shfl_xor_sync(0xffffffffu, v[0], 2);
  v[0] += __shfl_xor_sync(0xffffffffu, v[0], 1);
  return v[0];
}

// (kAttnThreads, 5): <= 48 registers, five CTAs per SM instead of four
// (61 registers): 2048 (head, token) CTAs in 2.8 waves instead of 3.5;
// LM 11.19 -> 11.39 k tokens/s, attention 0.87 -> 0.91 of HBM (six per SM
// spilled and measured 10.59 k)
__global__ void __launch_bounds__(kAttnThreads, 5)
    attn_dec_kernel(const __nv_bfloat16 *__restrict__ q, __nv_bfloat16 *__restrict__ ctx,
                    const __nv_bfloat16 *__restrict__ kc, const __nv_bfloat16 *__restrict__ vc,
                    const int64_t *__restrict__ ids, const int32_t *n_valid_dev, int n_valid_host,
                    const int32_t *__restrict__ slot_of_id, int64_t id_cap, const int32_t *__restrict__ pos_of_slot,
                    int n_slots, int nh, int kvh, int max_ctx, float scale) {
  extern __shared__ float sp[];                 // [max_ctx] scores / probabilities
  __shared__ float red[kAW];
  __shared__ float4 sacc[kAW][32];
  const int h = blockIdx.x, t = blockIdx.y;
  const int tid = threadIdx.x, warp = warp_id(), lane = lane_id();
  const int H = nh * kHd;
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  pdl_wait();
  pdl_trigger();
  const unsigned long long tl1 = tl_now();
  const int nv = n_valid_dev ? *n_valid_dev : n_valid_host;
  const int64_t id = ids[t];
  __nv_bfloat16 *out = ctx + (size_t)t * H + h * kHd;
  if (t >= nv || id < 0 || id >= id_cap) {     // padding row: finite zeros
    if (tid < kHd / 4) reinterpret_cast<uint2 *>(out)[tid] = make_uint2(0u, 0u);
    return;
  }
  const int slot = slot_of_id[id];
  const int pos = (slot >= 0 && slot < n_slots) ? pos_of_slot[slot] : -1;
  if (pos < 0 || pos >= max_ctx) {             // outside the cache (flagged by the QKV epilogue)
    if (tid < kHd / 4) reinterpret_cast<uint2 *>(out)[tid] = make_uint2(0u, 0u);
    return;
  }
  const int L = pos + 1;
  const int g = h / (nh / kvh);
  // lane owns dims 4*lane .. 4*lane+3 of q, of every key and every value row
  const uint2 qv = reinterpret_cast<const uint2 *>(q + (size_t)t * H + h * kHd)[lane];
  const float q0 = bf_lo(qv.x) * scale, q1 = bf_hi(qv.x) * scale, q2 = bf_lo(qv.y) * scale,
              q3 = bf_hi(qv.y) * scale;
  const size_t base = ((size_t)slot * kvh + g) * max_ctx * kHd;
  const uint2 *K = reinterpret_cast<const uint2 *>(kc + base) + lane;   // + j * 32 for key j
  // ---- scores: warp w takes keys [8s, 8s+8) for s = w, w + 8, ...; each key
  // row is one coalesced 256-byte warp load
  float lmax = -INFINITY;
  constexpr int kG = 2;                         // groups of kKeysPerStep keys in flight per warp step
  for (int j0 = warp * kG * kKeysPerStep; j0 < L; j0 += kAW * kG * kKeysPerStep) {
    uint2 kv[kG][kKeysPerStep];
#pragma unroll
    for (int gi = 0; gi < kG; ++gi)
#pragma unroll
      for (int i = 0; i < kKeysPerStep; ++i) {
        const int j = j0 + gi * kKeysPerStep + i;
        kv[gi][i] = (j < L) ? K[(size_t)j * (kHd / 4)] : make_uint2(0u, 0u);
      }
#pragma unroll
    for (int gi = 0; gi < kG; ++gi) {
      float d[kKeysPerStep];
#pragma unroll
      for (int i = 0; i < kKeysPerStep; ++i)
        d[i] = fmaf(q0, bf_lo(kv[gi][i].x),
                    fmaf(q1, bf_hi(kv[gi][i].x), fmaf(q2, bf_lo(kv[gi][i].y), q3 * bf_hi(kv[gi][i].y))));
      const float sc = reduce8(d, lane);
      const int k = ((lane >> 4) & 1) * 4 + ((lane >> 3) & 1) * 2 + ((lane >> 2) & 1);
      const int jj = j0 + gi * kKeysPerStep + k;
      if ((lane & 3) == 0 && jj < L) {
        sp[jj] = sc;
        lmax = fmaxf(lmax, sc);
      }
    }
  }
  const float m = block_reduce(lmax, red, true);
  float lsum = 0.f;
  for (int j = tid; j < L; j += kAttnThreads) {
    const float e = expf(sp[j] - m);
    sp[j] = e;
    lsum += e;
  }
  const float l = block_reduce(lsum, red, false);   // also orders the sp[] writes
  // ---- P V: warp w takes positions j = w mod 8, lane owns dims 4*lane .. +3
  const uint2 *V = reinterpret_cast<const uint2 *>(vc + base) + lane;
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll 16
  for (int j = warp; j < L; j += kAW) {
    const uint2 vv = V[(size_t)j * (kHd / 4)];
    const float p = sp[j];
    acc.x = fmaf(p, bf_lo(vv.x), acc.x);
    acc.y = fmaf(p, bf_hi(vv.x), acc.y);
    acc.z = fmaf(p, bf_lo(vv.y), acc.z);
    acc.w = fmaf(p, bf_hi(vv.y), acc.w);
  }
  sacc[warp][lane] = acc;
  __syncthreads();
  if (warp == 0) {
    float4 s4 = sacc[0][lane];
#pragma unroll
    for (int w = 1; w < kAW; ++w) {
      s4.x += sacc[w][lane].x;
      s4.y += sacc[w][lane].y;
      s4.z += sacc[w][lane].z;
      s4.w += sacc[w][lane].w;
    }
    const float il = 1.0f / l;
    uint2 o;
    o.x = pack_bf16(s4.x * il, s4.y * il);
    o.y = pack_bf16(s4.z * il, s4.w * il);
    reinterpret_cast<uint2 *>(out)[lane] = o;
  }
  if (tid == 0) tl_rec(tlb, 8600, tl0, tl1);
}

__global__ void __launch_bounds__(128) lm_decide_kernel(RampArgs a) {
  const int warp = warp_id(), lane = lane_id();
  const int b = blockIdx.x * 4 + warp;
  pdl_wait();
  pdl_trigger();
  if (b >= a.B) return;
  const int nv = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  const bool ok = b < nv && (a.init_alive || a.alive[b] != 0);
  if (!ok) {
    if (lane == 0 && a.init_alive) a.alive[b] = 0;
    return;
  }
  SoftStat st{-INFINITY, 0.f, 0.f, -1};
  for (int i = lane; i < a.lm_tiles; i += 32) {    // tile order within the lane
    const float4 v = a.lm_stats[(size_t)i * a.B + b];
    st = soft_merge(st, SoftStat{v.x, v.y, v.z, __float_as_int(v.w)});
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) st = soft_merge(st, soft_shfl_xor(st, o));
  float metric;
  bool pass;
  if (a.test == E3_TEST_PATIENCE) {   // one state update per row (lane 0), then broadcast
    if (lane == 0) pass = patience_step(a.ex.state, a.id[b], a.ex.capacity, st.idx, a.tau, &metric);
    pass = __shfl_sync(0xffffffffu, pass, 0);
    metric = __shfl_sync(0xffffffffu, metric, 0);
  } else if (a.test == E3_TEST_MAXPROB) {
    metric = 1.0f / st.s;
    pass = metric > a.tau;
  } else {
    metric = logf(st.s) - st.u / st.s;
    pass = metric < a.tau;
  }
  const bool exit_now = pass || a.final_ramp;
  if (lane == 0 && a.ex.ramp_metric && a.id[b] >= 0 && a.id[b] < a.ex.capacity)
    a.ex.ramp_metric[a.id[b] * a.ex.ramp_metric_stride + a.ramp_index] = metric;
  const int64_t id = a.id[b];
  if (exit_now && id >= 0 && id < a.ex.capacity) {
    if (lane == 0) {
      if (a.ex.exit_layer) a.ex.exit_layer[id] = a.layer;
      if (a.ex.label) a.ex.label[id] = st.idx;
      if (a.ex.conf) a.ex.conf[id] = metric;
    }
    if (a.ex.hidden && a.x) {   // the row it exits with (multi-step decode fills skipped layers' K/V from it)
      const uint4 *src = reinterpret_cast<const uint4 *>(a.x) + (size_t)b * (a.H / 8);
      uint4 *dst = reinterpret_cast<uint4 *>(a.ex.hidden) + (size_t)id * (a.H / 8);
      for (int k = lane; k < a.H / 8; k += 32) dst[k] = src[k];
    }
  }
  if (lane == 0) {
    a.alive[b] = exit_now ? 0 : 1;
    if (exit_now) {
      if (a.ex.n_exit) atomicAdd(a.ex.n_exit, 1);
      if (a.ex.ramp_count) atomicAdd(a.ex.ramp_count + a.ramp_index, 1);
    }
  }
}

// multi-step decode, fill of layer l (R27): token slot t of the
// chunk gets its exit hidden row (elem bytes per value) and the mask "its
// exit layer lies before l"; rows >= nv are zero with id -1
__global__ void fill_prep_kernel(const int64_t *__restrict__ ids, int nv, int B, const uint8_t *__restrict__ hidden,
                                 int64_t cap, const int32_t *__restrict__ exit_layer, int layer, int64_t row_bytes,
                                 uint8_t *__restrict__ x, int64_t *__restrict__ ids_out, uint8_t *__restrict__ mask) {
  const int t = blockIdx.x;
  const int64_t id = t < nv ? ids[t] : -1;
  const bool ok = id >= 0 && id < cap;
  const int el = ok ? exit_layer[id] : -1;
  const uint4 *src = reinterpret_cast<const uint4 *>(hidden + (ok ? id : 0) * row_bytes);
  uint4 *dst = reinterpret_cast<uint4 *>(x + (int64_t)t * row_bytes);
  for (int64_t k = threadIdx.x; k < row_bytes / 16; k += blockDim.x) dst[k] = ok ? src[k] : make_uint4(0, 0, 0, 0);
  if (threadIdx.x == 0) {
    ids_out[t] = ok ? id : -1;
    mask[t] = (ok && el >= 0 && el < layer) ? 1 : 0;
  }
}

// token i: tokens_out[i] = label; x[i] = embed[label]; its slot's position + 1
__global__ void decode_advance_kernel(const int64_t *__restrict__ ids, int64_t n, const int32_t *__restrict__ label,
                                      int64_t cap, int32_t *__restrict__ tokens_out, const uint8_t *__restrict__ embed,
                                      int32_t vocab, int64_t row_bytes, uint8_t *__restrict__ x,
                                      const int32_t *__restrict__ slot_of_id, int32_t *pos_of_slot, int n_slots,
                                      int *err) {
  const int64_t i = blockIdx.x;
  if (i >= n) return;
  const int64_t id = ids[i];
  const bool ok = id >= 0 && id < cap;
  const int y = ok ? label[id] : -1;
  const bool yok = y >= 0 && y < vocab;
  const uint4 *src = reinterpret_cast<const uint4 *>(embed + (yok ? (int64_t)y : 0) * row_bytes);
  uint4 *dst = reinterpret_cast<uint4 *>(x + i * row_bytes);
  for (int64_t k = threadIdx.x; k < row_bytes / 16; k += blockDim.x) dst[k] = yok ? src[k] : make_uint4(0, 0, 0, 0);
  if (threadIdx.x == 0) {
    if (tokens_out) tokens_out[i] = y;
    if (!yok && err) *err = 1;
    if (ok) {
      const int slot = slot_of_id[id];
      if (slot >= 0 && slot < n_slots) pos_of_slot[slot] += 1;
      else if (err) *err = 1;
    }
  }
}

}  // namespace

E3_TL_SETTER(tl_set_llama)

e3_status fill_prep_run(const int64_t *ids, int nv, int B, const void *hidden, int64_t cap, const int32_t *exit_layer,
                        int layer, int64_t row_bytes, void *x, int64_t *ids_out, uint8_t *mask, cudaStream_t st) {
  fill_prep_kernel<<<B, 128, 0, st>>>(ids, nv, B, reinterpret_cast<const uint8_t *>(hidden), cap, exit_layer, layer,
                                      row_bytes, reinterpret_cast<uint8_t *>(x), ids_out, mask);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status decode_advance_run(const int64_t *ids, int64_t n, const int32_t *label, int64_t cap, int32_t *tokens_out,
                             const void *embed, int32_t vocab, int64_t row_bytes, void *x, const int32_t *slot_of_id,
                             int32_t *pos_of_slot, int n_slots, int *err, cudaStream_t st) {
  if (n <= 0) return E3_OK;
  decode_advance_kernel<<<(unsigned)n, 128, 0, st>>>(ids, n, label, cap, tokens_out,
                                                     reinterpret_cast<const uint8_t *>(embed), vocab, row_bytes,
                                                     reinterpret_cast<uint8_t *>(x), slot_of_id, pos_of_slot, n_slots,
                                                     err);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

// One CTA (8 warps) per row for the decode batch's few long rows (T <= 128
// rows of H = 4096): a warp per row left 64 rows on 8 SMs, each lane summing
// and scaling 128 values in sequence.  Thread t owns the 16-byte vectors t,
// t + 256, ...; the sum of squares is reduced per warp by shuffles, then over
// the 8 warps in warp order (deterministic).
template <int VPT>
__global__ void __launch_bounds__(256) rmsnorm_cta_kernel(const __nv_bfloat16 *__restrict__ x,
                                                          const __nv_bfloat16 *__restrict__ g,
                                                          __nv_bfloat16 *__restrict__ y, int rows, int H, float eps) {
  __shared__ float red[8];
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  const int row = blockIdx.x, t = threadIdx.x, warp = warp_id(), lane = lane_id();
  const int nvec = H / 8;
  uint4 gv[VPT];
#pragma unroll
  for (int i = 0; i < VPT; ++i) {
    const int k = t + 256 * i;
    gv[i] = (k < nvec) ? __ldg(reinterpret_cast<const uint4 *>(g) + k) : make_uint4(0, 0, 0, 0);
  }
  pdl_wait();
  pdl_trigger();
  const unsigned long long tl1 = tl_now();
  if (row >= rows) return;
  const uint4 *xr = reinterpret_cast<const uint4 *>(x + (size_t)row * H);
  uint4 v[VPT];
  float ss = 0.f;
#pragma unroll
  for (int i = 0; i < VPT; ++i) {
    const int k = t + 256 * i;
    v[i] = (k < nvec) ? xr[k] : make_uint4(0, 0, 0, 0);
    const uint32_t w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
#pragma unroll
    for (int e = 0; e < 4; ++e) ss += bf_lo(w[e]) * bf_lo(w[e]) + bf_hi(w[e]) * bf_hi(w[e]);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) ss += __shfl_xor_sync(0xffffffffu, ss, o);
  if (lane == 0) red[warp] = ss;
  __syncthreads();
  float tot = red[0];
#pragma unroll
  for (int w = 1; w < 8; ++w) tot += red[w];
  const float rinv = 1.0f / sqrtf(tot / (float)H + eps);
  uint4 *yr = reinterpret_cast<uint4 *>(y + (size_t)row * H);
#pragma unroll
  for (int i = 0; i < VPT; ++i) {
    const int k = t + 256 * i;
    if (k >= nvec) continue;
    const uint32_t w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
    const uint32_t gw[4] = {gv[i].x, gv[i].y, gv[i].z, gv[i].w};
    uint32_t o[4];
#pragma unroll
    for (int e = 0; e < 4; ++e)
      o[e] = pack_bf16(bf_lo(w[e]) * rinv * bf_lo(gw[e]), bf_hi(w[e]) * rinv * bf_hi(gw[e]));
    yr[k] = make_uint4(o[0], o[1], o[2], o[3]);
  }
  if (threadIdx.x == 0) tl_rec(tlb, 8700, tl0, tl1);
}

// The split-K-by-4 decode GEMM's reduction + residual epilogue fused with the
// RMSNorm that follows it (O -> RMSNorm2, down -> the next RMSNorm1 or the LM
// ramp's final norm): h = bf16((((0 + p0) + p1) + p2) + p3 + r), the same sum
// order and rounding as the cluster split-K kernel's DSMEM reduction and
// RESID epilogue, stored; then the rmsnorm_cta_kernel arithmetic on the
// rounded h.  Replaces the cluster's two barriers, the DSMEM reduction and the
// separate RMSNorm launch (~6 us per GEMM + norm pair, r02 llama_timeline).
template <int VPT>
__global__ void __launch_bounds__(256) reduce_rmsnorm_kernel(const float *__restrict__ part,
                                                             const __nv_bfloat16 *__restrict__ resid,
                                                             __nv_bfloat16 *__restrict__ h_out,
                                                             const __nv_bfloat16 *__restrict__ g,
                                                             __nv_bfloat16 *__restrict__ y, int rows, int H,
                                                             float eps) {
  __shared__ float red[8];
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  const int row = blockIdx.x, t = threadIdx.x, warp = warp_id(), lane = lane_id();
  const int nvec = H / 8;
  const size_t qstride = (size_t)rows * H;
  uint4 gv[VPT];
#pragma unroll
  for (int i = 0; i < VPT; ++i) {
    const int k = t + 256 * i;
    gv[i] = (g && k < nvec) ? __ldg(reinterpret_cast<const uint4 *>(g) + k) : make_uint4(0, 0, 0, 0);
  }
  pdl_wait();
  pdl_trigger();
  const unsigned long long tl1 = tl_now();
  if (row >= rows) return;
  uint4 v[VPT];
  float ss = 0.f;
#pragma unroll
  for (int i = 0; i < VPT; ++i) {
    const int k = t + 256 * i;
    if (k >= nvec) {
      v[i] = make_uint4(0, 0, 0, 0);
      continue;
    }
    const float4 *p = reinterpret_cast<const float4 *>(part + (size_t)row * H + 8 * k);
    float4 a0[4], a1[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      a0[q] = __ldcg(p + q * (qstride / 4));
      a1[q] = __ldcg(p + q * (qstride / 4) + 1);
    }
    const uint4 rv = __ldg(reinterpret_cast<const uint4 *>(resid + (size_t)row * H) + k);
    float acc[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) acc[e] = 0.f;
#pragma unroll
    for (int q = 0; q < 4; ++q) {   // rank order
      acc[0] += a0[q].x; acc[1] += a0[q].y; acc[2] += a0[q].z; acc[3] += a0[q].w;
      acc[4] += a1[q].x; acc[5] += a1[q].y; acc[6] += a1[q].z; acc[7] += a1[q].w;
    }
    const uint32_t rw[4] = {rv.x, rv.y, rv.z, rv.w};
    uint32_t o[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) o[e] = pack_bf16(acc[2 * e] + bf_lo(rw[e]), acc[2 * e + 1] + bf_hi(rw[e]));
    v[i] = make_uint4(o[0], o[1], o[2], o[3]);
    reinterpret_cast<uint4 *>(h_out + (size_t)row * H)[k] = v[i];
#pragma unroll
    for (int e = 0; e < 4; ++e) ss += bf_lo(o[e]) * bf_lo(o[e]) + bf_hi(o[e]) * bf_hi(o[e]);
  }
  if (!g) {
    if (t == 0) tl_rec(tlb, 8710, tl0, tl1);
    return;
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) ss += __shfl_xor_sync(0xffffffffu, ss, o);
  if (lane == 0) red[warp] = ss;
  __syncthreads();
  float tot = red[0];
#pragma unroll
  for (int w = 1; w < 8; ++w) tot += red[w];
  const float rinv = 1.0f / sqrtf(tot / (float)H + eps);
  uint4 *yr = reinterpret_cast<uint4 *>(y + (size_t)row * H);
#pragma unroll
  for (int i = 0; i < VPT; ++i) {
    const int k = t + 256 * i;
    if (k >= nvec) continue;
    const uint32_t w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
    const uint32_t gw[4] = {gv[i].x, gv[i].y, gv[i].z, gv[i].w};
    uint32_t o[4];
#pragma unroll
    for (int e = 0; e < 4; ++e)
      o[e] = pack_bf16(bf_lo(w[e]) * rinv * bf_lo(gw[e]), bf_hi(w[e]) * rinv * bf_hi(gw[e]));
    yr[k] = make_uint4(o[0], o[1], o[2], o[3]);
  }
  if (t == 0) tl_rec(tlb, 8710, tl0, tl1);
}

e3_status reduce_rmsnorm_run(const float *part, const void *resid, void *h_out, const void *g, void *y, int rows,
                             int H, float eps, cudaStream_t st) {
  if (H % 8 || H > 8192 || (g && !y)) {
    set_error("reduce_rmsnorm: need H % 8 == 0, H <= 8192");
    return E3_EUNSUPPORTED;
  }
  auto *rp = reinterpret_cast<const __nv_bfloat16 *>(resid);
  auto *hp = reinterpret_cast<__nv_bfloat16 *>(h_out);
  auto *gp = reinterpret_cast<const __nv_bfloat16 *>(g);
  auto *yp = reinterpret_cast<__nv_bfloat16 *>(y);
  const int vpt = (H / 8 + 255) / 256;
  if (vpt <= 2) E3_CUDA_TRY(launch_k(reduce_rmsnorm_kernel<2>, dim3(rows), dim3(256), 0, st, part, rp, hp, gp, yp, rows, H, eps));
  else E3_CUDA_TRY(launch_k(reduce_rmsnorm_kernel<4>, dim3(rows), dim3(256), 0, st, part, rp, hp, gp, yp, rows, H, eps));
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status rmsnorm_run(const void *x, const void *g, void *y, int rows, int H, float eps, cudaStream_t st) {
  if (H % 8 || H > 8192) {
    set_error("rmsnorm: need H % 8 == 0, H <= 8192");
    return E3_EUNSUPPORTED;
  }
  auto *xp = reinterpret_cast<const __nv_bfloat16 *>(x);
  auto *gp = reinterpret_cast<const __nv_bfloat16 *>(g);
  auto *yp = reinterpret_cast<__nv_bfloat16 *>(y);
  if (H >= 2048 && rows <= 256) {      // few long rows: one CTA per row
    const int vpt = (H / 8 + 255) / 256;
    if (vpt <= 2) E3_CUDA_TRY(launch_k(rmsnorm_cta_kernel<2>, dim3(rows), dim3(256), 0, st, xp, gp, yp, rows, H, eps));
    else E3_CUDA_TRY(launch_k(rmsnorm_cta_kernel<4>, dim3(rows), dim3(256), 0, st, xp, gp, yp, rows, H, eps));
    E3_CUDA_TRY(cudaGetLastError());
    count_launch();
    return E3_OK;
  }
  const dim3 grid((rows + 7) / 8);
  const int vpl = (H / 8 + 31) / 32;
  if (vpl <= 1) E3_CUDA_TRY(launch_k(rmsnorm_kernel<1>, grid, dim3(256), 0, st, xp, gp, yp, rows, H, eps));
  else if (vpl <= 4) E3_CUDA_TRY(launch_k(rmsnorm_kernel<4>, grid, dim3(256), 0, st, xp, gp, yp, rows, H, eps));
  else if (vpl <= 16) E3_CUDA_TRY(launch_k(rmsnorm_kernel<16>, grid, dim3(256), 0, st, xp, gp, yp, rows, H, eps));
  else E3_CUDA_TRY(launch_k(rmsnorm_kernel<32>, grid, dim3(256), 0, st, xp, gp, yp, rows, H, eps));
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status attn_dec_run(const void *q, void *ctx, const void *kc, const void *vc, const int64_t *ids,
                       const int32_t *n_valid_dev, int n_valid_host, const int32_t *slot_of_id, int64_t id_cap,
                       const int32_t *pos_of_slot, int n_slots, int T, int nh, int kvh, int max_ctx,
                       cudaStream_t st) {
  if (max_ctx > 16384 || nh % kvh) {
    set_error("decode attention: need max_ctx <= 16384 and heads % kv_heads == 0");
    return E3_EUNSUPPORTED;
  }
  const size_t smem = (size_t)max_ctx * 4;
  static size_t attr_done = 0;
  if (smem > 48 * 1024 && smem > attr_done) {
    E3_CUDA_TRY(cudaFuncSetAttribute(attn_dec_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr_done = smem;
  }
  E3_CUDA_TRY(launch_k(attn_dec_kernel, dim3(nh, T), dim3(kAttnThreads), smem, st,
                       reinterpret_cast<const __nv_bfloat16 *>(q), reinterpret_cast<__nv_bfloat16 *>(ctx),
                       reinterpret_cast<const __nv_bfloat16 *>(kc), reinterpret_cast<const __nv_bfloat16 *>(vc),
                       ids, n_valid_dev, n_valid_host, slot_of_id, id_cap, pos_of_slot, n_slots, nh, kvh, max_ctx,
                       1.0f / sqrtf((float)kHd)));
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status lm_decide_run(const RampArgs &a, cudaStream_t st) {
  E3_CUDA_TRY(launch_k(lm_decide_kernel, dim3((a.B + 3) / 4), dim3(128), 0, st, a));
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace e3
