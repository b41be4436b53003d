// FP32 mode of the encoder split (E3_DTYPE_FP32; SURVEY §8(b) dtype, §8(c)
// C13; R14): the same split semantics as the bf16 path -- layers,
// fused ramp + threshold test, stable compaction into the next split's queue
// -- with fp32 activations everywhere, so a whole job can be held to the
// north_star's "1e-4 at fp32" against the fp64 oracle.  Weights stay the bf16
// values the model was generated with (exactly representable in fp32, so the
// oracle sees the same numbers).  Paper precision is unstated.
//
// This mode exists to prove the chained pipeline at tight bounds; its kernels
// are plain SIMT with fp32 STORAGE of every activation and fp64 accumulation
// of every dot product / reduction (an fp32 x bf16 product is exact in fp64;
// over 32 LLaMA layers fp32 accumulation alone drifted 3e-4 in the logits),
// fixed summation order, no atomics in any value path, so rows are
// batch-position invariant like the bf16 path:
//   f32_gemm_kernel    Y = epi(A W^T + b): 128 x 128 CTA tile, 8 x 8 per
//                      thread, K in steps of 16 staged in shared memory
//   f32_attn_kernel    one CTA per (input, head): K, V of the head in shared
//                      memory, a warp per query row, exact softmax
//   f32_ln_kernel      warp per row, two-pass statistics
//   f32_ramp_kernel    CTA per row: (LN) / pooler -> classifier -> softmax
//                      metric -> strict threshold -> exit record, alive flag
// Survivors are compacted by the byte-exact ln_compact kernel in copy mode.
#include "common.cuh"
#include "exitrule.cuh"
#include "fp32_path.h"
#include "prof.h"

namespace e3 {

namespace {

constexpr int kGT = 256;   // GEMM threads
constexpr int kBM = 128, kBN = 128, kBK = 16;

template <int EPI>
__global__ void __launch_bounds__(kGT)
    f32_gemm_kernel(const float *__restrict__ A, int lda, const __nv_bfloat16 *__restrict__ W,
                    const __nv_bfloat16 *__restrict__ bias, const float *__restrict__ R, float *__restrict__ Y, int M,
                    int N, int K) {
  __shared__ __align__(16) float As[kBK][kBM + 4];
  __shared__ __align__(16) float Ws[kBK][kBN + 4];
  const int tid = threadIdx.x;
  const int m0 = blockIdx.y * kBM, n0 = blockIdx.x * kBN;
  const int ty = tid / 16, tx = tid % 16;
  double acc[8][8];   // fp64 accumulation: fp32 x bf16 products are exact in fp64
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.0;
  for (int k0 = 0; k0 < K; k0 += kBK) {
#pragma unroll
    for (int u = 0; u < 2; ++u) {   // A tile: 128 rows x 16 k as float4
      const int idx = tid + u * kGT;
      const int row = idx >> 2, kq = idx & 3;
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (m0 + row < M) v = *reinterpret_cast<const float4 *>(A + (size_t)(m0 + row) * lda + k0 + kq * 4);
      As[kq * 4 + 0][row] = v.x;
      As[kq * 4 + 1][row] = v.y;
      As[kq * 4 + 2][row] = v.z;
      As[kq * 4 + 3][row] = v.w;
    }
    {   // W tile: 128 output rows x 16 k (bf16, 8 per 16-byte load)
      const int n = tid >> 1, kh = tid & 1;
      uint4 w = make_uint4(0u, 0u, 0u, 0u);
      if (n0 + n < N) w = *reinterpret_cast<const uint4 *>(W + (size_t)(n0 + n) * K + k0 + kh * 8);
      const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        Ws[kh * 8 + 2 * e][n] = bf_lo(ws[e]);
        Ws[kh * 8 + 2 * e + 1][n] = bf_hi(ws[e]);
      }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kBK; ++k) {
      float a[8], b[8];
      *reinterpret_cast<float4 *>(a) = *reinterpret_cast<const float4 *>(&As[k][ty * 8]);
      *reinterpret_cast<float4 *>(a + 4) = *reinterpret_cast<const float4 *>(&As[k][ty * 8 + 4]);
      *reinterpret_cast<float4 *>(b) = *reinterpret_cast<const float4 *>(&Ws[k][tx * 8]);
      *reinterpret_cast<float4 *>(b + 4) = *reinterpret_cast<const float4 *>(&Ws[k][tx * 8 + 4]);
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = fma((double)a[i], (double)b[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = m0 + ty * 8 + i;
    if (r >= M) continue;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int c = n0 + tx * 8 + j;
      if (c >= N) continue;
      double v = acc[i][j] + (bias ? (double)bf2f(bias[c]) : 0.0);
      if (EPI == E3_EPI_BIAS_GELU) v = 0.5 * v * (1.0 + erf(v * 0.70710678118654752440));
      if (EPI == E3_EPI_BIAS_RESID) v += (double)R[(size_t)r * N + c];
      Y[(size_t)r * N + c] = (float)v;
    }
  }
}

constexpr int kAT = 256;   // attention threads (8 warps)
constexpr int kAW = kAT / 32;

// ctx[b, i, h*64 + d] = sum_j softmax_j(q_i . k_j / 8) v_j[d] for the head h
__global__ void __launch_bounds__(kAT) f32_attn_kernel(const float *__restrict__ qkv, float *__restrict__ ctx, int S,
                                                       int H) {
  extern __shared__ double smd[];
  double *Ps = smd;                     // [warps][S] scores / probabilities (fp64)
  float *Ks = reinterpret_cast<float *>(Ps + (size_t)kAW * S);   // [S][65] (padded: lane j reads key row j)
  float *Vs = Ks + (size_t)S * 65;      // [S][64]
  float *Qs = Vs + (size_t)S * 64;      // [warps][64]
  const int b = blockIdx.x / (H / 64), h = blockIdx.x % (H / 64);
  const float *base = qkv + (size_t)b * S * 3 * H;
  for (int idx = threadIdx.x; idx < S * 64; idx += kAT) {
    const int j = idx >> 6, d = idx & 63;
    Ks[j * 65 + d] = base[(size_t)j * 3 * H + H + h * 64 + d];
    Vs[j * 64 + d] = base[(size_t)j * 3 * H + 2 * H + h * 64 + d];
  }
  __syncthreads();
  const int warp = warp_id(), lane = lane_id();
  float *q = Qs + warp * 64;
  double *p = Ps + (size_t)warp * S;
  for (int i = warp; i < S; i += kAW) {
    q[lane] = base[(size_t)i * 3 * H + h * 64 + lane];
    q[lane + 32] = base[(size_t)i * 3 * H + h * 64 + lane + 32];
    __syncwarp();
    double mx = -INFINITY;
    for (int j = lane; j < S; j += 32) {
      double s = 0.0;
#pragma unroll 16
      for (int d = 0; d < 64; ++d) s = fma((double)q[d], (double)Ks[j * 65 + d], s);
      s *= 0.125;   // 1 / sqrt(64), exact
      p[j] = s;
      mx = fmax(mx, s);
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    double l = 0.0;
    for (int j = lane; j < S; j += 32) {
      const double e = exp(p[j] - mx);
      p[j] = e;
      l += e;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) l += __shfl_xor_sync(0xffffffffu, l, o);
    __syncwarp();
    double o0 = 0.0, o1 = 0.0;
    for (int j = 0; j < S; ++j) {
      const double pj = p[j];
      o0 = fma(pj, (double)Vs[j * 64 + lane], o0);
      o1 = fma(pj, (double)Vs[j * 64 + lane + 32], o1);
    }
    float *out = ctx + ((size_t)b * S + i) * H + h * 64;
    out[lane] = (float)(o0 / l);
    out[lane + 32] = (float)(o1 / l);
    __syncwarp();
  }
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

__device__ __forceinline__ double warp_sumd(double v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// y = (x - mean) / sqrt(var + eps) * g + b per row, biased variance (fp64 sums)
__global__ void __launch_bounds__(256) f32_ln_kernel(const float *__restrict__ x, const __nv_bfloat16 *__restrict__ g,
                                                     const __nv_bfloat16 *__restrict__ bb, float *__restrict__ y,
                                                     int rows, int H, float eps) {
  const int row = blockIdx.x * 8 + warp_id(), lane = lane_id();
  if (row >= rows) return;
  const float *xr = x + (size_t)row * H;
  double s = 0.0;
  for (int k = lane; k < H; k += 32) s += xr[k];
  const double mean = warp_sumd(s) / H;
  double q = 0.0;
  for (int k = lane; k < H; k += 32) {
    const double d = xr[k] - mean;
    q = fma(d, d, q);
  }
  const double rstd = 1.0 / sqrt(warp_sumd(q) / H + (double)eps);
  float *yr = y + (size_t)row * H;
  for (int k = lane; k < H; k += 32) yr[k] = (float)((xr[k] - mean) * rstd * bf2f(g[k]) + bf2f(bb[k]));
}

constexpr int kRT = 256;

// One CTA per batch row: the ramp of DESIGN.md R1 in fp32 and the exit test
// (R3/R4/R6/R12), with the bf16 ramp's row semantics (padding never exits,
// rows that exited at an earlier ramp of the split are skipped).
__global__ void __launch_bounds__(kRT) f32_ramp_kernel(RampArgs a) {
  extern __shared__ float rs[];
  const int H = a.H, C = a.C;
  float *c = rs;          // [H] CLS row (ViT: normalised)
  float *p = c + H;       // [H] pooler output (BERT)
  // [C] logits: shared memory, or this row's slice of a global scratch
  // (a.pool_ws, [B][C]) when C does not fit (Llama-3 vocabulary, 128256)
  float *z = a.pool_ws ? a.pool_ws + (size_t)blockIdx.x * C : p + H;
  __shared__ double red[kRT / 32][3];
  __shared__ int redi[kRT / 32];
  const int b = blockIdx.x, tid = threadIdx.x, warp = warp_id(), lane = lane_id();
  const int n_valid = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  const bool ok = a.init_alive ? (b < n_valid) : (a.alive[b] != 0);
  if (!ok) {
    if (a.init_alive && tid == 0) a.alive[b] = 0;
    return;
  }
  const float *x = reinterpret_cast<const float *>(a.x) + (size_t)b * a.S * H;   // token 0
  for (int k = tid; k < H; k += kRT) c[k] = x[k];
  __syncthreads();
  const bool vit = a.arch == E3_ARCH_VIT;
  if (a.arch == E3_ARCH_LLAMA_DECODE) {   // nf = RMSNorm_f(c) (R22)
    if (warp == 0) {
      double q = 0.0;
      for (int k = lane; k < H; k += 32) q = fma((double)c[k], (double)c[k], q);
      const double r = 1.0 / sqrt(warp_sumd(q) / H + (double)a.eps);
      const __nv_bfloat16 *g = reinterpret_cast<const __nv_bfloat16 *>(a.w.ln_g);
      for (int k = lane; k < H; k += 32) p[k] = (float)(c[k] * r * bf2f(g[k]));
    }
  } else if (vit) {   // n = LN_r(c)
    if (warp == 0) {
      double s = 0.0;
      for (int k = lane; k < H; k += 32) s += c[k];
      const double mean = warp_sumd(s) / H;
      double q = 0.0;
      for (int k = lane; k < H; k += 32) q = fma(c[k] - mean, c[k] - mean, q);
      const double rstd = 1.0 / sqrt(warp_sumd(q) / H + (double)a.eps);
      const __nv_bfloat16 *g = reinterpret_cast<const __nv_bfloat16 *>(a.w.ln_g);
      const __nv_bfloat16 *bb = reinterpret_cast<const __nv_bfloat16 *>(a.w.ln_b);
      for (int k = lane; k < H; k += 32) p[k] = (float)((c[k] - mean) * rstd * bf2f(g[k]) + bf2f(bb[k]));
    }
  } else {     // p = tanh(W_p c + b_p): a warp per output, lanes over k
    const __nv_bfloat16 *wp = reinterpret_cast<const __nv_bfloat16 *>(a.w.w_p);
    const __nv_bfloat16 *bp = reinterpret_cast<const __nv_bfloat16 *>(a.w.b_p);
    for (int o = warp; o < H; o += kRT / 32) {
      double s = 0.0;
      for (int k = lane; k < H; k += 32) s = fma((double)bf2f(wp[(size_t)o * H + k]), (double)c[k], s);
      s = warp_sumd(s);
      if (lane == 0) p[o] = (float)tanh(s + bf2f(bp[o]));
    }
  }
  __syncthreads();
  {   // z = W_c p + b_c: a warp per class
    const __nv_bfloat16 *wc = reinterpret_cast<const __nv_bfloat16 *>(a.w.w_c);
    const __nv_bfloat16 *bc = reinterpret_cast<const __nv_bfloat16 *>(a.w.b_c);
    for (int o = warp; o < C; o += kRT / 32) {
      double s = 0.0;
      for (int k = lane; k < H; k += 32) s = fma((double)bf2f(wc[(size_t)o * H + k]), (double)p[k], s);
      s = warp_sumd(s);
      if (lane == 0) z[o] = (float)(s + (bc ? bf2f(bc[o]) : 0.f));
    }
  }
  __syncthreads();
  // max and argmax (lowest index on ties, R12)
  double m = -INFINITY;
  int arg = 0x7fffffff;
  for (int k = tid; k < C; k += kRT)
    if (z[k] > m) { m = z[k]; arg = k; }   // k ascending per thread: first max kept
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    const double m2 = __shfl_xor_sync(0xffffffffu, m, o);
    const int a2 = __shfl_xor_sync(0xffffffffu, arg, o);
    if (m2 > m || (m2 == m && a2 < arg)) { m = m2; arg = a2; }
  }
  if (lane == 0) { red[warp][0] = m; redi[warp] = arg; }
  __syncthreads();
  if (tid == 0) {
    for (int w = 1; w < kRT / 32; ++w)
      if (red[w][0] > red[0][0] || (red[w][0] == red[0][0] && redi[w] < redi[0])) {
        red[0][0] = red[w][0];
        redi[0] = redi[w];
      }
  }
  __syncthreads();
  m = red[0][0];
  const int label = redi[0];
  double se = 0.0, sq = 0.0;
  for (int k = tid; k < C; k += kRT) {
    const double e = exp((double)z[k] - m);
    se += e;
    sq = fma(e, (double)z[k] - m, sq);
  }
  se = warp_sumd(se);
  sq = warp_sumd(sq);
  __syncthreads();
  if (lane == 0) { red[warp][1] = se; red[warp][2] = sq; }
  __syncthreads();
  __shared__ int s_exit;
  __shared__ int64_t s_id;
  if (tid == 0) {
    double sum = 0.0, qz = 0.0;
    for (int w = 0; w < kRT / 32; ++w) { sum += red[w][1]; qz += red[w][2]; }
    float metric;
    bool pass;
    if (a.test == E3_TEST_PATIENCE) {
      pass = patience_step(a.ex.state, a.id[b], a.ex.capacity, label, a.tau, &metric);
    } else if (a.test == E3_TEST_MAXPROB) {   // the metric is reported (and tested) as fp32
      metric = (float)(1.0 / sum);
      pass = metric > a.tau;
    } else {
      metric = (float)(log(sum) - qz / sum);
      pass = metric < a.tau;
    }
    const bool exit_now = pass || a.final_ramp;
    if (a.ex.ramp_metric && a.id[b] >= 0 && a.id[b] < a.ex.capacity)
      a.ex.ramp_metric[a.id[b] * a.ex.ramp_metric_stride + a.ramp_index] = metric;
    const int64_t id = a.id[b];
    const bool rec = exit_now && id >= 0 && id < a.ex.capacity;
    if (rec) {
      if (a.ex.exit_layer) a.ex.exit_layer[id] = a.layer;
      if (a.ex.label) a.ex.label[id] = label;
      if (a.ex.conf) a.ex.conf[id] = metric;
    }
    if (exit_now) {
      if (a.ex.n_exit) atomicAdd(a.ex.n_exit, 1);
      if (a.ex.ramp_count) atomicAdd(a.ex.ramp_count + a.ramp_index, 1);
    }
    a.alive[b] = exit_now ? 0 : 1;
    s_exit = rec;
    s_id = id;
  }
  __syncthreads();
  if (s_exit && a.ex.logits)
    for (int k = tid; k < C; k += kRT) a.ex.logits[s_id * C + k] = z[k];
  if (s_exit && a.ex.hidden && a.arch == E3_ARCH_LLAMA_DECODE)   // the exit row (multi-step decode)
    for (int k = tid; k < H; k += kRT) reinterpret_cast<float *>(a.ex.hidden)[s_id * H + k] = c[k];
}

// ---- LLaMA decode (R22) in fp32 --------------------------------------

// y = x / sqrt(mean(x^2) + eps) * g per row
__global__ void __launch_bounds__(256) f32_rms_kernel(const float *__restrict__ x, const __nv_bfloat16 *__restrict__ g,
                                                      float *__restrict__ y, int rows, int H, float eps) {
  const int row = blockIdx.x * 8 + warp_id(), lane = lane_id();
  if (row >= rows) return;
  const float *xr = x + (size_t)row * H;
  double q = 0.0;
  for (int k = lane; k < H; k += 32) q = fma((double)xr[k], (double)xr[k], q);
  const double r = 1.0 / sqrt(warp_sumd(q) / H + (double)eps);
  float *yr = y + (size_t)row * H;
  for (int k = lane; k < H; k += 32) yr[k] = (float)(xr[k] * r * bf2f(g[k]));
}

// a = SiLU(g) * u elementwise
__global__ void f32_swiglu_kernel(const float *__restrict__ g, const float *__restrict__ u, float *__restrict__ a,
                                  size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    const double x = g[i];
    a[i] = (float)(x / (1.0 + exp(-x)) * u[i]);
  }
}

// token t: q <- RoPE(q) into qo [T, nh*128]; k <- RoPE(k), v appended to the
// fp32 cache at (slot, pos) -- only for valid rows still alive in the split
// (R15); slot / pos outside the cache -> *err, row skipped
__global__ void f32_rope_kv_kernel(const float *__restrict__ qkv, float *__restrict__ qo, float *__restrict__ kc,
                                   float *__restrict__ vc, const float2 *__restrict__ rope, DecArgs a) {
  const int t = blockIdx.x, j = threadIdx.x;   // 64 threads: rotation pairs (j, j + 64)
  const int nv = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  const int64_t id = a.ids[t];
  const bool live = t < nv && (a.init_alive || a.alive == nullptr || a.alive[t] != 0) && id >= 0 && id < a.id_cap;
  int slot = -1, pos = 0;
  if (live) {
    slot = a.slot_of_id[id];
    if (slot < 0 || slot >= a.n_slots) {
      slot = -1;
      if (j == 0 && a.err) *a.err = 1;
    } else {
      pos = a.pos_of_slot[slot];
      if (pos < 0 || pos >= a.max_ctx) {
        slot = -1;
        pos = 0;
        if (j == 0 && a.err) *a.err = 1;
      }
    }
  }
  const int ld = (a.nh + 2 * a.kvh) * 128;
  const float *row = qkv + (size_t)t * ld;
  const float2 csf = rope[(size_t)pos * 64 + j];
  const double2 cs = make_double2(csf.x, csf.y);
  for (int h = 0; h < a.nh; ++h) {
    const float lo = row[h * 128 + j], hi = row[h * 128 + j + 64];
    qo[(size_t)t * a.nh * 128 + h * 128 + j] = (float)(lo * cs.x - hi * cs.y);
    qo[(size_t)t * a.nh * 128 + h * 128 + j + 64] = (float)(hi * cs.x + lo * cs.y);
  }
  if (slot < 0) return;
  for (int h = 0; h < a.kvh; ++h) {
    const float lo = row[(a.nh + h) * 128 + j], hi = row[(a.nh + h) * 128 + j + 64];
    float *kd = kc + (((size_t)slot * a.kvh + h) * a.max_ctx + pos) * 128;
    float *vd = vc + (((size_t)slot * a.kvh + h) * a.max_ctx + pos) * 128;
    kd[j] = (float)(lo * cs.x - hi * cs.y);
    kd[j + 64] = (float)(hi * cs.x + lo * cs.y);
    vd[j] = row[(a.nh + a.kvh + h) * 128 + j];
    vd[j + 64] = row[(a.nh + a.kvh + h) * 128 + j + 64];
  }
}

// ctx[t, h*128 + d] = sum_p softmax_p(q . K[p] / sqrt 128) V[p][d], p = 0..pos
__global__ void __launch_bounds__(128) f32_attn_dec_kernel(const float *__restrict__ q, float *__restrict__ ctx,
                                                           const float *__restrict__ kc, const float *__restrict__ vc,
                                                           DecArgs a) {
  extern __shared__ double sp[];   // [max_ctx]
  __shared__ float qs[128];
  __shared__ double red[4];
  const int h = blockIdx.x, t = blockIdx.y, tid = threadIdx.x, warp = warp_id(), lane = lane_id();
  const int nv = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  const int64_t id = a.ids[t];
  float *out = ctx + (size_t)t * a.nh * 128 + h * 128;
  int pos = -1, slot = -1;
  if (t < nv && id >= 0 && id < a.id_cap) {
    slot = a.slot_of_id[id];
    if (slot >= 0 && slot < a.n_slots) pos = a.pos_of_slot[slot];
  }
  if (pos < 0 || pos >= a.max_ctx) {   // padding / outside the cache: finite zeros
    out[tid] = 0.f;
    return;
  }
  const int g = h / (a.nh / a.kvh);
  qs[tid] = q[(size_t)t * a.nh * 128 + h * 128 + tid];
  __syncthreads();
  const float *K = kc + ((size_t)slot * a.kvh + g) * a.max_ctx * 128;
  const float *V = vc + ((size_t)slot * a.kvh + g) * a.max_ctx * 128;
  const double scale = 1.0 / sqrt(128.0);
  double mx = -INFINITY;
  for (int p = tid; p <= pos; p += 128) {
    double s = 0.0;
    for (int d = 0; d < 128; ++d) s = fma((double)qs[d], (double)K[(size_t)p * 128 + d], s);
    s *= scale;
    sp[p] = s;
    mx = fmax(mx, s);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if (lane == 0) red[warp] = mx;
  __syncthreads();
  mx = fmax(fmax(red[0], red[1]), fmax(red[2], red[3]));
  __syncthreads();
  double l = 0.0;
  for (int p = tid; p <= pos; p += 128) {
    const double e = exp(sp[p] - mx);
    sp[p] = e;
    l += e;
  }
  l = warp_sumd(l);
  if (lane == 0) red[warp] = l;
  __syncthreads();
  l = red[0] + red[1] + red[2] + red[3];
  double o = 0.0;
  for (int p = 0; p <= pos; ++p) o = fma(sp[p], (double)V[(size_t)p * 128 + tid], o);
  out[tid] = (float)(o / l);
}

}  // namespace

e3_status f32_rms_run(const float *x, const void *g, float *y, int rows, int H, float eps, cudaStream_t st) {
  f32_rms_kernel<<<(rows + 7) / 8, 256, 0, st>>>(x, reinterpret_cast<const __nv_bfloat16 *>(g), y, rows, H, eps);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status f32_swiglu_run(const float *g, const float *u, float *a, size_t n, cudaStream_t st) {
  f32_swiglu_kernel<<<(unsigned)((n + 255) / 256 < 4096 ? (n + 255) / 256 : 4096), 256, 0, st>>>(g, u, a, n);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status f32_rope_kv_run(const float *qkv, float *qo, float *kc, float *vc, const float2 *rope, const DecArgs &a,
                          cudaStream_t st) {
  f32_rope_kv_kernel<<<a.T, 64, 0, st>>>(qkv, qo, kc, vc, rope, a);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status f32_attn_dec_run(const float *q, float *ctx, const float *kc, const float *vc, const DecArgs &a,
                           cudaStream_t st) {
  const size_t smem = (size_t)a.max_ctx * sizeof(double);
  static size_t attr = 0;
  if (smem > 48 * 1024 && smem > attr) {
    E3_CUDA_TRY(cudaFuncSetAttribute(f32_attn_dec_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = smem;
  }
  f32_attn_dec_kernel<<<dim3(a.nh, a.T), 128, smem, st>>>(q, ctx, kc, vc, a);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status f32_gemm_run(const float *A, int lda, const void *W, const void *bias, const float *R, float *Y, int M,
                       int N, int K, int epi, cudaStream_t st) {
  if (K % kBK || lda % 4) {
    set_error("fp32 GEMM: need K % 16 == 0 and lda % 4 == 0");
    return E3_EUNSUPPORTED;
  }
  const dim3 grid((N + kBN - 1) / kBN, (M + kBM - 1) / kBM);
  auto *w = reinterpret_cast<const __nv_bfloat16 *>(W);
  auto *b = reinterpret_cast<const __nv_bfloat16 *>(bias);
  if (epi == E3_EPI_BIAS) f32_gemm_kernel<E3_EPI_BIAS><<<grid, kGT, 0, st>>>(A, lda, w, b, R, Y, M, N, K);
  else if (epi == E3_EPI_BIAS_GELU) f32_gemm_kernel<E3_EPI_BIAS_GELU><<<grid, kGT, 0, st>>>(A, lda, w, b, R, Y, M, N, K);
  else f32_gemm_kernel<E3_EPI_BIAS_RESID><<<grid, kGT, 0, st>>>(A, lda, w, b, R, Y, M, N, K);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status f32_attn_run(const float *qkv, float *ctx, int B, int S, int H, cudaStream_t st) {
  if (H % 64 || S > 256) {
    set_error("fp32 attention: need head_dim 64 and S <= 256");
    return E3_EUNSUPPORTED;
  }
  const size_t smem = ((size_t)S * (65 + 64) + kAW * 64) * sizeof(float) + (size_t)kAW * S * sizeof(double);
  static size_t attr = 0;
  if (smem > 48 * 1024 && smem > attr) {
    E3_CUDA_TRY(cudaFuncSetAttribute(f32_attn_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = smem;
  }
  f32_attn_kernel<<<B * (H / 64), kAT, smem, st>>>(qkv, ctx, S, H);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status f32_ln_run(const float *x, const void *g, const void *b, float *y, int rows, int H, float eps,
                     cudaStream_t st) {
  f32_ln_kernel<<<(rows + 7) / 8, 256, 0, st>>>(x, reinterpret_cast<const __nv_bfloat16 *>(g),
                                                reinterpret_cast<const __nv_bfloat16 *>(b), y, rows, H, eps);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status f32_ramp_run(const RampArgs &a, cudaStream_t st) {
  // a.pool_ws: global [B][C] logits scratch (large vocabularies), else shared memory
  const size_t smem = (2 * (size_t)a.H + (a.pool_ws ? 0 : a.C)) * sizeof(float);
  static size_t attr = 0;
  if (smem > 48 * 1024 && smem > attr) {
    E3_CUDA_TRY(cudaFuncSetAttribute(f32_ramp_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = smem;
  }
  f32_ramp_kernel<<<a.B, kRT, smem, st>>>(a);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace e3
