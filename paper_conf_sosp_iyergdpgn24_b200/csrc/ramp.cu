// Fused exit ramp + threshold test.
//
// DeeBERT ramp after an encoder block: "a bertpooler, a dropout layer, and a
// fully connected layer" (R1):
//     c = x[b, 0, :]   p = tanh(W_p c + b_p)   z = W_c p + b_c
// exit test (R3/R4/R12): max softmax(z) > tau, or
// entropy(softmax(z)) < tau; the model's last ramp exits every row (R6).
//
// One launch, two phases:
//   phase 1 (all CTAs)  CTA (j, g) computes pooler outputs 8j..8j+7 for rows
//                       16g..16g+15: warp = one output, lanes split H in
//                       16-byte vectors, W_p row held in registers, CLS
//                       vectors of 4 rows in flight at once, dot products
//                       reduced with __shfl_xor_sync; fp32 result to a [B,H]
//                       workspace.
//   phase 2 (last CTA   the CTA of row group g that retires last (threadfence +
//    of each group)     atomic ticket per group) runs the classifier of its 16
//                       rows: warp per row, lanes split H in 8-wide vectors,
//                       per-class warp-shuffle reductions, then softmax /
//                       max-prob / entropy, argmax (lowest index on ties),
//                       threshold test, exit record by id, alive flag.
// All ramp math is fp32, never rounded to bf16 (rounding contract).
#include "common.cuh"
#include "kernels.h"
#include "prof.h"

namespace e3 {

namespace {

constexpr int kMaxC = 16;
constexpr int kRowsPerCta = kRampRowsPerCta;
constexpr int kRowUnroll = 4;   // rows whose CLS vectors are in flight together

__device__ __forceinline__ float dot8(uint4 c4, uint4 w4, float acc) {
  const uint32_t cw[4] = {c4.x, c4.y, c4.z, c4.w};
  const uint32_t ww[4] = {w4.x, w4.y, w4.z, w4.w};
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    acc = fmaf(bf_lo(cw[e]), bf_lo(ww[e]), acc);
    acc = fmaf(bf_hi(cw[e]), bf_hi(ww[e]), acc);
  }
  return acc;
}

__device__ __forceinline__ bool row_alive(const RampArgs &a, int b, int n_valid) {
  return b < a.B && (a.init_alive ? (b < n_valid) : (a.alive[b] != 0));
}

// grid (H/8 pooler-output groups, ceil(B/16) row groups); 8 warps per CTA
template <int VPL>
__global__ void __launch_bounds__(256)
    ramp_bert_kernel(RampArgs a) {
  const int warp = warp_id(), lane = lane_id();
  const int H = a.H;
  const int nvec = H / 8;
  const __nv_bfloat16 *x = reinterpret_cast<const __nv_bfloat16 *>(a.x);
  const size_t row_stride = (size_t)a.S * H;
  const int n_valid = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  const int b0 = blockIdx.y * kRowsPerCta;

  // ---------------------------------------------------------- phase 1
  // warp = pooler output o; its W_p row lives in registers; the CLS vectors
  // of kRowUnroll rows are loaded before any arithmetic (memory parallelism).
  {
    const int o = blockIdx.x * 8 + warp;
    const uint4 *wrow = reinterpret_cast<const uint4 *>(a.w.w_p) + (size_t)o * nvec;
    uint4 w[VPL];
#pragma unroll
    for (int i = 0; i < VPL; ++i) {
      const int k = lane + 32 * i;
      w[i] = (k < nvec) ? __ldg(wrow + k) : make_uint4(0, 0, 0, 0);
    }
    const float bias = bf2f(reinterpret_cast<const __nv_bfloat16 *>(a.w.b_p)[o]);
#pragma unroll 1
    for (int r0 = b0; r0 < b0 + kRowsPerCta; r0 += kRowUnroll) {
      uint4 c[kRowUnroll][VPL];
      bool al[kRowUnroll];
#pragma unroll
      for (int u = 0; u < kRowUnroll; ++u) {
        al[u] = row_alive(a, r0 + u, n_valid);
        const uint4 *cr = reinterpret_cast<const uint4 *>(x + (size_t)(r0 + u) * row_stride);
#pragma unroll
        for (int i = 0; i < VPL; ++i) {
          const int k = lane + 32 * i;
          c[u][i] = (al[u] && k < nvec) ? __ldg(cr + k) : make_uint4(0, 0, 0, 0);
        }
      }
#pragma unroll
      for (int u = 0; u < kRowUnroll; ++u) {
        if (!al[u]) continue;   // warp-uniform
        float acc = 0.f;
#pragma unroll
        for (int i = 0; i < VPL; ++i) acc = dot8(c[u][i], w[i], acc);
#pragma unroll
        for (int s = 16; s; s >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, s);
        if (lane == 0) a.pool_ws[(size_t)(r0 + u) * H + o] = tanhf(acc + bias);
      }
    }
  }

  // ---------------------------------------------------------- ticket
  // the last CTA of this row group (over the H/8 output groups) classifies it
  __shared__ bool is_last;
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned t = atomicAdd(a.done_ctr + blockIdx.y, 1u);
    is_last = (t == gridDim.x - 1);
    if (is_last) a.done_ctr[blockIdx.y] = 0;   // re-arm for the next launch (stream-ordered)
  }
  __syncthreads();
  if (!is_last) return;
  __threadfence();

  // ---------------------------------------------------------- phase 2
  // warp per row: lanes split H into 8-wide vectors, one warp-shuffle
  // reduction per class, then softmax / metric / test on lane 0.
  const int C = a.C;
  const uint4 *wc = reinterpret_cast<const uint4 *>(a.w.w_c);
  const __nv_bfloat16 *bc = reinterpret_cast<const __nv_bfloat16 *>(a.w.b_c);
  const float tau = a.tau;
  for (int b = b0 + warp; b < b0 + kRowsPerCta && b < a.B; b += 8) {
    if (!row_alive(a, b, n_valid)) {
      if (a.init_alive && lane == 0) a.alive[b] = 0;
      continue;
    }
    const float4 *pr = reinterpret_cast<const float4 *>(a.pool_ws + (size_t)b * H);
    float p[VPL][8];
#pragma unroll
    for (int i = 0; i < VPL; ++i) {
      const int k = lane + 32 * i;
      const float4 lo = (k < nvec) ? __ldcg(pr + 2 * k) : make_float4(0.f, 0.f, 0.f, 0.f);
      const float4 hi = (k < nvec) ? __ldcg(pr + 2 * k + 1) : make_float4(0.f, 0.f, 0.f, 0.f);
      p[i][0] = lo.x; p[i][1] = lo.y; p[i][2] = lo.z; p[i][3] = lo.w;
      p[i][4] = hi.x; p[i][5] = hi.y; p[i][6] = hi.z; p[i][7] = hi.w;
    }
    float z[kMaxC];
#pragma unroll
    for (int c = 0; c < kMaxC; ++c) {
      z[c] = 0.f;
      if (c < C) {
        uint4 wv[VPL];
#pragma unroll
        for (int i = 0; i < VPL; ++i) {
          const int k = lane + 32 * i;
          wv[i] = (k < nvec) ? __ldg(wc + (size_t)c * nvec + k) : make_uint4(0, 0, 0, 0);
        }
        float acc = 0.f;
#pragma unroll
        for (int i = 0; i < VPL; ++i) {
          const uint32_t ww[4] = {wv[i].x, wv[i].y, wv[i].z, wv[i].w};
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            acc = fmaf(p[i][2 * e], bf_lo(ww[e]), acc);
            acc = fmaf(p[i][2 * e + 1], bf_hi(ww[e]), acc);
          }
        }
#pragma unroll
        for (int s = 16; s; s >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, s);
        z[c] = acc + bf2f(bc[c]);
      }
    }
    if (lane == 0) {
      float m = z[0];
      int label = 0;
#pragma unroll
      for (int c = 1; c < kMaxC; ++c)
        if (c < C && z[c] > m) { m = z[c]; label = c; }   // lowest index on ties
      float sum = 0.f, qz = 0.f;
#pragma unroll
      for (int c = 0; c < kMaxC; ++c)
        if (c < C) {
          const float e = expf(z[c] - m);
          sum += e;
          qz += e * (z[c] - m);
        }
      float metric;
      bool pass;
      if (a.test == E3_TEST_MAXPROB) {
        metric = 1.0f / sum;                       // max_c softmax(z)_c
        pass = metric > tau;
      } else {
        metric = logf(sum) - qz / sum;             // H = lse - sum_c q_c z_c
        pass = metric < tau;
      }
      const bool exit_now = pass || a.final_ramp;
      if (exit_now) {
        const int64_t id = a.id[b];
        if (id >= 0 && id < a.ex.capacity) {
          if (a.ex.exit_layer) a.ex.exit_layer[id] = a.layer;
          if (a.ex.label) a.ex.label[id] = label;
          if (a.ex.conf) a.ex.conf[id] = metric;
          if (a.ex.logits) {
#pragma unroll
            for (int c = 0; c < kMaxC; ++c)
              if (c < C) a.ex.logits[id * C + c] = z[c];
          }
        }
        if (a.ex.n_exit) atomicAdd(a.ex.n_exit, 1);
        if (a.ex.ramp_count) atomicAdd(a.ex.ramp_count + a.ramp_index, 1);
      }
      a.alive[b] = exit_now ? 0 : 1;
    }
  }
}

}  // namespace

e3_status ramp_run(const RampArgs &a, cudaStream_t st) {
  if (a.arch != E3_ARCH_BERT) {
    set_error("ramp: only the BERT (pooler) ramp is implemented");
    return E3_EUNSUPPORTED;
  }
  if (a.C < 1 || a.C > kMaxC || a.H % 8 || a.H > 4096) {
    set_error("ramp: need 1 <= C <= 16, H % 8 == 0, H <= 4096");
    return E3_EUNSUPPORTED;
  }
  dim3 grid(a.H / 8, (a.B + kRowsPerCta - 1) / kRowsPerCta);
  const int vpl = (a.H / 8 + 31) / 32;
  if (vpl <= 1) ramp_bert_kernel<1><<<grid, 256, 0, st>>>(a);
  else if (vpl <= 3) ramp_bert_kernel<3><<<grid, 256, 0, st>>>(a);
  else if (vpl <= 4) ramp_bert_kernel<4><<<grid, 256, 0, st>>>(a);
  else if (vpl <= 8) ramp_bert_kernel<8><<<grid, 256, 0, st>>>(a);
  else ramp_bert_kernel<16><<<grid, 256, 0, st>>>(a);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace e3
