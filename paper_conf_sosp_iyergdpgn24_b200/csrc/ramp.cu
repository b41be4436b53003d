// Fused exit ramp + threshold test.
//
// DeeBERT ramp after an encoder block: "a bertpooler, a dropout layer, and a
// fully connected layer" (R1):
//     c = x[b, 0, :]   p = tanh(W_p c + b_p)   z = W_c p + b_c
// exit test (R3/R4/R12): max softmax(z) > tau, or
// entropy(softmax(z)) < tau; the model's last ramp exits every row (R6).
//
// One launch; grid (H / 32 pooler-output tiles, ceil(B / 16) row groups),
// 4 warps per CTA:
//   stage    the 32 W_p rows of the tile by cp.async into padded smem (row
//            pitch H + 8 bf16: conflict-free fragments) and the 16 CLS rows:
//            either copied (cp.async) or, at a split's last layer, read
//            PRE-LayerNorm and normalised here by the shared warp-per-row LN
//            (ln_row.cuh) -- bit-identical to what the fused LN + compaction
//            writes for the survivors, and no full LN2 pass is needed;
//   pooler   warp w owns outputs 8w..8w+7 of the tile: mma.sync m16n8k16
//            bf16 -> fp32 over K = H (a 16 x 32 x H GEMM per CTA is far too
//            small for a tcgen05 tile; the tensor pipe is still the one used);
//   partial  p = tanh(acc + b_p) stays in registers and is immediately folded
//            into partial logits sum_{o in tile} p[b,o] W_c[c,o], reduced over
//            the quad with __shfl_xor_sync and over the 4 warps in smem, and
//            written to a per-tile slot (deterministic, no float atomics);
//   decide   the CTA of row group g that retires last (threadfence + atomic
//            ticket) reduces the H/32 partials per (row, class) with one
//            warp-shuffle butterfly per row (fixed order), then softmax /
//            max-prob / entropy, argmax (lowest index on ties), threshold
//            test, exit record by input id and the alive flag.
// All ramp math is fp32, never rounded to bf16 (rounding contract).
#include "common.cuh"
#include "kernels.h"
#include "ln_row.cuh"
#include "prof.h"

namespace e3 {

namespace {

constexpr int kMaxC = 16;
constexpr int kRows = kRampRowsPerCta;   // 16 = mma M
constexpr int kTileN = 32;               // pooler outputs per CTA (4 warps x n8)
constexpr int kThreads = 128;

__device__ __forceinline__ void cp_async16(void *smem, const void *gmem) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

__device__ __forceinline__ void mma_bf16_16816(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0, %1, %2, %3}, {%4, %5, %6, %7}, {%8, %9}, "
      "{%0, %1, %2, %3};"
      : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

__device__ __forceinline__ bool row_alive(const RampArgs &a, int b, int n_valid) {
  return b < a.B && (a.init_alive ? (b < n_valid) : (a.alive[b] != 0));
}

template <int VPL>
__global__ void __launch_bounds__(kThreads)
    ramp_bert_kernel(RampArgs a) {
  extern __shared__ uint8_t smem_raw[];
  const int H = a.H;
  const int P = H + 8;                                   // padded pitch (bf16)
  __nv_bfloat16 *sC = reinterpret_cast<__nv_bfloat16 *>(smem_raw);   // [16][P]
  __nv_bfloat16 *sW = sC + kRows * P;                                 // [32][P]
  float *sZ = reinterpret_cast<float *>(sW + kTileN * P);             // [4 warps][16 rows][kMaxC]
  __shared__ bool is_last;
  __shared__ bool row_ok[kRows];

  const int warp = warp_id(), lane = lane_id();
  const int g = lane >> 2, t = lane & 3;
  const int b0 = blockIdx.y * kRows;
  const int o0 = blockIdx.x * kTileN;
  const int C = a.C;
  const int nvec = H / 8;
  const __nv_bfloat16 *x = reinterpret_cast<const __nv_bfloat16 *>(a.x);
  const size_t row_stride = (size_t)a.S * H;

  // ---------------------------------------------------------- stage
  const uint4 *wp = reinterpret_cast<const uint4 *>(a.w.w_p);
  for (int i = threadIdx.x; i < kTileN * nvec; i += kThreads) {   // weights first: no dependency
    const int r = i / nvec, k = i - r * nvec;
    cp_async16(reinterpret_cast<uint4 *>(sW + r * P) + k, wp + (size_t)(o0 + r) * nvec + k);
  }
  pdl_wait();                      // CLS rows / alive flags of the previous kernels now visible
  pdl_trigger();
  const int n_valid = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  if (threadIdx.x < kRows) row_ok[threadIdx.x] = row_alive(a, b0 + threadIdx.x, n_valid);
  __syncthreads();
  if (a.ln_g) {
    LnParams<VPL> lp;
    ln_load_params<VPL>(lp, reinterpret_cast<const __nv_bfloat16 *>(a.ln_g),
                        reinterpret_cast<const __nv_bfloat16 *>(a.ln_b), H, lane);
    constexpr int kPerWarp = kRows / (kThreads / 32);   // 4 CLS rows per warp, loads in flight together
    uint4 v[kPerWarp][VPL];
#pragma unroll
    for (int u = 0; u < kPerWarp; ++u) {
      const int r = warp + u * (kThreads / 32);
      if (row_ok[r]) {
        ln_load_row<VPL>(v[u], x + (size_t)(b0 + r) * row_stride, H, lane);
      } else {
#pragma unroll
        for (int i = 0; i < VPL; ++i) v[u][i] = make_uint4(0, 0, 0, 0);
      }
    }
#pragma unroll
    for (int u = 0; u < kPerWarp; ++u) {
      const int r = warp + u * (kThreads / 32);
      if (row_ok[r]) ln_apply<VPL>(v[u], lp, H, a.eps, lane);
      ln_store_row<VPL>(v[u], sC + r * P, H, lane);
    }
  } else {
    for (int i = threadIdx.x; i < kRows * nvec; i += kThreads) {
      const int r = i / nvec, k = i - r * nvec;
      uint4 *dst = reinterpret_cast<uint4 *>(sC + r * P) + k;
      if (row_ok[r])
        cp_async16(dst, reinterpret_cast<const uint4 *>(x + (size_t)(b0 + r) * row_stride) + k);
      else
        *dst = make_uint4(0, 0, 0, 0);
    }
  }
  cp_async_wait_all();
  __syncthreads();

  // ---------------------------------------------------------- pooler (mma.sync)
  float acc[4] = {0.f, 0.f, 0.f, 0.f};
  {
    const __nv_bfloat16 *a_lo = sC + g * P + 2 * t;           // row g
    const __nv_bfloat16 *a_hi = sC + (g + 8) * P + 2 * t;     // row g + 8
    const __nv_bfloat16 *bp = sW + (warp * 8 + g) * P + 2 * t;
#pragma unroll 4
    for (int kk = 0; kk < H; kk += 16) {
      uint32_t af[4];
      af[0] = *reinterpret_cast<const uint32_t *>(a_lo + kk);
      af[1] = *reinterpret_cast<const uint32_t *>(a_hi + kk);
      af[2] = *reinterpret_cast<const uint32_t *>(a_lo + kk + 8);
      af[3] = *reinterpret_cast<const uint32_t *>(a_hi + kk + 8);
      const uint32_t bf0 = *reinterpret_cast<const uint32_t *>(bp + kk);
      const uint32_t bf1 = *reinterpret_cast<const uint32_t *>(bp + kk + 8);
      mma_bf16_16816(acc, af, bf0, bf1);
    }
  }

  // ---------------------------------------------------------- partial logits
  {
    const __nv_bfloat16 *bpool = reinterpret_cast<const __nv_bfloat16 *>(a.w.b_p);
    const __nv_bfloat16 *wc = reinterpret_cast<const __nv_bfloat16 *>(a.w.w_c);
    const int col = o0 + warp * 8 + 2 * t;                  // this lane's two pooler outputs
    const float bb0 = bf2f(bpool[col]), bb1 = bf2f(bpool[col + 1]);
    const float p00 = tanhf(acc[0] + bb0), p01 = tanhf(acc[1] + bb1);   // row g
    const float p10 = tanhf(acc[2] + bb0), p11 = tanhf(acc[3] + bb1);   // row g + 8
#pragma unroll
    for (int c = 0; c < kMaxC; ++c) {
      if (c < C) {
        const float w0 = bf2f(wc[(size_t)c * H + col]), w1 = bf2f(wc[(size_t)c * H + col + 1]);
        float z0 = fmaf(p00, w0, p01 * w1);
        float z1 = fmaf(p10, w0, p11 * w1);
        z0 += __shfl_xor_sync(0xffffffffu, z0, 1);
        z0 += __shfl_xor_sync(0xffffffffu, z0, 2);
        z1 += __shfl_xor_sync(0xffffffffu, z1, 1);
        z1 += __shfl_xor_sync(0xffffffffu, z1, 2);
        if (t == 0) {
          sZ[(warp * kRows + g) * kMaxC + c] = z0;
          sZ[(warp * kRows + g + 8) * kMaxC + c] = z1;
        }
      }
    }
  }
  __syncthreads();
  float *part = a.pool_ws;   // [gridDim.x tiles][B][C]
  for (int i = threadIdx.x; i < kRows * C; i += kThreads) {
    const int r = i / C, c = i - r * C;
    if (b0 + r < a.B) {
      float s = sZ[(0 * kRows + r) * kMaxC + c];
#pragma unroll
      for (int w = 1; w < 4; ++w) s += sZ[(w * kRows + r) * kMaxC + c];
      part[((size_t)blockIdx.x * a.B + b0 + r) * C + c] = s;
    }
  }

  // ---------------------------------------------------------- ticket
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned tk = atomicAdd(a.done_ctr + blockIdx.y, 1u);
    is_last = (tk == gridDim.x - 1);
    if (is_last) a.done_ctr[blockIdx.y] = 0;   // re-arm for the next launch (stream-ordered)
  }
  __syncthreads();
  if (!is_last) return;
  __threadfence();

  // ---------------------------------------------------------- decide
  // warp per row; lane l < ntiles holds tile l's partial logits, butterfly sum
  const int ntiles = gridDim.x;                // <= 32 (H <= 1024)
  const __nv_bfloat16 *bc = reinterpret_cast<const __nv_bfloat16 *>(a.w.b_c);
  for (int r = warp; r < kRows; r += kThreads / 32) {
    const int b = b0 + r;
    if (b >= a.B) break;
    if (!row_ok[r]) {
      if (a.init_alive && lane == 0) a.alive[b] = 0;
      continue;
    }
    float z[kMaxC];
#pragma unroll
    for (int c = 0; c < kMaxC; ++c)
      z[c] = (c < C && lane < ntiles) ? __ldcg(part + ((size_t)lane * a.B + b) * C + c) : 0.f;
#pragma unroll
    for (int c = 0; c < kMaxC; ++c) {
      if (c < C) {
#pragma unroll
        for (int o = 16; o; o >>= 1) z[c] += __shfl_xor_sync(0xffffffffu, z[c], o);
        z[c] += bf2f(bc[c]);
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
        pass = metric > a.tau;
      } else {
        metric = logf(sum) - qz / sum;             // H = lse - sum_c q_c z_c
        pass = metric < a.tau;
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
  if (a.C < 1 || a.C > kMaxC || a.H % kTileN || a.H > 1024) {
    set_error("ramp: need 1 <= C <= 16, H % 32 == 0, H <= 1024");
    return E3_EUNSUPPORTED;
  }
  const int smem = (kRows + kTileN) * (a.H + 8) * 2 + 4 * kRows * kMaxC * 4;
  const int smem_max = (kRows + kTileN) * (1024 + 8) * 2 + 4 * kRows * kMaxC * 4;
  dim3 grid(a.H / kTileN, (a.B + kRows - 1) / kRows);
  const int vpl = (a.H / 8 + 31) / 32;
#define E3_RAMP(V)                                                                                        \
  do {                                                                                                    \
    static bool attr_done = false;                                                                        \
    if (!attr_done) {                                                                                     \
      E3_CUDA_TRY(cudaFuncSetAttribute(ramp_bert_kernel<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                       smem_max));                                                        \
      attr_done = true;                                                                                   \
    }                                                                                                     \
    E3_CUDA_TRY(launch_k(ramp_bert_kernel<V>, grid, dim3(kThreads), smem, st, a));                        \
  } while (0)
  if (vpl <= 1) E3_RAMP(1);
  else if (vpl <= 3) E3_RAMP(3);
  else E3_RAMP(4);
#undef E3_RAMP
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace e3
