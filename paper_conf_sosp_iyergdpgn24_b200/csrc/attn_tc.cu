// Self-attention of the split's encoder layers on the
// sm_100a tensor cores.  S <= 256 fits one KV tile, so there is no online
// rescaling: one CTA owns (input b, head h, 128-query tile):
//
//   TMA   Q [128x64], K [SKVx64], V [SKVx64] (128B swizzle, OOB rows -> 0)
//   MMA1  S = Q K^T          tcgen05 128 x SKV x 64, fp32 in TMEM
//   soft  thread r owns query row r (TMEM lane r): row max, p = 2^((s-m)*log2e/8),
//         l = sum p (fp32, unrounded), bf16(p) -> smem in the K-major SW128
//         layout the next MMA reads as its A operand
//   MMA2  O = P V            tcgen05 128 x 64 x SKV, V read MN-major
//   out   ctx = bf16(O / l)  (rounding contract)
//
// Keys >= S are masked to -inf; query rows >= S are not stored.
#include "common.cuh"
#include "kernels.h"
#include "prof.h"

namespace e3 {

namespace {

constexpr int D = 64;          // head dim
constexpr int QT = 128;        // query rows per CTA

template <int SKV>
struct ACfg {
  static constexpr int kQ = QT * D * 2;          // 16 KB
  static constexpr int kKV = SKV * D * 2;        // 16 / 32 KB
  static constexpr int kP = QT * SKV * 2;        // 32 / 64 KB
  static constexpr int kSmem = kQ + 2 * kKV + kP + 1024 + 64;
  static constexpr int kTmemCols = (SKV + D <= 256) ? 256 : 512;
};

template <int SKV>
__global__ void __launch_bounds__(128)
    attn_tc_kernel(const __grid_constant__ CUtensorMap tq, const __grid_constant__ CUtensorMap tkv,
                   __nv_bfloat16 *__restrict__ ctx, int S, int H, int heads) {
  using CF = ACfg<SKV>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *sQ = smem;
  uint8_t *sK = sQ + CF::kQ;
  uint8_t *sV = sK + CF::kKV;
  uint8_t *sP = sV + CF::kKV;
  uint64_t *bars = reinterpret_cast<uint64_t *>(sP + CF::kP);   // [0] load, [1] S, [2] O
  uint32_t *tslot = reinterpret_cast<uint32_t *>(bars + 3);

  const int bh = blockIdx.x;
  const int b = bh / heads, h = bh % heads;
  const int q0 = blockIdx.y * QT;
  const int warp = warp_id(), lane = lane_id();
  const int tid = threadIdx.x;

  if (tid == 0) {
    tma_prefetch(&tq);
    tma_prefetch(&tkv);
    mbar_init(&bars[0], 1);
    mbar_init(&bars[1], 1);
    mbar_init(&bars[2], 1);
    fence_barrier_init();
  }
  if (warp == 0) tmem_alloc(tslot, CF::kTmemCols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tslot;
  const uint32_t t_s = tbase;          // S accumulator: columns [0, SKV)
  const uint32_t t_o = tbase + SKV;    // O accumulator: columns [SKV, SKV+64)

  if (tid == 0) {
    mbar_expect_tx(&bars[0], CF::kQ + 2 * CF::kKV);
    tma_load_3d(sQ, &tq, &bars[0], h * D, q0, b);
    tma_load_3d(sK, &tkv, &bars[0], H + h * D, 0, b);
    tma_load_3d(sV, &tkv, &bars[0], 2 * H + h * D, 0, b);
    mbar_wait(&bars[0], 0);
    tc_fence_after();
    const uint32_t idesc = idesc_bf16_f32(QT, SKV, 0);
    const uint64_t dq = smem_desc_sw128(smem_u32(sQ), 16, 1024);
    const uint64_t dk = smem_desc_sw128(smem_u32(sK), 16, 1024);
#pragma unroll
    for (int k = 0; k < D / 16; ++k) tc_mma_f16(t_s, dq + 2 * k, dk + 2 * k, idesc, k != 0);
    tc_commit(&bars[1]);
  }
  __syncwarp();

  // ------------------------------------------------------------ softmax
  mbar_wait(&bars[1], 0);
  tc_fence_after();
  const int row = warp * 32 + lane;                       // query row within tile == TMEM lane
  const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
  float mx = -INFINITY;
#pragma unroll 1
  for (int c = 0; c < SKV; c += 32) {
    uint32_t r[32];
    tmem_ld32(t_s + lane_off + c, r);
    tmem_wait_ld();
#pragma unroll
    for (int j = 0; j < 32; ++j)
      if (c + j < S) mx = fmaxf(mx, __uint_as_float(r[j]));
  }
  const float sl2 = 1.4426950408889634f * 0.125f;   // log2(e) / sqrt(64)
  const float mb = mx * sl2;
  float l = 0.f;
  uint8_t *prow = sP + row * 128;
#pragma unroll 1
  for (int c = 0; c < SKV; c += 32) {
    uint32_t r[32];
    tmem_ld32(t_s + lane_off + c, r);
    tmem_wait_ld();
    float p[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) {
      p[j] = (c + j < S) ? exp2f(fmaf(__uint_as_float(r[j]), sl2, -mb)) : 0.f;
      l += p[j];
    }
    // columns c..c+31 -> block c/64, 16-byte chunks (c%64)/8 .. +3, XOR-swizzled by row%8
    uint8_t *blk = prow + (c / 64) * (QT * 128);
    const int ch0 = (c % 64) / 8;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      uint4 o;
      o.x = pack_bf16(p[8 * j + 0], p[8 * j + 1]);
      o.y = pack_bf16(p[8 * j + 2], p[8 * j + 3]);
      o.z = pack_bf16(p[8 * j + 4], p[8 * j + 5]);
      o.w = pack_bf16(p[8 * j + 6], p[8 * j + 7]);
      *reinterpret_cast<uint4 *>(blk + (((ch0 + j) ^ (row & 7)) << 4)) = o;
    }
  }
  fence_proxy_async_smem();     // generic-proxy smem writes -> visible to the tensor core
  tc_fence_before();
  __syncthreads();

  if (tid == 0) {
    tc_fence_after();
    const uint32_t idesc = idesc_bf16_f32(QT, D, 1);   // B (= V) is MN-major
#pragma unroll
    for (int kk = 0; kk < SKV / 16; ++kk) {
      const uint64_t dp = smem_desc_sw128(smem_u32(sP + (kk / 4) * (QT * 128) + (kk % 4) * 32), 16, 1024);
      const uint64_t dv = smem_desc_sw128(smem_u32(sV + kk * 16 * 128), SKV * 128, 1024);
      tc_mma_f16(t_o, dp, dv, idesc, kk != 0);
    }
    tc_commit(&bars[2]);
  }
  __syncwarp();
  mbar_wait(&bars[2], 0);
  tc_fence_after();
  const float inv_l = 1.0f / l;
  const int q = q0 + row;
#pragma unroll
  for (int c = 0; c < D; c += 32) {
    uint32_t r[32];
    tmem_ld32(t_o + lane_off + c, r);
    tmem_wait_ld();
    if (q < S) {
      uint4 *dst = reinterpret_cast<uint4 *>(ctx + ((size_t)b * S + q) * H + h * D + c);
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        uint4 o;
        o.x = pack_bf16(__uint_as_float(r[8 * j + 0]) * inv_l, __uint_as_float(r[8 * j + 1]) * inv_l);
        o.y = pack_bf16(__uint_as_float(r[8 * j + 2]) * inv_l, __uint_as_float(r[8 * j + 3]) * inv_l);
        o.z = pack_bf16(__uint_as_float(r[8 * j + 4]) * inv_l, __uint_as_float(r[8 * j + 5]) * inv_l);
        o.w = pack_bf16(__uint_as_float(r[8 * j + 6]) * inv_l, __uint_as_float(r[8 * j + 7]) * inv_l);
        dst[j] = o;
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tbase, CF::kTmemCols);
}

template <int SKV>
e3_status launch_attn(const AttnMaps &m, void *ctx, int B, int S, int H, int heads, cudaStream_t st) {
  auto kern = attn_tc_kernel<SKV>;
  static bool attr_done = false;
  if (!attr_done) {
    E3_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, ACfg<SKV>::kSmem));
    attr_done = true;
  }
  dim3 grid(B * heads, (S + QT - 1) / QT);
  kern<<<grid, 128, ACfg<SKV>::kSmem, st>>>(m.q, m.kv, reinterpret_cast<__nv_bfloat16 *>(ctx), S, H, heads);
  count_launch();
  E3_CUDA_TRY(cudaGetLastError());
  return E3_OK;
}

}  // namespace

e3_status attn_tmaps(AttnMaps *m, const void *qkv, int B, int S, int H) {
  m->skv = S <= 128 ? 128 : 256;
  const uint64_t W3 = 3ull * H;
  e3_status s = make_tmap_3d(&m->q, qkv, W3, (uint64_t)S, (uint64_t)B, W3, W3 * S, D, QT, 1);
  if (s != E3_OK) return s;
  return make_tmap_3d(&m->kv, qkv, W3, (uint64_t)S, (uint64_t)B, W3, W3 * S, D, (uint32_t)m->skv, 1);
}

e3_status attn_run(const AttnMaps &m, void *ctx, int B, int S, int H, int heads, cudaStream_t st) {
  if (m.skv == 128) return launch_attn<128>(m, ctx, B, S, H, heads, st);
  return launch_attn<256>(m, ctx, B, S, H, heads, st);
}

}  // namespace e3
