// Layer GEMMs of the split on the sm_100a 5th-gen tensor
// cores: C[M,N] = epi(A[M,K] . W[N,K]^T), bf16 operands, fp32 accumulation in
// TMEM, one rounding to bf16 in the epilogue.
//
// Design:
//   * persistent grid (<= #SMs CTAs), static round-robin over 128 x BN tiles,
//     n-fastest so concurrently running CTAs share the A tile through L2;
//   * warp 0 = TMA producer (128B-swizzled 128x64 A and BNx64 W boxes into a
//     STAGES-deep smem ring guarded by full/empty mbarriers);
//   * warp 1 = MMA issuer: one thread issues tcgen05.mma.cta_group::1.kind::f16
//     128xBNx16 per 16-wide K step, tcgen05.commit frees the smem stage;
//   * two TMEM accumulators (2*BN columns) so the epilogue of tile i overlaps
//     the MMAs of tile i+1;
//   * warps 4..11 = epilogue: tcgen05.ld 32x32b.x32 -> +bias (+GELU | +residual)
//     -> bf16 -> 16-byte global stores; each warp owns its TMEM lane quarter
//     (warp % 4) and one half of the BN columns.
#include "common.cuh"
#include "kernels.h"
#include "prof.h"

namespace e3 {

namespace {

constexpr int BM = 128;
constexpr int BK = 64;
constexpr int kThreads = 384;   // 4 control warps + 8 epilogue warps

template <int BN>
struct Cfg {
  static constexpr int kABytes = BM * BK * 2;
  static constexpr int kBBytes = BN * BK * 2;
  static constexpr int kStageBytes = kABytes + kBBytes;
  static constexpr int kStages = (192 * 1024) / kStageBytes;
  static constexpr int kTmemCols = 2 * BN;   // 128 / 256 / 512: powers of two
  static constexpr int kSmem = kStages * kStageBytes + 1024 /*align*/ + 256 /*barriers*/;
};

template <int BN, int EPI>
__global__ void __launch_bounds__(kThreads, 1)
    gemm_bf16_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                        __nv_bfloat16 *__restrict__ C, const __nv_bfloat16 *__restrict__ bias,
                        const __nv_bfloat16 *__restrict__ R, int M, int N, int K) {
  using CF = Cfg<BN>;
  constexpr int S = CF::kStages;
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *sA = smem;                                   // S x 16 KB
  uint8_t *sB = smem + S * CF::kABytes;                 // S x BN*128 B
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + S * CF::kStageBytes);
  uint64_t *empty = full + S;
  uint64_t *tfull = empty + S;        // [2]
  uint64_t *tempty = tfull + 2;       // [2]
  uint32_t *tmem_base_slot = reinterpret_cast<uint32_t *>(tempty + 2);

  const int warp = warp_id();
  const int lane = lane_id();
  const int num_m = (M + BM - 1) / BM;
  const int num_n = N / BN;
  const int num_tiles = num_m * num_n;
  const int num_kb = K / BK;

  if (warp == 0 && lane == 0) {
    tma_prefetch(&tmA);
    tma_prefetch(&tmB);
  }
  if (warp == 1 && lane == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&tfull[i], 1);
      mbar_init(&tempty[i], 8);   // one arrive per epilogue warp
    }
    fence_barrier_init();
  }
  if (warp == 2) tmem_alloc(tmem_base_slot, CF::kTmemCols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_base_slot;

  if (warp == 0) {
    // ------------------------------------------------ TMA producer
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
        const int m_blk = t / num_n, n_blk = t % num_n;
        for (int kb = 0; kb < num_kb; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          mbar_expect_tx(&full[stage], CF::kStageBytes);
          tma_load_2d(sA + stage * CF::kABytes, &tmA, &full[stage], kb * BK, m_blk * BM);
          tma_load_2d(sB + stage * CF::kBBytes, &tmB, &full[stage], kb * BK, n_blk * BN);
          if (++stage == S) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer
    constexpr uint32_t idesc = idesc_bf16_f32(BM, BN, 0);
    int stage = 0;
    uint32_t phase = 0;
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
      mbar_wait(&tempty[acc], acc_phase ^ 1);
      tc_fence_after();
      const uint32_t d_tmem = tmem_base + acc * BN;
      for (int kb = 0; kb < num_kb; ++kb) {
        mbar_wait(&full[stage], phase);
        tc_fence_after();
        if (lane == 0) {
          const uint64_t da = smem_desc_sw128(smem_u32(sA + stage * CF::kABytes), 16, 1024);
          const uint64_t db = smem_desc_sw128(smem_u32(sB + stage * CF::kBBytes), 16, 1024);
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            // +32 bytes per 16-element K step inside the 128-byte swizzle atom
            tc_mma_f16(d_tmem, da + (uint64_t)(2 * k), db + (uint64_t)(2 * k), idesc, (kb | k) != 0);
          }
          tc_commit(&empty[stage]);
        }
        __syncwarp();
        if (++stage == S) { stage = 0; phase ^= 1; }
      }
      if (lane == 0) tc_commit(&tfull[acc]);
      __syncwarp();
      if (++acc == 2) { acc = 0; acc_phase ^= 1; }
    }
  } else if (warp >= 4) {
    // ------------------------------------------------ epilogue
    const int q = warp & 3;              // TMEM lane quarter this warp may access
    const int half = (warp - 4) >> 2;    // which half of the BN columns
    const int row = q * 32 + lane;
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int t = blockIdx.x; t < num_tiles; t += gridDim.x) {
      const int m_blk = t / num_n, n_blk = t % num_n;
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const int m = m_blk * BM + row;
      const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN;
#pragma unroll 1
      for (int c = half * (BN / 2); c < (half + 1) * (BN / 2); c += 32) {
        uint32_t r[32];
        tmem_ld32(taddr + c, r);
        tmem_wait_ld();
        const int n0 = n_blk * BN + c;
        float v[32];
        const uint4 *bp = reinterpret_cast<const uint4 *>(bias + n0);
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          uint4 b4 = __ldg(bp + j);
          uint32_t bw[4] = {b4.x, b4.y, b4.z, b4.w};
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            v[j * 8 + 2 * e] = __uint_as_float(r[j * 8 + 2 * e]) + bf_lo(bw[e]);
            v[j * 8 + 2 * e + 1] = __uint_as_float(r[j * 8 + 2 * e + 1]) + bf_hi(bw[e]);
          }
        }
        if (m < M) {
          if (EPI == E3_EPI_BIAS_GELU) {
#pragma unroll
            for (int j = 0; j < 32; ++j) v[j] = gelu_erf(v[j]);
          }
          if (EPI == E3_EPI_BIAS_RESID) {
            const uint4 *rp = reinterpret_cast<const uint4 *>(R + (size_t)m * N + n0);
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              uint4 r4 = rp[j];
              uint32_t rw[4] = {r4.x, r4.y, r4.z, r4.w};
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                v[j * 8 + 2 * e] += bf_lo(rw[e]);
                v[j * 8 + 2 * e + 1] += bf_hi(rw[e]);
              }
            }
          }
          uint4 *cp = reinterpret_cast<uint4 *>(C + (size_t)m * N + n0);
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            uint4 o;
            o.x = pack_bf16(v[j * 8 + 0], v[j * 8 + 1]);
            o.y = pack_bf16(v[j * 8 + 2], v[j * 8 + 3]);
            o.z = pack_bf16(v[j * 8 + 4], v[j * 8 + 5]);
            o.w = pack_bf16(v[j * 8 + 6], v[j * 8 + 7]);
            cp[j] = o;
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[acc]);
      if (++acc == 2) { acc = 0; acc_phase ^= 1; }
    }
  }
  __syncthreads();
  if (warp == 2) tmem_dealloc(tmem_base, CF::kTmemCols);
}

template <int BN, int EPI>
e3_status launch(const CUtensorMap &ta, const CUtensorMap &tb, __nv_bfloat16 *C, const __nv_bfloat16 *bias,
                 const __nv_bfloat16 *R, int M, int N, int K, int sms, cudaStream_t st) {
  auto kern = gemm_bf16_tc_kernel<BN, EPI>;
  static bool attr_done = false;   // per instantiation
  if (!attr_done) {
    E3_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<BN>::kSmem));
    attr_done = true;
  }
  const int tiles = ((M + BM - 1) / BM) * (N / BN);
  const int grid = tiles < sms ? tiles : sms;
  kern<<<grid, kThreads, Cfg<BN>::kSmem, st>>>(ta, tb, C, bias, R, M, N, K);
  count_launch();
  E3_CUDA_TRY(cudaGetLastError());
  return E3_OK;
}

template <int BN>
e3_status launch_epi(int epi, const CUtensorMap &ta, const CUtensorMap &tb, __nv_bfloat16 *C,
                     const __nv_bfloat16 *bias, const __nv_bfloat16 *R, int M, int N, int K, int sms,
                     cudaStream_t st) {
  switch (epi) {
    case E3_EPI_BIAS: return launch<BN, E3_EPI_BIAS>(ta, tb, C, bias, R, M, N, K, sms, st);
    case E3_EPI_BIAS_GELU: return launch<BN, E3_EPI_BIAS_GELU>(ta, tb, C, bias, R, M, N, K, sms, st);
    case E3_EPI_BIAS_RESID: return launch<BN, E3_EPI_BIAS_RESID>(ta, tb, C, bias, R, M, N, K, sms, st);
  }
  set_error("bad epilogue");
  return E3_EINVAL;
}

}  // namespace

int gemm_pick_bn(int M, int N, int sms) {
  // Minimise (waves x per-tile cost), per-tile cost ~ BN + 16 (fixed
  // prologue / epilogue overhead in column units).
  int best = 0;
  long best_cost = 0;
  const int cands[3] = {256, 128, 64};
  for (int i = 0; i < 3; ++i) {
    const int bn = cands[i];
    if (N % bn) continue;
    const long tiles = (long)((M + BM - 1) / BM) * (N / bn);
    const long waves = (tiles + sms - 1) / sms;
    const long cost = waves * (bn + 16);
    if (best == 0 || cost < best_cost) { best = bn; best_cost = cost; }
  }
  return best;
}

e3_status gemm_tmaps(GemmMaps *g, const void *A, int64_t lda, const void *W, int M, int N, int K, int bn) {
  e3_status s = make_tmap_2d(&g->a, A, (uint64_t)M, (uint64_t)K, (uint64_t)lda, BM, BK);
  if (s != E3_OK) return s;
  s = make_tmap_2d(&g->b, W, (uint64_t)N, (uint64_t)K, (uint64_t)K, (uint32_t)bn, BK);
  g->bn = bn;
  return s;
}

e3_status gemm_run(const GemmMaps &g, void *C, const void *bias, const void *R, int M, int N, int K, int epi,
                   int sms, cudaStream_t st) {
  auto *c = reinterpret_cast<__nv_bfloat16 *>(C);
  auto *b = reinterpret_cast<const __nv_bfloat16 *>(bias);
  auto *r = reinterpret_cast<const __nv_bfloat16 *>(R);
  switch (g.bn) {
    case 256: return launch_epi<256>(epi, g.a, g.b, c, b, r, M, N, K, sms, st);
    case 128: return launch_epi<128>(epi, g.a, g.b, c, b, r, M, N, K, sms, st);
    case 64: return launch_epi<64>(epi, g.a, g.b, c, b, r, M, N, K, sms, st);
  }
  set_error("unsupported GEMM N tile");
  return E3_EUNSUPPORTED;
}

}  // namespace e3
