// Attention output projection with the following LayerNorm fused into its
// epilogue (DESIGN.md §6 K1b):
//   BERT (post-LN):  x1 = bf16(LN1(y1)),  y1 = bf16(ctx W_o^T + b_o + x)
//   ViT  (pre-LN):   y1 = bf16(ctx W_o^T + b_o + x)   (the residual stream, stored)
//                    n2 = bf16(LN2(y1))
// Same rounding points as the unfused kernels:
// y1 is rounded to bf16 before its statistics are taken.
//
// A LayerNorm needs whole rows (H <= 1024 columns), more than one TMEM
// accumulator holds (512 fp32 columns), so a CLUSTER OF 2 CTAs owns a
// 128-row block: CTA rank r computes columns [r*H/2, (r+1)*H/2) with
// tcgen05.mma.cta_group::1 (M = 128, N = H/2 split into <= 256-column
// MMAs), and the two CTAs exchange per-row partial sums through DSMEM.  M = 8192 rows at BB is 64
// clusters = 128 CTAs, one wave.
//   warp 0   TMA producer (W_o boxes for the first stages are issued before
//            the PDL wait: they do not depend on the previous kernel)
//   warp 1   single-thread MMA issuer
//   warp 2   TMEM allocator
//   warps 4-11 epilogue: TMEM -> +bias +residual -> bf16 y1 into a 128-byte
//            swizzled smem tile (reusing the drained pipeline stages) -> row
//            statistics (sum and sum of squares in one pass, packed fp32x2
//            arithmetic: this epilogue is issue-bound) -> one DSMEM exchange
//            -> normalise in place -> TMA stores.
// Replaces the O-projection GEMM + the LayerNorm kernel: one launch and one
// full read + write of the [M, H] activations fewer per layer.
#include "common.cuh"
#include "kernels.h"
#include "prof.h"

namespace e3 {

namespace {

constexpr int LM = 128;           // rows per CTA (MMA M)
constexpr int LBK = 64;           // K per stage (one 128-byte swizzle atom)
constexpr int kLThreads = 384;
constexpr int kLSmemMax = 232448;

template <int NH>
struct LCfg {
  static constexpr int NMMA = (NH + 255) / 256;      // MMAs per k16 step
  static constexpr int NSUB = NH / NMMA;             // columns per MMA (<= 256, % 16 == 0)
  static constexpr int kA = LM * LBK * 2;            // 16 KB
  static constexpr int kW = NH * LBK * 2;
  static constexpr int kStage = kA + kW;
  static constexpr int kExtra = 1024 + 512 + (2 * 3 + 4) * LM * 4 + 3 * NH * 2;   // align, barriers, partials, params
  static constexpr int kStages = (kLSmemMax - kExtra) / kStage;
  static constexpr int kY = LM * NH * 2;             // bf16 y tile, [NH/64 blocks][128 rows][128 B]
  static_assert(kStages >= 2, "pipeline too shallow");
  static_assert(kStages * kStage >= kY, "y tile must fit in the drained stage buffers");
  static constexpr int kTmem = NH <= 128 ? 128 : NH <= 256 ? 256 : 512;
  static constexpr int kSmem = kStages * kStage + kExtra;
};

__device__ __forceinline__ void epi_bar256() { asm volatile("bar.sync 1, 256;" ::: "memory"); }
template <int NT>
__device__ __forceinline__ void epi_bar_n() { asm volatile("bar.sync 1, %0;" ::"n"(NT) : "memory"); }

template <int NH>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kLThreads, 1)
    gemm_ln_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmW,
                   const __grid_constant__ CUtensorMap tmR, const __grid_constant__ CUtensorMap tmPre,
                   const __grid_constant__ CUtensorMap tmOut, LnGemmArgs a) {
  using CF = LCfg<NH>;
  constexpr int S = CF::kStages;
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  extern __shared__ uint8_t smem_raw[];
  // 1024-B aligned by offset arithmetic on the __shared__ array, so the
  // compiler keeps the shared address space (LDS / STS, not generic LD / ST)
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t *sA = smem;
  uint8_t *sW = smem + S * CF::kA;
  uint8_t *sY = smem;                                   // after the mainloop: y / LN tile
  // epilogue warps: all 12 where NH splits into three 32-column-aligned
  // parts (BB's 384), else warps 4-11 (two parts); the producer, MMA and
  // allocator warps are idle once the accumulator is complete
  constexpr int EW = (NH % 96 == 0) ? 12 : 8;
  constexpr int NPART = EW / 4;                                    // column parts per row
  float *xs = reinterpret_cast<float *>(smem + S * CF::kStage);    // [NPART][128] local sums
  float *xr2 = xs + NPART * LM;                                    // [NPART][128] local squares
  float *xr1 = xr2 + NPART * LM;                                   // [2 ranks][128][2] exchange
  __nv_bfloat16 *sPar = reinterpret_cast<__nv_bfloat16 *>(xr1 + 4 * LM);   // [3][NH]: bias, gamma, beta
  uint64_t *full = reinterpret_cast<uint64_t *>(sPar + 3 * NH);
  uint64_t *empty = full + S;
  uint64_t *tfull = empty + S;
  uint64_t *rbar = tfull + 1;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(rbar + 1);

  const int warp = warp_id(), lane = lane_id();
  const uint32_t rank = cluster_ctarank();
  const int m0 = (blockIdx.x >> 1) * LM;
  const int n0 = (int)rank * NH;
  const int nkb = a.K / LBK;
  // split cluster barrier: arrive now, wait before the first DSMEM store
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");

  if (warp == 0 && lane == 0) {
    tma_prefetch(&tmA);
    tma_prefetch(&tmW);
    tma_prefetch(&tmOut);
    tma_prefetch(&tmR);
    if (a.store_pre) tma_prefetch(&tmPre);
  }
  if (warp == 1 && lane == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    mbar_init(tfull, 1);
    mbar_init(rbar, 1);
    fence_barrier_init();
  }
  if (warp == 2) tmem_alloc(tmem_slot, CF::kTmem);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ producer
    if (lane == 0) {
      const int pre = nkb < S ? nkb : S;
      for (int kb = 0; kb < pre; ++kb) {          // weights first
        mbar_expect_tx(&full[kb], CF::kStage);
#pragma unroll
        for (int s = 0; s < CF::NMMA; ++s)
          tma_load_2d(sW + kb * CF::kW + s * CF::NSUB * 128, &tmW, &full[kb], kb * LBK, n0 + s * CF::NSUB);
      }
      pdl_wait();
      pdl_trigger();
      for (int kb = 0; kb < pre; ++kb) tma_load_2d(sA + kb * CF::kA, &tmA, &full[kb], kb * LBK, m0);
      int stage = pre % S;
      uint32_t phase = (pre == S) ? 1 : 0;
      for (int kb = pre; kb < nkb; ++kb) {
        mbar_wait(&empty[stage], phase ^ 1);
        mbar_expect_tx(&full[stage], CF::kStage);
        tma_load_2d(sA + stage * CF::kA, &tmA, &full[stage], kb * LBK, m0);
#pragma unroll
        for (int s = 0; s < CF::NMMA; ++s)
          tma_load_2d(sW + stage * CF::kW + s * CF::NSUB * 128, &tmW, &full[stage], kb * LBK, n0 + s * CF::NSUB);
        if (++stage == S) { stage = 0; phase ^= 1; }
      }
      // The residual tile lands, by TMA, exactly where y1 will be written (the
      // same 128-byte-swizzled 64-column blocks, over the drained stages):
      // block b is issued as soon as the last MMA reading any stage region it
      // overlaps has completed, so most of it arrives during the last k-blocks
      // instead of one round trip after the mainloop (~2 us, r02 timeline)
      mbar_expect_tx(rbar, LM * NH * 2);
      for (int blk = 0; blk < NH / 64; ++blk) {
        const int lo = blk * LM * 128, hi = lo + LM * 128;
        int last = -1;                            // latest k-block reading an overlapped region
        for (int s2 = 0; s2 < S && s2 < nkb; ++s2) {
          const int alo = s2 * CF::kA, wlo = S * CF::kA + s2 * CF::kW;
          const bool ov = (lo < alo + CF::kA && hi > alo) || (lo < wlo + CF::kW && hi > wlo);
          const int kl = s2 + ((nkb - 1 - s2) / S) * S;   // the stage's final k-block
          if (ov && kl > last) last = kl;
        }
        if (last >= 0) mbar_wait(&empty[last % S], (uint32_t)((last / S) & 1));   // no later phase exists
        tma_load_2d(sY + lo, &tmR, rbar, n0 + blk * 64, m0);
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    pdl_wait();
    pdl_trigger();
    if (lane == 0) {
      constexpr uint32_t idesc = idesc_bf16_f32(LM, CF::NSUB, 0);
      int stage = 0;
      uint32_t phase = 0;
      for (int kb = 0; kb < nkb; ++kb) {
        mbar_wait(&full[stage], phase);
        tc_fence_after();
        const uint64_t da = smem_desc_sw128(smem_u32(sA + stage * CF::kA), 16, 1024);
#pragma unroll
        for (int s = 0; s < CF::NMMA; ++s) {
          const uint64_t db = smem_desc_sw128(smem_u32(sW + stage * CF::kW + s * CF::NSUB * 128), 16, 1024);
#pragma unroll
          for (int k = 0; k < LBK / 16; ++k)
            tc_mma_f16(tmem_base + s * CF::NSUB, da + (uint64_t)(2 * k), db + (uint64_t)(2 * k), idesc,
                       (kb | k) != 0);
        }
        tc_commit(&empty[stage]);
        if (++stage == S) { stage = 0; phase ^= 1; }
      }
      tc_commit(tfull);
    }
  } else if (warp >= 4) {
    // bias / gamma / beta of this CTA's columns -> smem (independent of the
    // previous kernel), while the mainloop runs
    for (int i = threadIdx.x - 128; i < NH / 8; i += 256) {
      reinterpret_cast<uint4 *>(sPar)[i] = __ldg(reinterpret_cast<const uint4 *>(a.bias + n0) + i);
      reinterpret_cast<uint4 *>(sPar + NH)[i] = __ldg(reinterpret_cast<const uint4 *>(a.g + n0) + i);
      reinterpret_cast<uint4 *>(sPar + 2 * NH)[i] = __ldg(reinterpret_cast<const uint4 *>(a.b + n0) + i);
    }
    pdl_wait();
    pdl_trigger();
  }
  __syncwarp();
  asm volatile("barrier.cluster.wait.aligned;" ::: "memory");   // the peer CTA is running

  // ---------------------------------------------------------------- epilogue
  const bool epi = EW == 12 || warp >= 4;
  const int q = warp & 3, h = EW == 12 ? (warp >> 2) : ((warp - 4) >> 2);   // lane quarter, column part
  const int row = q * 32 + lane;
  const int m = m0 + row;
  constexpr int HC = NH / NPART;                  // columns per epilogue thread
  float2 sum2 = make_float2(0.f, 0.f), sq2 = make_float2(0.f, 0.f);   // row sum, sum of squares
  unsigned long long tlA = 0, tlB = 0, tlR = 0, tlP = 0, tlX = 0;
  if (epi) {
    mbar_wait(tfull, 0);                          // all MMAs done: the stage buffers are drained
    tc_fence_after();
    tlA = tl_now();
    // (the residual tile was issued by the producer as the stages drained)
    epi_bar_n<EW * 32>();                                 // sPar written by every epilogue thread
    mbar_wait(rbar, 0);
    tlR = tl_now();
    const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16);
#pragma unroll 1
    for (int c = 0; c < HC; c += 32) {
      const int col = h * HC + c;                 // within this CTA's NH columns
      uint32_t r[32];
      tmem_ld32(taddr + col, r);
      uint8_t *blk = sY + (col / 64) * (LM * 128) + row * 128;
      const int ch0 = (col % 64) / 8;
      uint4 rv[4], bv[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        rv[j] = *reinterpret_cast<const uint4 *>(blk + (((ch0 + j) ^ (row & 7)) << 4));
        bv[j] = reinterpret_cast<const uint4 *>(sPar + col)[j];
      }
      tmem_wait_ld();
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t rw[4] = {rv[j].x, rv[j].y, rv[j].z, rv[j].w};
        const uint32_t bw[4] = {bv[j].x, bv[j].y, bv[j].z, bv[j].w};
        uint32_t o[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) {   // packed fp32x2 arithmetic: the epilogue is issue-bound
          const float2 acc2 = make_float2(__uint_as_float(r[j * 8 + 2 * e]), __uint_as_float(r[j * 8 + 2 * e + 1]));
          const float2 y2 = __fadd2_rn(__fadd2_rn(acc2, make_float2(bf_lo(bw[e]), bf_hi(bw[e]))),
                                       make_float2(bf_lo(rw[e]), bf_hi(rw[e])));
          o[e] = pack_bf16(y2.x, y2.y);
          const float2 yr = make_float2(bf_lo(o[e]), bf_hi(o[e]));   // statistics of the ROUNDED y1
          sum2 = __fadd2_rn(sum2, yr);
          sq2 = __ffma2_rn(yr, yr, sq2);
        }
        *reinterpret_cast<uint4 *>(blk + (((ch0 + j) ^ (row & 7)) << 4)) = make_uint4(o[0], o[1], o[2], o[3]);
      }
    }
    fence_proxy_async_smem();                     // y1 tile -> visible to the TMA (async proxy)
    // this CTA's (sum, sum of squares) of the row (fixed order: half 0 +
    // half 1) -> both CTAs' slot [rank]; one exchange round (the second
    // moment about 0 is exact enough in fp32 for LayerNorm inputs of O(1))
    tlP = tl_now();
    xs[h * LM + row] = sum2.x + sum2.y;
    xr2[h * LM + row] = sq2.x + sq2.y;
    epi_bar_n<EW * 32>();
    if (h == 0) {
      float s1 = xs[row], s2 = xr2[row];
#pragma unroll
      for (int pp = 1; pp < NPART; ++pp) {        // parts in order
        s1 += xs[pp * LM + row];
        s2 += xr2[pp * LM + row];
      }
      xr1[2 * rank * LM + 2 * row] = s1;          // xr1 here: [2 ranks][128 rows][2]
      xr1[2 * rank * LM + 2 * row + 1] = s2;
      const uint32_t dst = mapa_shared(smem_u32(&xr1[2 * rank * LM + 2 * row]), rank ^ 1);
      asm volatile("st.shared::cluster.v2.f32 [%0], {%1, %2};" ::"r"(dst), "f"(s1), "f"(s2) : "memory");
    }
  }
  // y1 (the residual stream, ViT) is an output too: stored before the tile is
  // normalised in place (every thread's y1 writes were fenced above)
  if (a.store_pre) {
    if (epi) epi_bar_n<EW * 32>();
    if (warp == 4 && lane == 0) {
      for (int blk = 0; blk < NH / 64; ++blk) tma_store_2d(&tmPre, sY + blk * (LM * 128), n0 + blk * 64, m0);
      bulk_commit();
    }
  }
  tlX = tl_now();
  cluster_sync();                                 // both CTAs' row statistics visible
  if (epi) {
    tlB = tl_now();
    const float s1 = xr1[2 * row] + xr1[2 * LM + 2 * row], s2 = xr1[2 * row + 1] + xr1[2 * LM + 2 * row + 1];
    const float mean = s1 / (float)a.N;
    const float var = fmaxf(s2 / (float)a.N - mean * mean, 0.f);
    const float rstd = 1.0f / sqrtf(var + a.eps);
    const float2 nmean2 = make_float2(-mean, -mean), rstd2 = make_float2(rstd, rstd);
    if (a.store_pre) {                            // the y1 stores must have read the tile
      if (warp == 4 && lane == 0) bulk_wait_read<0>();
      epi_bar_n<EW * 32>();
    }
#pragma unroll 1
    for (int c = 0; c < HC; c += 8) {
      const int col = h * HC + c;
      uint4 *p = reinterpret_cast<uint4 *>(sY + (col / 64) * (LM * 128) + row * 128 +
                                           ((((col % 64) / 8) ^ (row & 7)) << 4));
      const uint4 v = *p;
      const uint4 gv = *reinterpret_cast<const uint4 *>(sPar + NH + col);
      const uint4 bv = *reinterpret_cast<const uint4 *>(sPar + 2 * NH + col);
      const uint32_t w[4] = {v.x, v.y, v.z, v.w};
      const uint32_t gw[4] = {gv.x, gv.y, gv.z, gv.w};
      const uint32_t bw[4] = {bv.x, bv.y, bv.z, bv.w};
      uint32_t o[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 d2 = __fadd2_rn(make_float2(bf_lo(w[e]), bf_hi(w[e])), nmean2);
        const float2 t2 = __fmul2_rn(rstd2, make_float2(bf_lo(gw[e]), bf_hi(gw[e])));
        const float2 r2 = __ffma2_rn(d2, t2, make_float2(bf_lo(bw[e]), bf_hi(bw[e])));
        o[e] = pack_bf16(r2.x, r2.y);
      }
      *p = make_uint4(o[0], o[1], o[2], o[3]);
    }
    fence_proxy_async_smem();
    epi_bar_n<EW * 32>();
    if (warp == 4 && lane == 0) {
      for (int blk = 0; blk < NH / 64; ++blk) tma_store_2d(&tmOut, sY + blk * (LM * 128), n0 + blk * 64, m0);
      bulk_commit();
      bulk_wait_read<0>();                        // smem read before exit; the global writes complete with the grid
      tl_rec(tlb, 77, tlA, tlB);                  // mainloop done, statistics exchanged, stored
      tl_rec(tlb, 78, tlR, tlP);                  // residual landed, pass 1 done, (before cluster sync)
      tl_rec(tlb, 79, tlX, tlX);
    }
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2) tmem_dealloc(tmem_base, CF::kTmem);
  if (threadIdx.x == 0) tl_rec(tlb, 7, tl0, tl0);
}

template <int NH>
e3_status ln_launch(const LnGemmMaps &m, const LnGemmArgs &a, cudaStream_t st) {
  auto kern = gemm_ln_kernel<NH>;
  static bool attr_done = false;
  if (!attr_done) {
    E3_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, LCfg<NH>::kSmem));
    attr_done = true;
  }
  const int grid = 2 * ((a.M + LM - 1) / LM);
  E3_CUDA_TRY(launch_k(kern, dim3(grid), dim3(kLThreads), LCfg<NH>::kSmem, st, m.a, m.w, m.r, m.pre, m.out, a));
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}


// ---------------------------------------------------------------------------
// CTA-PAIR variant (DESIGN.md §6 K1b, r02): a CLUSTER OF 4 owns 256 rows.
// Ranks 0,1 (pair 0) compute columns [0, NH), ranks 2,3 (pair 1) columns
// [NH, 2NH); inside a pair, rank parity selects the 128-row half and the
// leader (even rank) issues tcgen05.mma.cta_group::2 (M = 256) while each CTA
// TMA-loads only its 128 A rows and HALF of the pair's W columns.  Per CTA
// the smem fill drops from (128 + NH) x K to (128 + NH/2) x K elements (BB:
// 786 -> 491 KB): the fused O + LN1 was TMA-fill-bound (r01 timeline 18 us
// after release for 5 us of MMA).  The epilogue is the one above; the row
// statistics travel to rank ^ 2 (same rows, the other column half).
template <int NH>
struct L2Cfg {
  static constexpr int NMMA = (NH + 255) / 256;       // MMAs per k16 step (N <= 256 each)
  static constexpr int NSUB = NH / NMMA;              // MMA N
  static constexpr int kBox = NSUB / 2;               // W rows per CTA per MMA
  static constexpr int kA = LM * LBK * 2;             // 16 KB
  static constexpr int kW = (NH / 2) * LBK * 2;       // this CTA's half of the pair's W tile
  static constexpr int kStage = kA + kW;
  static constexpr int kExtra = 1024 + 512 + 4 * 2 * LM * 4 + 3 * NH * 2;
  static constexpr int kStages = (kLSmemMax - kExtra) / kStage;
  static constexpr int kY = LM * NH * 2;
  static_assert(kStages >= 2, "pipeline too shallow");
  static_assert(kStages * kStage >= kY, "y tile must fit in the drained stage buffers");
  static_assert(kBox % 8 == 0 && NSUB % 16 == 0, "MMA shape");
  static constexpr int kTmem = NH <= 128 ? 128 : NH <= 256 ? 256 : 512;
  static constexpr int kSmem = kStages * kStage + kExtra;
};

template <int NH>
__global__ void __cluster_dims__(4, 1, 1) __launch_bounds__(kLThreads, 1)
    gemm_ln2_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmW,
                    const __grid_constant__ CUtensorMap tmR, const __grid_constant__ CUtensorMap tmPre,
                    const __grid_constant__ CUtensorMap tmOut, LnGemmArgs a) {
  using CF = L2Cfg<NH>;
  constexpr int S = CF::kStages;
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  extern __shared__ uint8_t smem_raw[];
  // 1024-B aligned by offset arithmetic on the __shared__ array, so the
  // compiler keeps the shared address space (LDS / STS, not generic LD / ST)
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t *sA = smem;
  uint8_t *sW = smem + S * CF::kA;
  uint8_t *sY = smem;                                   // after the mainloop: y / LN tile
  float *xs = reinterpret_cast<float *>(smem + S * CF::kStage);    // [2 halves][128] local sums
  float *xr2 = xs + 2 * LM;                                        // [2 halves][128] local squares
  float *xr1 = xr2 + 2 * LM;                                       // [2 column halves][128][2] exchange
  __nv_bfloat16 *sPar = reinterpret_cast<__nv_bfloat16 *>(xr1 + 4 * LM);   // [3][NH]: bias, gamma, beta
  uint64_t *full = reinterpret_cast<uint64_t *>(sPar + 3 * NH);
  uint64_t *empty = full + S;
  uint64_t *tfull = empty + S;
  uint64_t *rbar = tfull + 1;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(rbar + 1);

  const int warp = warp_id(), lane = lane_id();
  const uint32_t rank = cluster_ctarank();
  const uint32_t chalf = rank >> 1, sub = rank & 1u;   // column half (pair), row half (in the pair)
  const bool leader = sub == 0;
  const uint32_t lead_rank = rank & ~1u;
  const uint16_t pair_mask = (uint16_t)(0x3u << lead_rank);
  const int m0 = (blockIdx.x >> 2) * (2 * LM) + (int)sub * LM;   // this CTA's rows
  const int n0 = (int)chalf * NH;                                 // the pair's columns
  const int nkb = a.K / LBK;

  if (warp == 0 && lane == 0) {
    tma_prefetch(&tmA);
    tma_prefetch(&tmW);
    tma_prefetch(&tmOut);
    tma_prefetch(&tmR);
    if (a.store_pre) tma_prefetch(&tmPre);
  }
  if (warp == 1 && lane == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    mbar_init(tfull, 1);
    mbar_init(rbar, 1);
    fence_barrier_init();
  }
  if (warp == 2) tmem_alloc2(tmem_slot, CF::kTmem);
  tc_fence_before();
  cluster_sync();                                       // peers' barriers initialised, TMEM allocated
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ producer
    if (lane == 0) {
      auto fb = [&](int st) { return mapa_shared(smem_u32(&full[st]), lead_rank); };
      auto load_w = [&](int st, int kb) {
#pragma unroll
        for (int mm = 0; mm < CF::NMMA; ++mm)
          tma_load_2d_2sm(sW + st * CF::kW + mm * CF::kBox * 128, &tmW, fb(st), kb * LBK,
                          n0 + mm * CF::NSUB + (int)sub * CF::kBox);
      };
      const int pre = nkb < S ? nkb : S;
      for (int kb = 0; kb < pre; ++kb) {          // weights first: independent of the previous kernel
        if (leader) mbar_expect_tx(&full[kb], 2 * CF::kStage);
        load_w(kb, kb);
      }
      pdl_wait();
      pdl_trigger();
      for (int kb = 0; kb < pre; ++kb) tma_load_2d_2sm(sA + kb * CF::kA, &tmA, fb(kb), kb * LBK, m0);
      int stage = pre % S;
      uint32_t phase = (pre == S) ? 1 : 0;
      for (int kb = pre; kb < nkb; ++kb) {
        mbar_wait(&empty[stage], phase ^ 1);
        if (leader) mbar_expect_tx(&full[stage], 2 * CF::kStage);
        tma_load_2d_2sm(sA + stage * CF::kA, &tmA, fb(stage), kb * LBK, m0);
        load_w(stage, kb);
        if (++stage == S) { stage = 0; phase ^= 1; }
      }
    } else {
      pdl_wait();
      pdl_trigger();
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer (pair leader)
    pdl_wait();
    pdl_trigger();
    if (leader && lane == 0) {
      constexpr uint32_t idesc = idesc_bf16_f32(2 * LM, CF::NSUB, 0);
      int stage = 0;
      uint32_t phase = 0;
      for (int kb = 0; kb < nkb; ++kb) {
        mbar_wait(&full[stage], phase);
        tc_fence_after();
        const uint64_t da = smem_desc_sw128(smem_u32(sA + stage * CF::kA), 16, 1024);
#pragma unroll
        for (int mm = 0; mm < CF::NMMA; ++mm) {
          const uint64_t db = smem_desc_sw128(smem_u32(sW + stage * CF::kW + mm * CF::kBox * 128), 16, 1024);
#pragma unroll
          for (int k = 0; k < LBK / 16; ++k)
            tc_mma2_f16(tmem_base + mm * CF::NSUB, da + (uint64_t)(2 * k), db + (uint64_t)(2 * k), idesc,
                        (kb | k) != 0);
        }
        tc_commit2_mc(&empty[stage], pair_mask);
        if (++stage == S) { stage = 0; phase ^= 1; }
      }
      tc_commit2_mc(tfull, pair_mask);
    }
  } else if (warp >= 4) {
    for (int i = threadIdx.x - 128; i < NH / 8; i += 256) {
      reinterpret_cast<uint4 *>(sPar)[i] = __ldg(reinterpret_cast<const uint4 *>(a.bias + n0) + i);
      reinterpret_cast<uint4 *>(sPar + NH)[i] = __ldg(reinterpret_cast<const uint4 *>(a.g + n0) + i);
      reinterpret_cast<uint4 *>(sPar + 2 * NH)[i] = __ldg(reinterpret_cast<const uint4 *>(a.b + n0) + i);
    }
    pdl_wait();
    pdl_trigger();
  }
  __syncwarp();

  // ---------------------------------------------------------------- epilogue
  const bool epi = warp >= 4;
  const int q = warp & 3, h = (warp - 4) >> 2;   // lane quarter, column half of this pair's NH
  const int row = q * 32 + lane;
  constexpr int HC = NH / 2;
  float2 sum2 = make_float2(0.f, 0.f), sq2 = make_float2(0.f, 0.f);
  if (epi) {
    mbar_wait(tfull, 0);                          // all MMAs done: the stage buffers are drained
    tc_fence_after();
    if (warp == 4 && lane == 0) {                 // the residual tile lands where y1 will be written
      mbar_expect_tx(rbar, LM * NH * 2);
      for (int blk = 0; blk < NH / 64; ++blk) tma_load_2d(sY + blk * (LM * 128), &tmR, rbar, n0 + blk * 64, m0);
    }
    epi_bar256();
    mbar_wait(rbar, 0);
    const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16);
#pragma unroll 1
    for (int c = 0; c < HC; c += 32) {
      const int col = h * HC + c;
      uint32_t r[32];
      tmem_ld32(taddr + col, r);
      uint8_t *blk = sY + (col / 64) * (LM * 128) + row * 128;
      const int ch0 = (col % 64) / 8;
      uint4 rv[4], bv[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        rv[j] = *reinterpret_cast<const uint4 *>(blk + (((ch0 + j) ^ (row & 7)) << 4));
        bv[j] = reinterpret_cast<const uint4 *>(sPar + col)[j];
      }
      tmem_wait_ld();
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t rw[4] = {rv[j].x, rv[j].y, rv[j].z, rv[j].w};
        const uint32_t bw[4] = {bv[j].x, bv[j].y, bv[j].z, bv[j].w};
        uint32_t o[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float2 acc2 = make_float2(__uint_as_float(r[j * 8 + 2 * e]), __uint_as_float(r[j * 8 + 2 * e + 1]));
          const float2 y2 = __fadd2_rn(__fadd2_rn(acc2, make_float2(bf_lo(bw[e]), bf_hi(bw[e]))),
                                       make_float2(bf_lo(rw[e]), bf_hi(rw[e])));
          o[e] = pack_bf16(y2.x, y2.y);
          const float2 yr = make_float2(bf_lo(o[e]), bf_hi(o[e]));   // statistics of the ROUNDED y1
          sum2 = __fadd2_rn(sum2, yr);
          sq2 = __ffma2_rn(yr, yr, sq2);
        }
        *reinterpret_cast<uint4 *>(blk + (((ch0 + j) ^ (row & 7)) << 4)) = make_uint4(o[0], o[1], o[2], o[3]);
      }
    }
    fence_proxy_async_smem();
    xs[h * LM + row] = sum2.x + sum2.y;
    xr2[h * LM + row] = sq2.x + sq2.y;
    epi_bar256();
    if (h == 0) {   // this CTA's (sum, sum of squares) -> slot [column half] here and in rank ^ 2
      const float s1 = xs[row] + xs[LM + row], s2 = xr2[row] + xr2[LM + row];
      xr1[2 * chalf * LM + 2 * row] = s1;
      xr1[2 * chalf * LM + 2 * row + 1] = s2;
      const uint32_t dst = mapa_shared(smem_u32(&xr1[2 * chalf * LM + 2 * row]), rank ^ 2u);
      asm volatile("st.shared::cluster.v2.f32 [%0], {%1, %2};" ::"r"(dst), "f"(s1), "f"(s2) : "memory");
    }
  }
  if (a.store_pre) {
    if (epi) epi_bar256();
    if (warp == 4 && lane == 0) {
      for (int blk = 0; blk < NH / 64; ++blk) tma_store_2d(&tmPre, sY + blk * (LM * 128), n0 + blk * 64, m0);
      bulk_commit();
    }
  }
  cluster_sync();                                 // both column halves' row statistics visible
  if (epi) {
    const float s1 = xr1[2 * row] + xr1[2 * LM + 2 * row], s2 = xr1[2 * row + 1] + xr1[2 * LM + 2 * row + 1];
    const float mean = s1 / (float)a.N;
    const float var = fmaxf(s2 / (float)a.N - mean * mean, 0.f);
    const float rstd = 1.0f / sqrtf(var + a.eps);
    const float2 nmean2 = make_float2(-mean, -mean), rstd2 = make_float2(rstd, rstd);
    if (a.store_pre) {
      if (warp == 4 && lane == 0) bulk_wait_read<0>();
      epi_bar256();
    }
#pragma unroll 1
    for (int c = 0; c < HC; c += 8) {
      const int col = h * HC + c;
      uint4 *p = reinterpret_cast<uint4 *>(sY + (col / 64) * (LM * 128) + row * 128 +
                                           ((((col % 64) / 8) ^ (row & 7)) << 4));
      const uint4 v = *p;
      const uint4 gv = *reinterpret_cast<const uint4 *>(sPar + NH + col);
      const uint4 bv = *reinterpret_cast<const uint4 *>(sPar + 2 * NH + col);
      const uint32_t w[4] = {v.x, v.y, v.z, v.w};
      const uint32_t gw[4] = {gv.x, gv.y, gv.z, gv.w};
      const uint32_t bw[4] = {bv.x, bv.y, bv.z, bv.w};
      uint32_t o[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 d2 = __fadd2_rn(make_float2(bf_lo(w[e]), bf_hi(w[e])), nmean2);
        const float2 t2 = __fmul2_rn(rstd2, make_float2(bf_lo(gw[e]), bf_hi(gw[e])));
        const float2 r2 = __ffma2_rn(d2, t2, make_float2(bf_lo(bw[e]), bf_hi(bw[e])));
        o[e] = pack_bf16(r2.x, r2.y);
      }
      *p = make_uint4(o[0], o[1], o[2], o[3]);
    }
    fence_proxy_async_smem();
    epi_bar256();
    if (warp == 4 && lane == 0) {
      for (int blk = 0; blk < NH / 64; ++blk) tma_store_2d(&tmOut, sY + blk * (LM * 128), n0 + blk * 64, m0);
      bulk_commit();
      bulk_wait_read<0>();                        // smem read before exit; the global writes complete with the grid
    }
  }
  tc_fence_before();
  cluster_sync();                                 // no CTA leaves while its peer may still signal it
  tc_fence_after();
  if (warp == 2) tmem_dealloc2(tmem_base, CF::kTmem);
  if (threadIdx.x == 0) tl_rec(tlb, 7, tl0, tl0);
}

template <int NH>
e3_status ln2_launch(const LnGemmMaps &m, const LnGemmArgs &a, cudaStream_t st) {
  auto kern = gemm_ln2_kernel<NH>;
  static bool attr_done = false;
  if (!attr_done) {
    E3_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, L2Cfg<NH>::kSmem));
    attr_done = true;
  }
  const int grid = 4 * ((a.M + 2 * LM - 1) / (2 * LM));
  E3_CUDA_TRY(launch_k(kern, dim3(grid), dim3(kLThreads), L2Cfg<NH>::kSmem, st, m.a, m.w2, m.r, m.pre, m.out, a));
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

bool ln2_enabled() {
  static const bool on = getenv("E3_LN_SINGLE") == nullptr;   // diagnostics: the 1-SM variant
  return on;
}

}  // namespace

bool ln_gemm_supported(int N, int K) {
  return K % LBK == 0 && (N == 128 || N == 256 || N == 384 || N == 512 || N == 640 || N == 768 || N == 1024);
}

e3_status ln_gemm_tmaps(LnGemmMaps *m, const void *A, const void *W, const void *R, const void *pre, const void *out,
                        int M, int N, int K) {
  const int NH = N / 2;
  const int nsub = NH / ((NH + 255) / 256);
  e3_status s = make_tmap_2d(&m->a, A, (uint64_t)M, (uint64_t)K, (uint64_t)K, LM, LBK);
  if (s == E3_OK) s = make_tmap_2d(&m->w, W, (uint64_t)N, (uint64_t)K, (uint64_t)K, (uint32_t)nsub, LBK);
  if (s == E3_OK) s = make_tmap_2d(&m->w2, W, (uint64_t)N, (uint64_t)K, (uint64_t)K, (uint32_t)(nsub / 2), LBK);
  if (s == E3_OK) s = make_tmap_2d(&m->out, out, (uint64_t)M, (uint64_t)N, (uint64_t)N, LM, 64);
  if (s == E3_OK) s = make_tmap_2d(&m->r, R, (uint64_t)M, (uint64_t)N, (uint64_t)N, LM, 64);
  if (s == E3_OK) s = make_tmap_2d(&m->pre, pre ? pre : out, (uint64_t)M, (uint64_t)N, (uint64_t)N, LM, 64);
  return s;
}

E3_TL_SETTER(tl_set_gemm_ln)

e3_status ln_gemm_run(const LnGemmMaps &m, const LnGemmArgs &a, cudaStream_t st) {
  // CTA-pair variant only where it measured faster (scripts/gemm_ln_bench.py,
  // B200, graph-replayed): N = 2048 rows of 1024 (BL shape) 50.2 vs 53.0 us;
  // at N = 768 (BB) the 1-SM kernel stays ahead, 16.4 vs 17.4 us -- the
  // halved W fill does not shorten a tile whose epilogue cannot overlap
  if (ln2_enabled() && a.N / 2 == 512) return ln2_launch<512>(m, a, st);
  switch (a.N / 2) {
    case 64: return ln_launch<64>(m, a, st);
    case 128: return ln_launch<128>(m, a, st);
    case 192: return ln_launch<192>(m, a, st);
    case 256: return ln_launch<256>(m, a, st);
    case 320: return ln_launch<320>(m, a, st);
    case 384: return ln_launch<384>(m, a, st);
    case 512: return ln_launch<512>(m, a, st);
  }
  set_error("fused projection + LayerNorm: unsupported width");
  return E3_EUNSUPPORTED;
}

}  // namespace e3
