// Layer GEMMs of the split on the sm_100a 5th-gen tensor
// cores: C[M,N] = epi(A[M,K] . W[N,K]^T), bf16 operands, fp32 accumulation in
// TMEM, one rounding to bf16 in the epilogue.
//
// Design (DESIGN.md §6 K1): CTA PAIRS (cluster of 2, cta_group::2).
//   * A pair owns a 256 x BN output tile (BN in {64,128,192,256}); CTA r of the
//     pair loads A rows [m0 + 128r, +128) and W rows [n0 + r*BN/2, +BN/2) per
//     64-wide K block by TMA (128-byte swizzle) into its own smem ring; the
//     completion bytes of both CTAs land on the LEADER's full barrier.  Per CTA
//     that is (128 + BN/2) x 128 B of smem fill per 128 x BN x 64 of MMA work,
//     twice the arithmetic intensity of a 1-SM 128 x BN tile (the L2 -> SM
//     fill rate, ~15 TB/s measured, otherwise caps the tensor pipe).
//   * the leader's single MMA thread issues tcgen05.mma.cta_group::2.kind::f16
//     256 x BN x 16; the hardware reads the A/W halves from both CTAs and
//     writes rows 0-127 of D to the leader's TMEM, rows 128-255 to the peer's;
//     tcgen05.commit multicasts "stage free" / "accumulator full" to both CTAs.
//   * persistent: pairs walk the tiles round-robin, n-fastest; two TMEM
//     accumulators (2*BN columns) so the epilogue of tile i overlaps the MMAs of
//     tile i+1; both CTAs' epilogue warps arrive on the leader's "accumulator
//     empty" barrier (remote mbarrier arrive through mapa).
//   * 8 epilogue warps per CTA; warp w owns TMEM lane quarter w % 4 (32 rows)
//     and one half of the BN columns, in chunks of 32 columns:
//     tcgen05.ld 32x32b.x32 -> +bias (+GELU | +residual, prefetched one chunk
//     ahead) -> bf16 -> 64-byte-swizzled smem staging (double buffered) ->
//     one TMA store of the 32 x 32 box.  Coalesced full-line writes instead of
//     32 scattered 16-byte stores per instruction (r01 measurement: the
//     scattered stores cost 8-25 us per GEMM launch).
#include "common.cuh"
#include "kernels.h"
#include "prof.h"

namespace e3 {

namespace {

constexpr int BM = 128;           // rows per CTA (256 per pair)
constexpr int BK = 64;            // K width of one 128-byte swizzle atom (TMA box)
constexpr int KSUB = 2;           // swizzle atoms per pipeline stage: 128-wide K stages
                                  // halve the per-MMA barrier / commit overhead
constexpr int kEpiBuf = 32 * 64;  // one 32 x 32 bf16 box
constexpr int kSmemMax = 232448;  // 227 KB opt-in limit

// Diagnostics: when e3_debug_gemm_trace() has set a device buffer, every CTA
// records globaltimer stamps per tile (<= kTrTiles tiles): [0] MMA issue
// start (accumulator free), [1] last commit issued, [2]/[3] epilogue warp 4
// start/end, [4]/[5] epilogue warp 11 start/end.
constexpr int kTrTiles = 16;
__device__ unsigned long long *g_gemm_trace = nullptr;
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void trace(int tile_local, int kind) {
  unsigned long long *b = g_gemm_trace;
  if (b && tile_local < kTrTiles) b[((size_t)blockIdx.x * kTrTiles + tile_local) * 6 + kind] = gtimer();
}

// Epilogue warps: 4 lane quarters x (BN / CW) column parts.  GELU: CW = 64
// columns per warp (two 32-column chunks), so a warp holds its whole share of
// the accumulator in registers and releases the TMEM buffer BEFORE the GELU
// math -- the MMA of tile i+2 no longer waits for the epilogue of tile i (r01
// trace, scripts/gemm_trace.py: with 8 warps the GELU epilogue took 4.1 us per
// 256 x 192 tile, as long as the tile's MMAs, and paced the kernel; FFN1
// 39.1 -> 37.8 us).  Bias and bias + residual keep 8 warps of BN / 2 columns
// released after the last chunk (the 12-warp variant measured 1 us slower on
// both N = 768 GEMMs: fewer pipeline stages fit beside its staging buffers).
template <int BN, int EPI>
struct Cfg {
  static constexpr int kEpiWarps = (EPI == E3_EPI_BIAS_GELU) ? 4 * (BN / 64) : (BN >= 128 ? 8 : 4);
  static constexpr int kCW = BN / (kEpiWarps / 4);       // columns per epilogue warp
  static constexpr int kNCW = kCW / 32;                  // 32-column chunks per warp
  static constexpr bool kEarly = kNCW <= 2;              // whole share in registers, early release
  static constexpr int kThreads = 128 + 32 * kEpiWarps;  // 4 control warps + epilogue warps
  static constexpr int kEpiBytes = kEpiWarps * 2 * kEpiBuf;
  // BN = 384 (a whole N = 768 GEMM in one wave of pair tiles): two N = 192
  // MMAs per K step, one TMEM accumulator (no epilogue overlap: one tile per
  // pair), 64-wide K stages so that four stages fit
  static constexpr int kNMma = BN > 256 ? 2 : 1;       // MMAs per k16 step (N <= 256 each)
  static constexpr int kNAcc = 2 * BN <= 512 ? 2 : 1;  // TMEM accumulators
  static constexpr int kKsub = BN > 256 ? 1 : KSUB;    // swizzle atoms per stage
  static constexpr int kBox = BN / (2 * kNMma);        // W rows per TMA box (one box per MMA per CTA)
  static constexpr int kASub = BM * BK * 2;            // 16 KB per swizzle atom column
  static constexpr int kBSub = (BN / 2) * BK * 2;      // this CTA's half of the W tile
  static constexpr int kABytes = kKsub * kASub;
  static constexpr int kBBytes = kKsub * kBSub;
  static constexpr int kStageBytes = kABytes + kBBytes;
  static constexpr int kStages = (kSmemMax - kEpiBytes - 1024 - 256) / kStageBytes;
  static constexpr int kTmemCols = (kNAcc * BN <= 128) ? 128 : (kNAcc * BN <= 256) ? 256 : 512;
  static constexpr int kSmem = kStages * kStageBytes + kEpiBytes + 1024 /*align*/ + 256 /*barriers*/;
};

// 64-byte swizzle of a [32 rows x 64 B] box: 16-byte chunk j of row r
__device__ __forceinline__ uint32_t sw64(int r, int j) { return r * 64 + ((j ^ ((r >> 1) & 3)) << 4); }

// MC (GEMM_MC_*): with multicast the cluster is two CTA pairs (ranks 0-1 and
// 2-3) walking 2-tile units in lockstep; the operand they share is loaded
// half by each pair and multicast to the same smem offset in both, so each
// CTA fetches (128 + BN/2) - 64 (A shared) or - BN/4 (W shared) rows per K
// element instead of 128 + BN/2 (ncu: 385 MB of L2 traffic per BB FFN1 at
// 31 % of the lts peak; cuBLAS's 2x2-cluster kernel moves 242 MB in the same
// time).  A stage is freed only when BOTH pairs' MMAs have read it (empty
// barriers count two commits, multicast to all four CTAs).  Off by default
// (E3_GEMM_MC): same results bit for bit, no faster (gemm_pick_bn).
template <int BN, int EPI, int MC>
__global__ void __cluster_dims__(MC ? 4 : 2, 1, 1) __launch_bounds__(Cfg<BN, EPI>::kThreads, 1)
    gemm_bf16_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                        const __grid_constant__ CUtensorMap tmC, const __nv_bfloat16 *__restrict__ bias,
                        const __nv_bfloat16 *__restrict__ R, int M, int N, int K) {
  using CF = Cfg<BN, EPI>;
  constexpr int S = CF::kStages;
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  extern __shared__ uint8_t smem_raw[];
  // identical layout (same offsets) in both CTAs of the pair
  // 1024-B aligned by offset arithmetic on the __shared__ array, so the
  // compiler keeps the shared address space (LDS / STS, not generic LD / ST)
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t *sA = smem;
  uint8_t *sB = smem + S * CF::kABytes;
  uint8_t *sE = smem + S * CF::kStageBytes;              // epilogue staging (1024-aligned)
  uint64_t *full = reinterpret_cast<uint64_t *>(sE + CF::kEpiBytes);
  uint64_t *empty = full + S;
  uint64_t *tfull = empty + S;        // [2]
  uint64_t *tempty = tfull + 2;       // [2]
  uint32_t *tmem_base_slot = reinterpret_cast<uint32_t *>(tempty + 2);

  const int warp = warp_id();
  const int lane = lane_id();
  constexpr int CL = MC ? 4 : 2;                 // CTAs per cluster
  const uint32_t rank = cluster_ctarank();
  const uint32_t rp = rank & 1;                  // rank within the pair
  const int pi = (int)(rank >> 1);               // pair within the cluster
  const bool leader = rp == 0;
  const uint32_t lead_rank = rank & ~1u;
  const int pair = blockIdx.x / CL;              // cluster index (one pair per cluster without MC)
  const int num_pairs = gridDim.x / CL;
  const int num_m = (M + 2 * BM - 1) / (2 * BM);
  const int num_n = N / BN;
  // work units: one pair tile (MC == 0) or two neighbouring tiles, one per pair
  const int num_tiles = MC == GEMM_MC_A ? num_m * (num_n / 2) : MC == GEMM_MC_B ? ((num_m + 1) / 2) * num_n
                                                                               : num_m * num_n;
  auto tile_m = [&](int t) { return MC == GEMM_MC_A ? t / (num_n / 2) : MC == GEMM_MC_B ? 2 * (t / num_n) + pi : t / num_n; };
  auto tile_n = [&](int t) { return MC == GEMM_MC_A ? 2 * (t % (num_n / 2)) + pi : t % num_n; };
  const uint16_t mc_mask = (uint16_t)((1u << rp) | (1u << (rp + 2)));   // this CTA's twin in the other pair
  const int num_kb = K / (BK * CF::kKsub);

  if (warp == 0 && lane == 0) {
    tma_prefetch(&tmA);
    tma_prefetch(&tmB);
    tma_prefetch(&tmC);
  }
  if (warp == 1 && lane == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);      // leader's arrive.expect_tx (bytes of both CTAs)
      mbar_init(&empty[i], MC ? 2 : 1);   // multicast tcgen05.commit of each pair's leader
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&tfull[i], 1);     // multicast tcgen05.commit
      mbar_init(&tempty[i], 2 * CF::kEpiWarps);   // epilogue warps of both CTAs (leader's copy is used)
    }
    fence_barrier_init();
  }
  if (warp == 2) tmem_alloc2(tmem_base_slot, CF::kTmemCols);
  tc_fence_before();
  cluster_sync();                  // peer barriers initialised, TMEM allocated in both CTAs
  tc_fence_after();
  const uint32_t tmem_base = *tmem_base_slot;
  if (warp != 0) {
    pdl_wait();                    // A / residual / C of the previous kernels now visible
    pdl_trigger();
  }
  const unsigned long long tl1 = tl_now();

  if (warp == 0) {
    // ------------------------------------------------ TMA producer (both CTAs)
    if (lane == 0) {
      // the W boxes of the first S stages do not depend on the previous
      // kernel: issued before griddepcontrol.wait, so the weight fetch
      // overlaps the hand-off; the A boxes of those stages follow the wait.
      // W rows of CTA r for MMA m: [n0 + m * BN / kNMma + r * kBox, + kBox),
      // so that D's columns map linearly onto the tile's N range
      auto load_w = [&](int st, int t, int kb) {
        const uint32_t fb = mapa_shared(smem_u32(&full[st]), lead_rank);
#pragma unroll
        for (int ks = 0; ks < CF::kKsub; ++ks)
#pragma unroll
          for (int m = 0; m < CF::kNMma; ++m) {
            const int wrow = tile_n(t) * BN + m * (BN / CF::kNMma) + (int)rp * CF::kBox;
            uint8_t *dst = sB + st * CF::kBBytes + ks * CF::kBSub + m * CF::kBox * 128;
            if (MC == GEMM_MC_B)   // half of the box from each pair, multicast to both
              tma_load_2d_2sm_mc(dst + pi * (CF::kBox / 2) * 128, &tmB, smem_u32(&full[st]),
                                 (kb * CF::kKsub + ks) * BK, wrow + pi * (CF::kBox / 2), mc_mask);
            else
              tma_load_2d_2sm(dst, &tmB, fb, (kb * CF::kKsub + ks) * BK, wrow);
          }
      };
      int npre = 0;
      for (int t = pair; t < num_tiles && npre < S; t += num_pairs) {
        for (int kb = 0; kb < num_kb && npre < S; ++kb, ++npre) {
          if (leader) mbar_expect_tx(&full[npre], 2 * CF::kStageBytes);
          load_w(npre, t, kb);
        }
      }
      pdl_wait();
      pdl_trigger();
      int stage = 0, it = 0;
      uint32_t phase = 0;
      for (int t = pair; t < num_tiles; t += num_pairs) {
        const int m_blk = tile_m(t);
        const int am = m_blk * 2 * BM + (int)rp * BM;
        for (int kb = 0; kb < num_kb; ++kb, ++it) {
          const uint32_t fb = mapa_shared(smem_u32(&full[stage]), lead_rank);
          const bool pre = it < npre;
          if (!pre) {
            mbar_wait(&empty[stage], phase ^ 1);
            if (leader) mbar_expect_tx(&full[stage], 2 * CF::kStageBytes);
          }
#pragma unroll
          for (int ks = 0; ks < CF::kKsub; ++ks) {
            if (MC == GEMM_MC_A)   // rows [64 pi, +64) of the block from this pair, multicast to both
              tma_load_2d_2sm_mc(sA + stage * CF::kABytes + ks * CF::kASub + pi * (BM / 2) * 128, &tmA,
                                 smem_u32(&full[stage]), (kb * CF::kKsub + ks) * BK, am + pi * (BM / 2), mc_mask);
            else
              tma_load_2d_2sm(sA + stage * CF::kABytes + ks * CF::kASub, &tmA, fb, (kb * CF::kKsub + ks) * BK, am);
          }
          if (!pre) load_w(stage, t, kb);
          if (++stage == S) { stage = 0; phase ^= 1; }
        }
      }
    } else {
      pdl_wait();
      pdl_trigger();
    }
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer (leader, one thread)
    if (leader && lane == 0) {
      constexpr uint32_t idesc = idesc_bf16_f32(2 * BM, BN / CF::kNMma, 0);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      int tl = 0;
      for (int t = pair; t < num_tiles; t += num_pairs, ++tl) {
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        trace(tl, 0);
        const uint32_t d_tmem = tmem_base + acc * BN;
        for (int kb = 0; kb < num_kb; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
#pragma unroll
          for (int ks = 0; ks < CF::kKsub; ++ks) {
            const uint64_t da = smem_desc_sw128(smem_u32(sA + stage * CF::kABytes + ks * CF::kASub), 16, 1024);
#pragma unroll
            for (int m = 0; m < CF::kNMma; ++m) {
              const uint64_t db =
                  smem_desc_sw128(smem_u32(sB + stage * CF::kBBytes + ks * CF::kBSub + m * CF::kBox * 128), 16, 1024);
#pragma unroll
              for (int k = 0; k < BK / 16; ++k)   // +32 bytes per 16-element K step inside the swizzle atom
                tc_mma2_f16(d_tmem + m * (BN / CF::kNMma), da + (uint64_t)(2 * k), db + (uint64_t)(2 * k), idesc,
                            (kb | ks | k) != 0);
            }
          }
          tc_commit2_mc(&empty[stage], MC ? 0xF : 0x3);   // both pairs' stages (MC: they share it)
          if (++stage == S) { stage = 0; phase ^= 1; }
        }
        tc_commit2_mc(&tfull[acc], (uint16_t)(0x3u << (2 * pi)));
        trace(tl, 1);
        if (++acc == CF::kNAcc) { acc = 0; acc_phase ^= 1; }
      }
    }
  } else if (warp >= 4) {
    // ------------------------------------------------ epilogue (both CTAs)
    constexpr int CW = CF::kCW, NCW = CF::kNCW;
    const int q = warp & 3;              // TMEM lane quarter this warp may access
    const int part = (warp - 4) >> 2;    // which CW-column part of the tile
    uint8_t *ebuf = sE + (warp - 4) * 2 * kEpiBuf;
    const uint32_t tempty_leader0 = mapa_shared(smem_u32(&tempty[0]), lead_rank);
    const uint32_t tempty_leader1 = mapa_shared(smem_u32(&tempty[1]), lead_rank);
    int acc = 0;
    uint32_t acc_phase = 0;
    int ci = 0;                          // chunk counter (selects the staging buffer)
    int tl = 0;
    for (int t = pair; t < num_tiles; t += num_pairs, ++tl) {
      const int m_blk = tile_m(t), n_blk = tile_n(t);
      const int m0 = m_blk * 2 * BM + (int)rp * BM + q * 32;     // this warp's first row
      const int m = m0 + lane;
      const int nw0 = n_blk * BN + part * CW;                     // this warp's first column
      const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN + part * CW;
      uint4 rnext[4];
      if (EPI == E3_EPI_BIAS_RESID) {
        const uint4 *rp = reinterpret_cast<const uint4 *>(R + (size_t)m * N + nw0);
#pragma unroll
        for (int j = 0; j < 4; ++j) rnext[j] = (m < M) ? __ldg(rp + j) : make_uint4(0, 0, 0, 0);
      }
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      if (lane == 0 && (warp == 4 || warp == 11)) trace(tl, warp == 4 ? 2 : 4);
      uint32_t racc[CF::kEarly ? NCW : 1][32];
      if (CF::kEarly) {
        // whole share -> registers, then hand the accumulator back to the MMA
#pragma unroll
        for (int c = 0; c < NCW; ++c) tmem_ld32(taddr + c * 32, racc[c]);
        tmem_wait_ld();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive_cluster(acc ? tempty_leader1 : tempty_leader0);
      }
#pragma unroll
      for (int c = 0; c < NCW; ++c) {
        const int n0 = nw0 + c * 32;
        uint32_t rl[32];
        const uint32_t *r = CF::kEarly ? racc[CF::kEarly ? c : 0] : rl;
        if (!CF::kEarly) tmem_ld32(taddr + c * 32, rl);
        uint4 rcur[4];
        if (EPI == E3_EPI_BIAS_RESID) {
#pragma unroll
          for (int j = 0; j < 4; ++j) rcur[j] = rnext[j];
          if (c + 1 < NCW) {              // prefetch the next chunk's residual
            const uint4 *rp = reinterpret_cast<const uint4 *>(R + (size_t)m * N + n0 + 32);
#pragma unroll
            for (int j = 0; j < 4; ++j) rnext[j] = (m < M) ? __ldg(rp + j) : make_uint4(0, 0, 0, 0);
          }
        }
        if (!CF::kEarly) tmem_wait_ld();
        float v[32];
        const uint4 *bp = reinterpret_cast<const uint4 *>(bias + n0);
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const uint4 b4 = __ldg(bp + j);
          const uint32_t bw[4] = {b4.x, b4.y, b4.z, b4.w};
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            v[j * 8 + 2 * e] = __uint_as_float(r[j * 8 + 2 * e]) + bf_lo(bw[e]);
            v[j * 8 + 2 * e + 1] = __uint_as_float(r[j * 8 + 2 * e + 1]) + bf_hi(bw[e]);
          }
        }
        if (EPI == E3_EPI_BIAS_GELU) {
#pragma unroll
          for (int j = 0; j < 32; j += 2) {
            const float2 gv = gelu_fast2(make_float2(v[j], v[j + 1]));
            v[j] = gv.x;
            v[j + 1] = gv.y;
          }
        }
        if (EPI == E3_EPI_BIAS_RESID) {
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const uint32_t rw[4] = {rcur[j].x, rcur[j].y, rcur[j].z, rcur[j].w};
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              v[j * 8 + 2 * e] += bf_lo(rw[e]);
              v[j * 8 + 2 * e + 1] += bf_hi(rw[e]);
            }
          }
        }
        // stage: buffer (ci & 1) was last used by chunk ci-2; its TMA store must
        // have finished reading smem
        uint8_t *buf = ebuf + (ci & 1) * kEpiBuf;
        if (lane == 0) bulk_wait_read<1>();
        __syncwarp();
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          uint4 o;
          o.x = pack_bf16(v[j * 8 + 0], v[j * 8 + 1]);
          o.y = pack_bf16(v[j * 8 + 2], v[j * 8 + 3]);
          o.z = pack_bf16(v[j * 8 + 4], v[j * 8 + 5]);
          o.w = pack_bf16(v[j * 8 + 6], v[j * 8 + 7]);
          *reinterpret_cast<uint4 *>(buf + sw64(lane, j)) = o;
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) {
          tma_store_2d(&tmC, buf, n0, m0);   // rows >= M are clipped by the tensor map
          bulk_commit();
        }
        ++ci;
      }
      if (!CF::kEarly) {
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive_cluster(acc ? tempty_leader1 : tempty_leader0);
      }
      if (lane == 0 && (warp == 4 || warp == 11)) trace(tl, warp == 4 ? 3 : 5);
      if (++acc == CF::kNAcc) { acc = 0; acc_phase ^= 1; }
    }
    if (lane == 0) bulk_wait_read<0>();   // smem read before exit; the global writes complete with the grid
  }
  tc_fence_before();
  cluster_sync();                  // no CTA leaves while its peer may still signal it
  tc_fence_after();
  if (warp == 2) tmem_dealloc2(tmem_base, CF::kTmemCols);
  if (threadIdx.x == 0) tl_rec(tlb, 1000 + BN + EPI, tl0, tl1);
}

template <int BN, int EPI, int MC>
e3_status launch(const GemmMaps &g, const __nv_bfloat16 *bias, const __nv_bfloat16 *R, int M, int N, int K, int sms,
                 cudaStream_t st) {
  auto kern = gemm_bf16_tc_kernel<BN, EPI, MC>;
  using CF = Cfg<BN, EPI>;
  constexpr int CL = MC ? 4 : 2;
  static int max_clusters = 0;     // per instantiation: clusters of CL CTAs resident at once
  if (!max_clusters) {
    E3_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, CF::kSmem));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(CL * 64);
    cfg.blockDim = dim3(CF::kThreads);
    cfg.dynamicSmemBytes = CF::kSmem;
    int n = 0;
    if (cudaOccupancyMaxActiveClusters(&n, kern, &cfg) != cudaSuccess || n <= 0) {
      cudaGetLastError();
      n = sms / CL;
    }
    max_clusters = n < sms / CL ? n : sms / CL;
  }
  const int num_m = (M + 2 * BM - 1) / (2 * BM), num_n = N / BN;
  const int units = MC == GEMM_MC_A ? num_m * (num_n / 2) : MC == GEMM_MC_B ? ((num_m + 1) / 2) * num_n : num_m * num_n;
  const int clusters = units < max_clusters ? units : max_clusters;
  E3_CUDA_TRY(launch_k(kern, dim3(CL * clusters), dim3(CF::kThreads), CF::kSmem, st, g.a, g.b, g.c, bias, R, M, N, K));
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

template <int BN, int MC>
e3_status launch_epi(int epi, const GemmMaps &g, const __nv_bfloat16 *bias, const __nv_bfloat16 *R, int M, int N,
                     int K, int sms, cudaStream_t st) {
  if (BN > 256) {   // 384: bias / residual epilogues only
    if (epi == E3_EPI_BIAS) return launch<(BN > 256 ? BN : 384), E3_EPI_BIAS, MC>(g, bias, R, M, N, K, sms, st);
    if (epi == E3_EPI_BIAS_RESID)
      return launch<(BN > 256 ? BN : 384), E3_EPI_BIAS_RESID, MC>(g, bias, R, M, N, K, sms, st);
    set_error("GEMM: N tile 384 has no GELU epilogue");
    return E3_EUNSUPPORTED;
  }
  switch (epi) {
    case E3_EPI_BIAS: return launch<BN, E3_EPI_BIAS, MC>(g, bias, R, M, N, K, sms, st);
    case E3_EPI_BIAS_GELU: return launch<BN, E3_EPI_BIAS_GELU, MC>(g, bias, R, M, N, K, sms, st);
    case E3_EPI_BIAS_RESID: return launch<BN, E3_EPI_BIAS_RESID, MC>(g, bias, R, M, N, K, sms, st);
  }
  set_error("bad epilogue");
  return E3_EINVAL;
}

template <int BN>
e3_status launch_mc(int mc, int epi, const GemmMaps &g, const __nv_bfloat16 *bias, const __nv_bfloat16 *R, int M,
                    int N, int K, int sms, cudaStream_t st) {
  switch (mc) {
    case GEMM_MC_NONE: return launch_epi<BN, GEMM_MC_NONE>(epi, g, bias, R, M, N, K, sms, st);
    case GEMM_MC_A: return launch_epi<BN, GEMM_MC_A>(epi, g, bias, R, M, N, K, sms, st);
    case GEMM_MC_B: return launch_epi<BN, GEMM_MC_B>(epi, g, bias, R, M, N, K, sms, st);
  }
  set_error("bad GEMM multicast mode");
  return E3_EINVAL;
}

}  // namespace

E3_TL_SETTER(tl_set_gemm)

e3_status gemm_set_trace(void *buf) {
  E3_CUDA_TRY(cudaMemcpyToSymbol(g_gemm_trace, &buf, sizeof(buf)));
  return E3_OK;
}

int gemm_pick_bn(int M, int N, int K, int sms, int epi) {
  // diagnostics: E3_GEMM_BN forces the N tile where it divides N, E3_GEMM_MC
  // the multicast mode (0 none, 1 A, 2 W) where it applies
  static const int forced = [] {
    const char *e = getenv("E3_GEMM_BN");
    return e ? atoi(e) : 0;
  }();
  static const int forced_mc = [] {
    const char *e = getenv("E3_GEMM_MC");
    return e ? atoi(e) : -1;
  }();
  // Minimise waves x per-tile cost over the pair tiles (256 x BN), in units
  // of one row of TMA fill per K element.  The mainloop is bound by the L2 ->
  // SM fill (the chip-wide LTS cap, ~42 B/clk per SM) or by the MMA (BN / 32
  // clk per K element per pair = 1.31 BN fill rows), whichever is slower: a
  // pair fetches 256 + BN rows per K element, 128 + BN with A multicast, 256 +
  // BN / 2 with W multicast.  The issue-bound GELU epilogue adds ~ BN / 2 per
  // K step, and BN = 384 (one TMEM accumulator: nothing to overlap its
  // epilogue with) pays ~ 1720 x BN for the exposed epilogue.  Calibrated on
  // scripts/gemm_bn_sweep*.sh: BL N = 1024 FFN2 102 us at BN 256 (120 at 128);
  // BB FFN1 + GELU 37.8 us at 192 (38.9 at 256); BB FFN2 (K = 3072) 31.6 us
  // at 384 (33.0 at 192) but BB O (K = 768) 14.1 us at 192 (14.8 at 384).
  int best = 0;
  long long best_cost = 0;
  const int cands[5] = {384, 256, 192, 128, 64};
  const int pairs = sms / 2;
  const int num_m = (M + 2 * BM - 1) / (2 * BM);
  for (int i = 0; i < 5; ++i) {
    const int bn = cands[i];
    if (N % bn || (bn == 384 && epi == E3_EPI_BIAS_GELU)) continue;
    if (forced && bn != forced) continue;
    const int num_n = N / bn;
    // multicast only on request: measured bitwise-equal but not faster on the
    // B200 (scripts/gemm_mc_check.py: BB FFN1 + GELU 34.9 us unicast, 36.8 A
    // multicast, 37.1 W multicast; FFN2 31.4 / 30.7 / 31.1; QKV 23.0 / - /
    // 24.8): the mainloop is bound by the bytes one SM keeps in flight (three
    // 56 KB stages beside the epilogue staging), not by the chip's L2 output
    for (int mc = 0; mc < (forced_mc > 0 ? 3 : 1); ++mc) {
      if (forced_mc >= 0 && mc != forced_mc) continue;
      if (mc == GEMM_MC_A && num_n % 2) continue;
      if (mc == GEMM_MC_B && num_m < 2) continue;
      const long long units = mc == GEMM_MC_A   ? (long long)num_m * (num_n / 2)
                              : mc == GEMM_MC_B ? (long long)((num_m + 1) / 2) * num_n
                                                : (long long)num_m * num_n;
      const long long slots = mc ? pairs / 2 : pairs;
      const long long waves = (units + slots - 1) / slots;
      const long long fill = (mc == GEMM_MC_A ? 128 : 256) + (mc == GEMM_MC_B ? bn / 2 : bn);
      const long long mma = (long long)bn * 21 / 16;
      const long long tile = (long long)K * (fill > mma ? fill : mma) +
                             (epi == E3_EPI_BIAS_GELU ? (long long)K * bn / 2 : 0) + (bn > 256 ? 1720LL * bn : 0);
      const long long cost = waves * tile;
      if (best == 0 || cost < best_cost) { best = bn | (mc << 12); best_cost = cost; }
    }
  }
  if (!best) {   // a forced combination that does not apply: the first N tile that divides N
    for (int i = 0; i < 5 && !best; ++i)
      if (N % cands[i] == 0 && !(cands[i] == 384 && epi == E3_EPI_BIAS_GELU)) best = cands[i];
  }
  return best;
}

e3_status gemm_tmaps(GemmMaps *g, const void *A, int64_t lda, const void *W, const void *C, int M, int N, int K,
                     int code) {
  const int bn = code & 0xFFF, mc = code >> 12;
  const uint32_t wbox = (uint32_t)(bn > 256 ? bn / 4 : bn / 2) / (mc == GEMM_MC_B ? 2 : 1);
  e3_status s = make_tmap_2d(&g->a, A, (uint64_t)M, (uint64_t)K, (uint64_t)lda, mc == GEMM_MC_A ? BM / 2 : BM, BK);
  if (s == E3_OK) s = make_tmap_2d(&g->b, W, (uint64_t)N, (uint64_t)K, (uint64_t)K, wbox, BK);
  if (s == E3_OK) s = make_tmap_2d_sw64(&g->c, C, (uint64_t)M, (uint64_t)N, (uint64_t)N, 32, 32);
  g->bn = code;
  return s;
}

e3_status gemm_run(const GemmMaps &g, const void *bias, const void *R, int M, int N, int K, int epi, int sms,
                   cudaStream_t st) {
  auto *b = reinterpret_cast<const __nv_bfloat16 *>(bias);
  auto *r = reinterpret_cast<const __nv_bfloat16 *>(R);
  const int bn = g.bn & 0xFFF, mc = g.bn >> 12;
  switch (bn) {
    case 384: return launch_mc<384>(mc, epi, g, b, r, M, N, K, sms, st);
    case 256: return launch_mc<256>(mc, epi, g, b, r, M, N, K, sms, st);
    case 192: return launch_mc<192>(mc, epi, g, b, r, M, N, K, sms, st);
    case 128: return launch_mc<128>(mc, epi, g, b, r, M, N, K, sms, st);
    case 64: return launch_mc<64>(mc, epi, g, b, r, M, N, K, sms, st);
  }
  set_error("unsupported GEMM N tile");
  return E3_EUNSUPPORTED;
}

}  // namespace e3
