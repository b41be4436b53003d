// Decode-shaped GEMMs of the LLaMA split:
//     Y[T, N] = epi( X[T, K] . W[N, K]^T ),   T = tokens of the batch (32..128)
// bf16 operands, fp32 accumulation in TMEM.
//
// T is far below one MMA tile and the weights are read exactly once per
// launch, so the path is bound by streaming W from HBM (405 MB per Llama-7B
// layer).  Design (DESIGN.md §6 K7):
//   * SWAP AB: the weight tile is the MMA's M side (128 rows of W), the
//     tokens are its N side: D[128, T] = W_tile . X^T with both operands
//     K-major in 128-byte-swizzled smem, tcgen05.mma.cta_group::1 M=128 N=T.
//     No padding of T up to a 128-row tile, no wasted tensor work.
//   * stream-K: one CTA per SM, each taking an equal contiguous range of the
//     (tile, 64-wide k-block) iterations, so every SM streams the same weight
//     bytes (a tile-granular split left SMs idle: W_o / W_down have only 32
//     tiles).  Tiles split between CTAs are finished by their last
//     contributor (atomic ticket), summing the contributors' fp32 partials in
//     contributor order (deterministic).
//   * warp 0 = TMA producer: the first stages' W boxes are issued BEFORE
//     griddepcontrol.wait (weights never depend on the previous kernel), so
//     the weight stream starts while the previous kernel drains; warp 1 = one
//     MMA thread; warps 2-5 = epilogue (TMEM lane quarter = warp % 4), through
//     an fp32 smem tile [128][T+1].
//   * epilogues: STORE, RESID (+ residual), SWIGLU (tile rows 0-63 = W_gate
//     rows, 64-127 = the matching W_up rows, two TMA boxes per stage; out =
//     SiLU(g) * u), QKV_ROPE (one head per tile since head_dim = 128: rotate
//     pairs (j, j+64) with a cos/sin table of exact angles, q -> Q buffer, k/v
//     -> the KV cache at (slot, pos) of each token), LOGITS (fp32 logits + per
//     tile softmax statistics (max, sum e, sum e*(z-max), argmax) per token).
#include <cmath>
#include <vector>

#include "common.cuh"
#include "kernels.h"
#include "prof.h"

namespace e3 {

namespace {

#ifndef E3_DEC_NO_LL
#define E3_DEC_NO_LL 0                // diagnostics builds: last-arrival reduction for every shared tile
#endif
constexpr int DM = 128;            // weight rows per tile (MMA M)
constexpr int DK = 64;             // K per 128-byte swizzle atom / TMA box
constexpr int DKS = 2 * DK;        // K per pipeline stage: two atoms, so the two 128-byte
                                   // pieces of a weight row are requested back to back
constexpr int kDThreads = 224;     // warp 0 W TMA, warp 1 MMA, warps 2-5 epilogue, warp 6 X TMA
constexpr int kSmemMax = 232448;

template <int T>
// Separate rings for W (HBM: deep, 9 stages at T = 64) and X (L2-resident
// tokens: 4 stages), each with its own producer warp: one shared ring of
// W + X stages held 7 x 16 KB of weights in flight per SM
struct DCfg {
  static constexpr int kWAtom = DM * DK * 2;                // 16 KB
  static constexpr int kXAtom = T * DK * 2;
  static constexpr int kWBytes = 2 * kWAtom;
  static constexpr int kXBytes = 2 * kXAtom;
  static constexpr int kXStages = T <= 64 ? 3 : 2;   // the third X stage is free at T <= 64 (same 4 W stages)
  static constexpr int kEBytes = DM * (T + 1) * 4;          // fp32 epilogue tile
  static constexpr int kStages = (kSmemMax - kEBytes - 1024 - 3072 - kXStages * kXBytes) / kWBytes;
  static constexpr int kTmemCols = (2 * T <= 32) ? 32 : (2 * T <= 64) ? 64 : (2 * T <= 128) ? 128 : 256;
  static constexpr int kSmem = kStages * kWBytes + kXStages * kXBytes + kEBytes + 1024 + 3072;   // + barriers, token tables
  static_assert(kStages >= 2, "weight ring too shallow");
};

__device__ __forceinline__ void epi_bar() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

// Stream-K work split: the tiles x (K / 64) k-block iterations are cut into
// gridDim.x equal contiguous ranges, one per CTA, so every SM streams the same
// number of weight bytes (with 96..250 tiles per launch a tile-granular split
// leaves up to half the SMs idle for the last wave).  A CTA's range crosses at
// most a few tiles; a tile computed by one CTA is finished in place, a tile
// shared by several CTAs is reduced by its last contributor (atomic ticket)
// from the contributors' fp32 partials in contributor order (deterministic).
struct SK {
  long total;   // tiles * nkb
  int nkb, G;
  __device__ long start(int c) const { return (long)c * total / G; }
  __device__ int owner(long i) const {   // CTA whose range holds iteration i
    int c = (int)((i * G) / total);
    while (c + 1 < G && start(c + 1) <= i) ++c;
    while (c > 0 && start(c) > i) --c;
    return c;
  }
};

__device__ __forceinline__ float ld_dsmem_f32(uint32_t addr) {
  float v;
  asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(addr) : "memory");
  return v;
}

// CSK > 1: cluster split-K instead of stream-K (the narrow W_o / W_down,
// 32 tiles): a cluster of CSK CTAs per tile, CTA r summing k-blocks
// [r nkb / CSK, (r + 1) nkb / CSK); the fp32 partial tiles stay in each CTA's
// smem and CTA r reduces rows [r 128 / CSK, +128 / CSK) of the tile over the
// cluster through DSMEM in rank order (deterministic; every tile has the same
// split, so a row's rounding does not depend on its position), then runs the
// epilogue on those rows.  No global partials, tickets or fences: the stream-K
// fixup cost ~5 us after the mainloop on these shapes (r01 dec_timeline).
template <int T, int EPI, int CSK>
__global__ void __launch_bounds__(kDThreads, 1)
    gemm_dec_kernel(const __grid_constant__ CUtensorMap tmW, const __grid_constant__ CUtensorMap tmW2,
                    const __grid_constant__ CUtensorMap tmX, DecArgs a) {
  using CF = DCfg<T>;
  constexpr int S = CF::kStages;
  constexpr int P = T + 1;
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  extern __shared__ uint8_t smem_raw[];
  // 1024-B aligned by offset arithmetic on the __shared__ array, so the
  // compiler keeps the shared address space (LDS / STS, not generic LD / ST)
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  constexpr int XS = CF::kXStages;
  uint8_t *sW = smem;
  uint8_t *sX = smem + S * CF::kWBytes;
  float *sE = reinterpret_cast<float *>(sX + XS * CF::kXBytes);
  uint64_t *full = reinterpret_cast<uint64_t *>(reinterpret_cast<uint8_t *>(sE) + CF::kEBytes);
  uint64_t *empty = full + S;
  uint64_t *xfull = empty + S;     // [XS]
  uint64_t *xempty = xfull + XS;   // [XS]
  uint64_t *tfull = xempty + XS;   // [2]
  uint64_t *tempty = tfull + 2;    // [2]
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(tempty + 2);
  int *s_last = reinterpret_cast<int *>(tmem_slot + 1);
  int *sPos = s_last + 1;          // [T]
  int *sSlot = sPos + T;           // [T]
  int64_t *sTok = reinterpret_cast<int64_t *>(sSlot + T + (T & 1));   // [T] LOGITS: exit-record row of token t

  const int warp = warp_id(), lane = lane_id();
  const int tiles = (EPI == E3_DEC_SWIGLU) ? a.N / 64 : (a.N + DM - 1) / DM;
  constexpr bool kCluster = CSK > 1 && EPI != E3_DEC_PARTIAL;
  SK sk;
  sk.nkb = a.K / DKS;
  sk.total = (long)tiles * sk.nkb;
  sk.G = gridDim.x;
  long my0, my1;
  if (CSK > 1) {
    const long tile = blockIdx.x / CSK, rr = blockIdx.x % CSK;   // rr == cluster rank (cluster dims CSK x 1 x 1)
    my0 = tile * sk.nkb + rr * sk.nkb / CSK;
    my1 = tile * sk.nkb + (rr + 1) * sk.nkb / CSK;
  } else {
    my0 = sk.start(blockIdx.x);
    my1 = sk.start(blockIdx.x + 1);
  }

  if (warp == 0 && lane == 0) {
    tma_prefetch(&tmW);
    if (EPI == E3_DEC_SWIGLU) tma_prefetch(&tmW2);
    tma_prefetch(&tmX);
  }
  if (warp == 1 && lane == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < XS; ++i) {
      mbar_init(&xfull[i], 1);
      mbar_init(&xempty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&tfull[i], 1);
      mbar_init(&tempty[i], 4);    // 4 epilogue warps
    }
    fence_barrier_init();
  }
  if (warp == 2) tmem_alloc(tmem_slot, CF::kTmemCols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------- TMA producer
    if (lane == 0) {
      const int total = (int)(my1 - my0);
      auto load_w = [&](int it, int st) {
        const long i = my0 + it;
        const int tile = (int)(i / sk.nkb), k0 = (int)(i % sk.nkb) * DKS;
#pragma unroll
        for (int sub = 0; sub < 2; ++sub) {
          uint8_t *dst = sW + st * CF::kWBytes + sub * CF::kWAtom;
          if (EPI == E3_DEC_SWIGLU) {
            tma_load_2d(dst, &tmW, &full[st], k0 + sub * DK, tile * 64);
            tma_load_2d(dst + CF::kWAtom / 2, &tmW2, &full[st], k0 + sub * DK, tile * 64);
          } else {
            tma_load_2d(dst, &tmW, &full[st], k0 + sub * DK, tile * DM);
          }
        }
      };
      const int pre = total < S ? total : S;
      // weights first: they do not depend on the previous kernel
      for (int it = 0; it < pre; ++it) {
        mbar_expect_tx(&full[it], CF::kWBytes);
        load_w(it, it);
      }
      pdl_wait();
      if (!a.late_trigger) pdl_trigger();
      int stage = pre % S;
      uint32_t phase = (pre == S) ? 1 : 0;
      for (int it = pre; it < total; ++it) {
        mbar_wait(&empty[stage], phase ^ 1);
        mbar_expect_tx(&full[stage], CF::kWBytes);
        load_w(it, stage);
        if (++stage == S) { stage = 0; phase ^= 1; }
      }
    }
  } else if (warp == 6) {
    // ------------------------------------------------------- X (tokens) producer
    pdl_wait();
    if (!a.late_trigger) pdl_trigger();
    if (lane == 0) {
      const int total = (int)(my1 - my0);
      int xs = 0;
      uint32_t xphase = 0;
      for (int it = 0; it < total; ++it) {
        mbar_wait(&xempty[xs], xphase ^ 1);
        mbar_expect_tx(&xfull[xs], CF::kXBytes);
#pragma unroll
        for (int sub = 0; sub < 2; ++sub)
          tma_load_2d(sX + xs * CF::kXBytes + sub * CF::kXAtom, &tmX, &xfull[xs],
                      (int)((my0 + it) % sk.nkb) * DKS + sub * DK, 0);
        if (++xs == XS) { xs = 0; xphase ^= 1; }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------- MMA issuer
    pdl_wait();
    if (!a.late_trigger) pdl_trigger();
    if (lane == 0) {
      constexpr uint32_t idesc = idesc_bf16_f32(DM, T, 0);
      int stage = 0, xs = 0;
      uint32_t phase = 0, xphase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      for (long i = my0; i < my1;) {                 // one segment = this CTA's part of one tile
        const int tile = (int)(i / sk.nkb);
        const long seg_end = min(my1, (long)(tile + 1) * sk.nkb);
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * T;
        for (long j = i; j < seg_end; ++j) {
          mbar_wait(&full[stage], phase);
          mbar_wait(&xfull[xs], xphase);
          tc_fence_after();
#pragma unroll
          for (int sub = 0; sub < 2; ++sub) {
            const uint64_t da = smem_desc_sw128(smem_u32(sW + stage * CF::kWBytes + sub * CF::kWAtom), 16, 1024);
            const uint64_t db = smem_desc_sw128(smem_u32(sX + xs * CF::kXBytes + sub * CF::kXAtom), 16, 1024);
#pragma unroll
            for (int k = 0; k < DK / 16; ++k)
              tc_mma_f16(d_tmem, da + (uint64_t)(2 * k), db + (uint64_t)(2 * k), idesc, (j != i) || sub != 0 || k != 0);
          }
          tc_commit(&empty[stage]);
          tc_commit(&xempty[xs]);
          if (++stage == S) { stage = 0; phase ^= 1; }
          if (++xs == XS) { xs = 0; xphase ^= 1; }
        }
        tc_commit(&tfull[acc]);
        if (++acc == 2) { acc = 0; acc_phase ^= 1; }
        i = seg_end;
      }
    }
  } else {
    // ------------------------------------------------------- epilogue (warps 2-5)
    pdl_wait();
    if (!a.late_trigger) pdl_trigger();
    const unsigned long long tl1 = tl_now();
    unsigned long long tlf = 0, tlm = 0;   // first / last accumulator ready
    const int q = warp & 3;
    const int r = q * 32 + lane;       // weight row of the tile == TMEM lane
    const int et = threadIdx.x - 64;   // 0..127
    if (EPI == E3_DEC_LOGITS) {
      const int nv = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
      for (int t = et; t < T; t += 128) {
        const int64_t id = a.ids ? a.ids[t] : -1;
        // only rows still alive at this ramp (a row that exited at an inner
        // ramp of the split keeps that ramp's logits)
        const bool live = t < nv && (a.init_alive || a.alive[t] != 0);
        sTok[t] = (live && id >= 0 && id < a.id_cap) ? id : -1;
      }
      epi_bar();
    }
    if (EPI == E3_DEC_QKV_ROPE) {
      const int nv = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
      for (int t = et; t < T; t += 128) {
        int pos = 0, slot = -1;
        const int64_t id = a.ids[t];
        // a row that exited at an earlier ramp of this split writes no K/V for
        // the layers it skips (R15; oracle.llama.run_split)
        const bool live = t < nv && (a.init_alive || a.alive == nullptr || a.alive[t] != 0);
        if (live && id >= 0 && id < a.id_cap) {
          slot = a.slot_of_id[id];
          if (slot < 0 || slot >= a.n_slots) {
            slot = -1;
            if (a.err) *a.err = 1;
          } else {
            pos = a.pos_of_slot[slot];
            if (pos < 0 || pos >= a.max_ctx) {
              slot = -1;
              pos = 0;
              if (a.err) *a.err = 1;
            }
          }
        }
        sPos[t] = pos;
        sSlot[t] = slot;
      }
      epi_bar();
    }
    int acc = 0;
    uint32_t acc_phase = 0;
    for (long i = my0; i < my1;) {
      const int tile = (int)(i / sk.nkb);
      const long t0i = (long)tile * sk.nkb, t1i = t0i + sk.nkb;
      const long seg_end = min(my1, t1i);
      const bool whole = (i == t0i) && (seg_end == t1i);
      i = seg_end;
      // Early fetch (T <= 64, two contributors): while this segment's MMAs
      // still run, look whether the tile's other contributor already
      // published its partial (the usual case for a CTA's last segment: the
      // head of a tile whose tail the next CTA computed first).  If so this
      // CTA is the tile's last arrival; the other partial is loaded into
      // registers now, so the reduction after the accumulator lands costs no
      // memory round trip on the kernel's critical path.
      bool early = false;
      int early_slot = 0;
      // Two contributors whose ranges BOTH end in this tile (with 3 ranges per
      // 2 tiles, every other tile): fixed roles instead of "last arrival
      // reduces" -- the head (slot 0) publishes its partial without reading
      // the ticket first, the tail (slot 1, this tile is its whole range)
      // waits for it and adds it as in the early fetch.  Before, both often
      // arrived together and each paid ticket read + partial write + fence +
      // atomic before either could reduce (~4.6 us, dec_segments).  The tail
      // waits only on the head's mainloop, which depends on nothing else.
      bool ll = false;
      if (T <= 64 && !whole) {
        const int c_first = sk.owner(t0i), c_last = sk.owner(t1i - 1);
        ll = !E3_DEC_NO_LL && c_last - c_first == 1 && sk.start(c_last + 1) == t1i;
        if (c_last - c_first == 1 && !(ll && blockIdx.x == c_first)) {
          const int slot = (int)blockIdx.x - c_first;
          if (et == 0) {
            volatile unsigned *tk = &a.tickets[tile];
            unsigned seen = *tk;
            if (ll) {
              // the head CTA is resident (the grid never exceeds the SMs, and
              // no dependent grid launches before every CTA has triggered);
              // a bound turns a broken invariant into an error, not a hang
              long spins = 0;
              while (seen != 1u) {
                __nanosleep(100);
                seen = *tk;
                if (++spins > (1L << 24)) __trap();
              }
            }
            *s_last = (seen == 1u) ? 3 : 0;
            if (seen == 1u) a.tickets[tile] = 0;   // both contributors accounted for: ready for the next launch
          }
          epi_bar();
          early = *s_last == 3;
          early_slot = slot;
          if (early) {
            // the other partial goes to sE (free: the previous segment's
            // epilogue has finished with it); the accumulator is added below
            __threadfence();
            const float4 *op = reinterpret_cast<const float4 *>(a.part) +
                               ((size_t)tile * a.max_contrib + (1 - slot)) * (T / 4) * DM + r;
#pragma unroll 1
            for (int k0 = 0; k0 < T / 4; k0 += 8) {   // 8 vectors in flight (registers)
              float4 pv[8];
#pragma unroll
              for (int k = 0; k < 8; ++k) pv[k] = __ldcg(op + (size_t)(k0 + k) * DM);
#pragma unroll
              for (int k = 0; k < 8; ++k) {
                sE[r * P + 4 * (k0 + k)] = pv[k].x;
                sE[r * P + 4 * (k0 + k) + 1] = pv[k].y;
                sE[r * P + 4 * (k0 + k) + 2] = pv[k].z;
                sE[r * P + 4 * (k0 + k) + 3] = pv[k].w;
              }
            }
          }
        }
      }
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      tlm = tl_now();
      if (!tlf) tlf = tlm;
      const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16) + acc * T;
#pragma unroll
      for (int c = 0; c < T / 32; ++c) {
        uint32_t v[32];
        tmem_ld32(taddr + c * 32, v);
        tmem_wait_ld();
        if (early) {   // contributor order: acc = (0 + p0) + p1, as the reduction below
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            const float own = __uint_as_float(v[j]), oth = sE[r * P + c * 32 + j];
            sE[r * P + c * 32 + j] = early_slot == 0 ? (0.f + own) + oth : (0.f + oth) + own;
          }
        } else {
#pragma unroll
          for (int j = 0; j < 32; ++j) sE[r * P + c * 32 + j] = __uint_as_float(v[j]);
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[acc]);
      if (++acc == 2) { acc = 0; acc_phase ^= 1; }
      epi_bar();
      if (CSK > 1) break;               // one segment; reduced across the cluster below

      unsigned long long tl_tk = 0, tl_rd = 0;
      if (early) {
        tl_rd = tl_now();   // reduced while the accumulator was read (each thread its own row)
      } else if (!whole) {
        // shared tile: publish this contributor's partial; the tile's last
        // arrival sums the contributors' partials in contributor order
        const int c_first = sk.owner(t0i), c_last = sk.owner(t1i - 1);
        const int slot = (int)blockIdx.x - c_first, ncon = c_last - c_first + 1;
        // partial layout [tile][slot][T/4][row] of float4 (4 tokens): each
        // thread moves its row's T values as 16-byte vectors and a warp's
        // access is 512 contiguous bytes
        float4 *part = reinterpret_cast<float4 *>(a.part) + ((size_t)tile * a.max_contrib + slot) * (T / 4) * DM + r;
        // every other contributor already arrived (the usual case for a
        // CTA's last segment, the head of a tile whose tail the next CTA
        // computed first): this CTA is the last, its partial stays in sE and
        // is summed in its contributor position below -- no write, fence and
        // ticket round trips on the kernel's critical path
        if (et == 0) {
          if (ll) {
            *s_last = 0;                        // the head of a two-late tile always publishes
          } else {
            const unsigned seen = *reinterpret_cast<volatile unsigned *>(&a.tickets[tile]);
            *s_last = (seen == (unsigned)(ncon - 1)) ? 2 : 0;
            if (*s_last) a.tickets[tile] = 0;   // every contributor arrived: ready for the next launch
          }
        }
        epi_bar();
        const bool own_in_smem = *s_last == 2;
        if (!own_in_smem) {
#pragma unroll
          for (int i = 0; i < T / 4; ++i)
            part[(size_t)i * DM] =
                make_float4(sE[r * P + 4 * i], sE[r * P + 4 * i + 1], sE[r * P + 4 * i + 2], sE[r * P + 4 * i + 3]);
          __threadfence();
          epi_bar();
          if (et == 0) {
            const unsigned prev = atomicAdd(&a.tickets[tile], 1u);
            *s_last = (prev == (unsigned)(ncon - 1));
            if (*s_last) a.tickets[tile] = 0;   // ready for the next launch
          }
          epi_bar();
        }
        tl_tk = tl_now();
        if (!*s_last) {
          if (threadIdx.x == 64) tl_rec(tlb, 8300 + EPI, tlm, tl_tk);   // segment: acc ready, ticket, (no reduction)
          continue;
        }
        const unsigned long long tlr0 = tl_now();
        __threadfence();
        // sum the contributors' partials in contributor order; contributor
        // j+1's loads are in flight while j is accumulated (one round trip
        // per contributor; a serial load -> add chain cost ~10 us, r01)
        const float4 *base = reinterpret_cast<const float4 *>(a.part) + (size_t)tile * a.max_contrib * (T / 4) * DM + r;
        const size_t cstride = (size_t)DM * T / 4;   // float4s between contributors
#pragma unroll 1
        for (int h = 0; h < T / 32 + (T % 32 ? 1 : 0); ++h) {   // 32 tokens per pass (registers)
          constexpr int NV = (T < 32 ? T : 32) / 4;
          float4 acc4[NV], cur[NV], nxt[NV];
          // contributor j's values: its partial in global memory, or this
          // CTA's own accumulator in sE when it skipped publishing it
          auto fetch = [&](int j, float4 *dst) {
#pragma unroll
            for (int i = 0; i < NV; ++i) {
              if (own_in_smem && j == slot) {
                const int t = h * 32 + 4 * i;
                dst[i] = make_float4(sE[r * P + t], sE[r * P + t + 1], sE[r * P + t + 2], sE[r * P + t + 3]);
              } else {
                dst[i] = __ldcg(base + j * cstride + (size_t)(h * NV + i) * DM);
              }
            }
          };
#pragma unroll
          for (int i = 0; i < NV; ++i) acc4[i] = make_float4(0.f, 0.f, 0.f, 0.f);
          fetch(0, cur);
#pragma unroll 1
          for (int j = 0; j < ncon; ++j) {
            if (j + 1 < ncon) fetch(j + 1, nxt);
#pragma unroll
            for (int i = 0; i < NV; ++i) {
              acc4[i].x += cur[i].x;
              acc4[i].y += cur[i].y;
              acc4[i].z += cur[i].z;
              acc4[i].w += cur[i].w;
              cur[i] = nxt[i];
            }
          }
#pragma unroll
          for (int i = 0; i < NV; ++i) {
            const int t = h * 32 + 4 * i;
            sE[r * P + t] = acc4[i].x;
            sE[r * P + t + 1] = acc4[i].y;
            sE[r * P + t + 2] = acc4[i].z;
            sE[r * P + t + 3] = acc4[i].w;
          }
        }
        epi_bar();
        if (threadIdx.x == 64) tl_rec(tlb, 8200 + EPI, tlr0, tlr0);   // reduction: start, end
        tl_rd = tl_now();
      }

      // ---------------------------------------------------- final epilogue
      // global loads of a token batch are issued together before its stores
      // (a load -> store chain per token cost ~1 us x T per launch)
      // STORE / RESID / SWIGLU: transposed through sE so that 16 (8) lanes
      // write one token's 128 (64) features as 16-byte vectors, 256 (128)
      // contiguous bytes; the residual is read the same way.  The per-thread
      // scalar form (one 2-byte load + store per token and feature) took
      // 4-14 us per tile (r01 dec_timeline: gate_up epilogue 14 us)
      const bool vec = (a.ldo % 8 == 0) && (a.N % 8 == 0) && ((reinterpret_cast<uintptr_t>(a.Y) & 15) == 0) &&
                       (EPI != E3_DEC_RESID || (reinterpret_cast<uintptr_t>(a.R) & 15) == 0);
      if ((EPI == E3_DEC_STORE || EPI == E3_DEC_RESID) && vec) {
        const int g = et & 15, n = tile * DM + 8 * g;
        if (n < a.N) {
          // every residual vector of this thread is loaded before the first
          // store (Y may alias R as far as the compiler knows, so a load
          // after a store would cost one round trip per token pass: ~5 us)
          uint4 rres[T / 8];
          if (EPI == E3_DEC_RESID) {
#pragma unroll
            for (int k = 0; k < T / 8; ++k)
              rres[k] = __ldg(reinterpret_cast<const uint4 *>(a.R + (size_t)((et >> 4) + 8 * k) * a.ldo + n));
          }
#pragma unroll
          for (int k = 0; k < T / 8; ++k) {
            const int t = (et >> 4) + 8 * k;
            float v[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) v[j] = sE[(8 * g + j) * P + t];
            if (EPI == E3_DEC_RESID) {
              const uint4 rr = rres[k];
              const uint32_t rw[4] = {rr.x, rr.y, rr.z, rr.w};
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                v[2 * e] += bf_lo(rw[e]);
                v[2 * e + 1] += bf_hi(rw[e]);
              }
            }
            *reinterpret_cast<uint4 *>(a.Y + (size_t)t * a.ldo + n) =
                make_uint4(pack_bf16(v[0], v[1]), pack_bf16(v[2], v[3]), pack_bf16(v[4], v[5]), pack_bf16(v[6], v[7]));
          }
        }
      } else if (EPI == E3_DEC_SWIGLU && vec) {
        const int g = et & 7, f = tile * 64 + 8 * g;
#pragma unroll 4
        for (int t = et >> 3; t < T; t += 16) {
          float o[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const float gv = sE[(8 * g + j) * P + t], up = sE[(64 + 8 * g + j) * P + t];
            // SiLU(g) * u (bf16 output); __fdividef has no slow path when
            // e^-g overflows (IEEE division / __frcp_rn took ~5 us per tile
            // on |g| > 88)
            o[j] = gv * __fdividef(1.0f, 1.0f + __expf(-gv)) * up;
          }
          *reinterpret_cast<uint4 *>(a.Y + (size_t)t * a.ldo + f) =
              make_uint4(pack_bf16(o[0], o[1]), pack_bf16(o[2], o[3]), pack_bf16(o[4], o[5]), pack_bf16(o[6], o[7]));
        }
      } else if (EPI == E3_DEC_STORE || EPI == E3_DEC_RESID) {
        const int n = tile * DM + r;
        if (n < a.N) {
#pragma unroll 1
          for (int tb = 0; tb < T; tb += 32) {
            float rv[32];
#pragma unroll
            for (int ii = 0; ii < 32; ++ii)
              rv[ii] = (EPI == E3_DEC_RESID) ? bf2f(a.R[(size_t)(tb + ii) * a.ldo + n]) : 0.f;
#pragma unroll
            for (int ii = 0; ii < 32; ++ii)
              a.Y[(size_t)(tb + ii) * a.ldo + n] = __float2bfloat16_rn(sE[r * P + tb + ii] + rv[ii]);
          }
        }
      } else if (EPI == E3_DEC_SWIGLU) {
        if (r < 64) {
          const int f = tile * 64 + r;
          for (int t = 0; t < T; ++t) {
            const float g = sE[r * P + t], up = sE[(r + 64) * P + t];
            a.Y[(size_t)t * a.ldo + f] = __float2bfloat16_rn(g / (1.0f + expf(-g)) * up);
          }
        }
      } else if (EPI == E3_DEC_QKV_ROPE && vec) {
        // tile = one head (head_dim 128): q heads, then k heads, then v heads.
        // Thread = (token t, dims 8g..8g+7 and their RoPE partners 64+8g..):
        // the (cos, sin) of the 8 pairs come as four 16-byte loads, both
        // halves leave as 16-byte stores (the scalar form's table loads
        // were a round trip per 16 tokens: ~6 us per tile, r01)
        const int hq = tile;
        const bool is_q = hq < a.nh, is_k = !is_q && hq < a.nh + a.kvh;
        const int g = et & 7;
        // all (cos, sin) vectors of this thread's tokens before the first
        // store (the stores may alias the table as far as the compiler knows)
        float4 rc[T / 16][4];
        if (is_q || is_k) {
#pragma unroll
          for (int k = 0; k < T / 16; ++k) {
            const float4 *cp = reinterpret_cast<const float4 *>(a.rope + (size_t)sPos[(et >> 3) + 16 * k] * 64 + 8 * g);
#pragma unroll
            for (int i = 0; i < 4; ++i) rc[k][i] = __ldg(cp + i);
          }
        }
#pragma unroll
        for (int k = 0; k < T / 16; ++k) {
          const int t = (et >> 3) + 16 * k;
          float lo[8], hi[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            lo[j] = sE[(8 * g + j) * P + t];
            hi[j] = sE[(64 + 8 * g + j) * P + t];
          }
          if (is_q || is_k) {
            const float cs[16] = {rc[k][0].x, rc[k][0].y, rc[k][0].z, rc[k][0].w, rc[k][1].x, rc[k][1].y,
                                  rc[k][1].z, rc[k][1].w, rc[k][2].x, rc[k][2].y, rc[k][2].z, rc[k][2].w,
                                  rc[k][3].x, rc[k][3].y, rc[k][3].z, rc[k][3].w};
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              const float c = cs[2 * j], sn = cs[2 * j + 1];
              const float l = fmaf(lo[j], c, -hi[j] * sn), h = fmaf(hi[j], c, lo[j] * sn);
              lo[j] = l;
              hi[j] = h;
            }
          }
          const uint4 olo = make_uint4(pack_bf16(lo[0], lo[1]), pack_bf16(lo[2], lo[3]), pack_bf16(lo[4], lo[5]),
                                       pack_bf16(lo[6], lo[7]));
          const uint4 ohi = make_uint4(pack_bf16(hi[0], hi[1]), pack_bf16(hi[2], hi[3]), pack_bf16(hi[4], hi[5]),
                                       pack_bf16(hi[6], hi[7]));
          __nv_bfloat16 *dst = nullptr;
          if (is_q) {
            dst = a.Y + (size_t)t * a.ldo + hq * 128;
          } else if (sSlot[t] >= 0) {
            const int kh = is_k ? hq - a.nh : hq - a.nh - a.kvh;
            __nv_bfloat16 *cache = is_k ? a.kc : a.vc;
            dst = cache + (((size_t)sSlot[t] * a.kvh + kh) * a.max_ctx + sPos[t]) * 128;
          }
          if (dst) {
            *reinterpret_cast<uint4 *>(dst + 8 * g) = olo;
            *reinterpret_cast<uint4 *>(dst + 64 + 8 * g) = ohi;
          }
        }
      } else if (EPI == E3_DEC_QKV_ROPE) {
        // tile = one head (head_dim 128): q heads, then k heads, then v heads
        const int hq = tile;
        const bool is_q = hq < a.nh, is_k = !is_q && hq < a.nh + a.kvh;
        const int j = r & 63;
#pragma unroll 1
        for (int tb = 0; tb < T; tb += 16) {
          float2 cs[16];
#pragma unroll
          for (int ii = 0; ii < 16; ++ii)
            cs[ii] = (is_q || is_k) ? a.rope[(size_t)sPos[tb + ii] * 64 + j] : make_float2(1.f, 0.f);
#pragma unroll
          for (int ii = 0; ii < 16; ++ii) {
            const int t = tb + ii;
            float v = sE[r * P + t];
            if (is_q || is_k) {
              const float pr = sE[(r ^ 64) * P + t];
              v = (r < 64) ? fmaf(v, cs[ii].x, -pr * cs[ii].y) : fmaf(v, cs[ii].x, pr * cs[ii].y);
            }
            const __nv_bfloat16 o = __float2bfloat16_rn(v);
            if (is_q) {
              a.Y[(size_t)t * a.ldo + hq * 128 + r] = o;
            } else if (sSlot[t] >= 0) {
              const int kh = is_k ? hq - a.nh : hq - a.nh - a.kvh;
              __nv_bfloat16 *cache = is_k ? a.kc : a.vc;
              cache[(((size_t)sSlot[t] * a.kvh + kh) * a.max_ctx + sPos[t]) * 128 + r] = o;
            }
          }
        }
      } else if (EPI == E3_DEC_LOGITS) {
        const int n0 = tile * DM;
        const int rows = (a.N - n0) < DM ? (a.N - n0) : DM;
        // logits go straight to the exit records, row id_t of [capacity, V]
        // (a row that does not exit here is rewritten by the ramp it exits
        // at -- the last ramp exits every row), so no second pass copies
        // 128 KB per exiting token; sTok[t] = id_t or -1 (padding / no logits)
        if (a.Z && r < rows)
          for (int t = 0; t < T; ++t)
            if (sTok[t] >= 0) a.Z[(size_t)sTok[t] * a.N + n0 + r] = sE[r * P + t];
        for (int t = et; t < T; t += 128) {
          float m = sE[t];
          int idx = 0;
          for (int i = 1; i < rows; ++i) {
            const float z = sE[i * P + t];
            if (z > m) { m = z; idx = i; }
          }
          float s = 0.f, uu = 0.f;
          for (int i = 0; i < rows; ++i) {
            const float d = sE[i * P + t] - m;
            const float e = expf(d);
            s += e;
            uu = fmaf(e, d, uu);
          }
          a.stats[(size_t)tile * T + t] = make_float4(m, s, uu, __int_as_float(n0 + idx));
        }
      }
      epi_bar();                        // sE is reused by the next unit
      if (threadIdx.x == 64) tl_rec(tlb, tl_rd ? 8400 + EPI : 8500 + EPI, tlm, tl_rd ? tl_rd : tlm);   // segment: acc ready, reduced, end
    }
    if (threadIdx.x == 64) {
      tl_rec(tlb, 8100 + EPI, tl0, tl1);
      tl_rec(tlb, 8000 + EPI, tlf, tlm);
    }
  }
  if (EPI == E3_DEC_PARTIAL && warp >= 2 && warp <= 5) {
    // this CTA's fp32 partial tile -> part_out[k][t][n] (k = its K quarter):
    // per token a warp writes 32 consecutive features (128 B)
    const int kq = blockIdx.x % CSK, tile = blockIdx.x / CSK;
    const int r = (warp & 3) * 32 + lane_id(), n = tile * DM + r;
    if (n < a.N) {
      float *po = a.part_out + (size_t)kq * a.T * a.N + n;
#pragma unroll 8
      for (int t = 0; t < T; ++t) po[(size_t)t * a.N] = sE[r * (T + 1) + t];
    }
  }
  if (kCluster) {
    constexpr int RPC = DM / CSK;       // rows reduced and stored by this CTA
    const int cr = (int)cluster_ctarank();
    const int tile = blockIdx.x / CSK;
    const unsigned long long tc0 = tl_now();
    cluster_sync();                     // every CTA's partial tile is in its smem
    const unsigned long long tc1 = tl_now();
    if (warp >= 2 && warp <= 5) {
      // every remote value of a batch of elements is loaded before the first
      // add (one load -> add chain per element and rank serialised ~48 DSMEM
      // round trips per thread: ~5 us after the mainloop, r02 llama_timeline)
      const int et = threadIdx.x - 64;
      constexpr int EB = 8;             // elements per batch
      static_assert((RPC * T) % (128 * EB) == 0, "CSK reduction batches");
#pragma unroll 1
      for (int e0 = et; e0 < RPC * T; e0 += 128 * EB) {
        float v[EB][CSK];
#pragma unroll
        for (int u = 0; u < EB; ++u) {
          const int e = e0 + 128 * u;
          const int row = cr * RPC + e / T, t = e % T;
          const uint32_t off = smem_u32(&sE[row * P + t]);
#pragma unroll
          for (int q = 0; q < CSK; ++q) v[u][q] = (q == cr) ? sE[row * P + t] : ld_dsmem_f32(mapa_shared(off, (uint32_t)q));
        }
#pragma unroll
        for (int u = 0; u < EB; ++u) {
          const int e = e0 + 128 * u;
          const int row = cr * RPC + e / T, t = e % T;
          float acc = 0.f;
#pragma unroll
          for (int q = 0; q < CSK; ++q) acc += v[u][q];   // rank order
          sE[row * P + t] = acc;        // only this CTA reads its own rows from here on
        }
      }
    }
    const unsigned long long tc2 = tl_now();
    // done reading the peers' smem; the matching wait is just before exit, so
    // the stores below overlap the barrier (no CTA leaves while a peer may
    // still read its smem)
    asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
    if (threadIdx.x == 64) tl_rec(tlb, 8800 + EPI, tc0, tc1);   // CSK tail: before / after sync 1, reduced
    if (threadIdx.x == 64) tl_rec(tlb, 8900 + EPI, tc2, tl_now());   // reduced, after sync 2, (stored: below)
    if (warp >= 2 && warp <= 5 && (EPI == E3_DEC_STORE || EPI == E3_DEC_RESID)) {
      const int et = threadIdx.x - 64;
      constexpr int NG = RPC / 8, TP = 128 / NG;   // 8-row groups, tokens per pass
      const int g = et % NG, n = tile * DM + cr * RPC + 8 * g;
      if (n < a.N) {
        uint4 rres[T / TP];
        if (EPI == E3_DEC_RESID) {
#pragma unroll
          for (int k = 0; k < T / TP; ++k)
            rres[k] = __ldg(reinterpret_cast<const uint4 *>(a.R + (size_t)(et / NG + TP * k) * a.ldo + n));
        }
#pragma unroll
        for (int k = 0; k < T / TP; ++k) {
          const int t = et / NG + TP * k;
          float v[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) v[j] = sE[(cr * RPC + 8 * g + j) * P + t];
          if (EPI == E3_DEC_RESID) {
            const uint32_t rw[4] = {rres[k].x, rres[k].y, rres[k].z, rres[k].w};
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              v[2 * e] += bf_lo(rw[e]);
              v[2 * e + 1] += bf_hi(rw[e]);
            }
          }
          *reinterpret_cast<uint4 *>(a.Y + (size_t)t * a.ldo + n) =
              make_uint4(pack_bf16(v[0], v[1]), pack_bf16(v[2], v[3]), pack_bf16(v[4], v[5]), pack_bf16(v[6], v[7]));
        }
      }
    }
  }
  if (kCluster && threadIdx.x == 64) tl_rec(tlb, 8950 + EPI, tl0, tl0);   // CSK tail: stored
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (a.late_trigger) pdl_trigger();
  if (warp == 2) tmem_dealloc(tmem_base, CF::kTmemCols);
  if (kCluster) asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
}

}  // namespace

E3_TL_SETTER(tl_set_dec)

namespace {

template <int T, int EPI, int CSK>
e3_status dec_launch(const DecMaps &m, const DecArgs &a, int grid, cudaStream_t st) {
  auto kern = gemm_dec_kernel<T, EPI, CSK>;
  static bool attr_done = false;
  if (!attr_done) {
    E3_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, DCfg<T>::kSmem));
    attr_done = true;
  }
  if (CSK > 1 && EPI != E3_DEC_PARTIAL) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(kDThreads);
    cfg.dynamicSmemBytes = DCfg<T>::kSmem;
    cfg.stream = st;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = CSK;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl_enabled() ? 2 : 1;
    E3_CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, m.w, m.w2, m.x, a));
  } else {
    E3_CUDA_TRY(launch_k(kern, dim3(grid), dim3(kDThreads), DCfg<T>::kSmem, st, m.w, m.w2, m.x, a));
  }
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

template <int T>
e3_status dec_launch_epi(const DecMaps &m, const DecArgs &a, int grid, int csk, cudaStream_t st) {
  switch (a.epi) {
    case E3_DEC_STORE:
      return csk == 4 ? dec_launch<T, E3_DEC_STORE, 4>(m, a, grid, st) : dec_launch<T, E3_DEC_STORE, 1>(m, a, grid, st);
    case E3_DEC_RESID:
      return csk == 4 ? dec_launch<T, E3_DEC_RESID, 4>(m, a, grid, st) : dec_launch<T, E3_DEC_RESID, 1>(m, a, grid, st);
    case E3_DEC_SWIGLU: return dec_launch<T, E3_DEC_SWIGLU, 1>(m, a, grid, st);
    case E3_DEC_QKV_ROPE: return dec_launch<T, E3_DEC_QKV_ROPE, 1>(m, a, grid, st);
    case E3_DEC_LOGITS: return dec_launch<T, E3_DEC_LOGITS, 1>(m, a, grid, st);
    case E3_DEC_PARTIAL: return dec_launch<T, E3_DEC_PARTIAL, 4>(m, a, grid, st);
  }
  set_error("bad decode epilogue");
  return E3_EINVAL;
}

}  // namespace

int dec_tiles(int N, int epi) { return epi == E3_DEC_SWIGLU ? N / 64 : (N + DM - 1) / DM; }

// Stream-K grid: every SM.  E3_DEC_MAXGRID caps it (diagnostics): one whole
// tile per CTA (Llama-7B QKV, 96 tiles) is faster standalone (30.8 -> 23.0
// us, scripts/dec_bench.py) and in a graph-replayed split (llama_timeline:
// 893 -> 859 us per 4 layers) but 0.3 % slower in the LM bench's pipeline
// (same box, A/B twice), so it is not the default.
// Most contributors any tile has when `total` iterations (tiles of nkb) are cut
// into G ranges start(c) = c total / G (the kernel's SK split).
static int sk_max_contrib(long total, int nkb, long G) {
  int worst = 0;
  long c = 0;   // first range touching the current tile
  for (long t0 = 0; t0 < total; t0 += nkb) {
    while (c + 1 < G && (c + 1) * total / G <= t0) ++c;
    long e = c;
    while (e + 1 < G && (e + 1) * total / G < t0 + nkb) ++e;
    if ((int)(e - c + 1) > worst) worst = (int)(e - c + 1);
  }
  return worst;
}

// Stream-K grid: one CTA per SM, except that a few SMs are left out when that
// bounds every tile at two contributors (Llama-7B QKV: 96 tiles x 32 k-blocks
// on 148 CTAs gives tiles of three contributors, whose last one pays the
// global fixup; 144 CTAs = 3 ranges per 2 tiles, two contributors each, and
// the second contributor fetches the first's partial while its MMAs run)
static int dec_grid(int N, int K, int epi, int sms) {
  const int nkb = K / DKS;
  const long total = (long)dec_tiles(N, epi) * nkb;
  static const int cap = getenv("E3_DEC_MAXGRID") ? atoi(getenv("E3_DEC_MAXGRID")) : 0;   // diagnostics
  static const bool any3 = getenv("E3_DEC_ANY_CONTRIB") != nullptr;                      // diagnostics: old grid
  if (cap > 0 && cap < sms) sms = cap;
  if (total <= sms) return (int)total;
  if (!any3 && sk_max_contrib(total, nkb, sms) > 2)
    for (int g = sms - 1; g >= (sms * 15) / 16; --g)
      if (sk_max_contrib(total, nkb, g) <= 2) return g;
  return sms;
}

int dec_max_contrib(int N, int K, int epi, int sms) {
  // every CTA's range holds >= floor(total / G) iterations, so a tile of nkb
  // iterations meets at most ceil(nkb / that) + 1 ranges
  const long nkb = K / DKS, total = (long)dec_tiles(N, epi) * nkb;
  const long G = dec_grid(N, K, epi, sms);
  const long per = total / G;
  return (int)((nkb + per - 1) / per + 1);
}

e3_status dec_tmaps(DecMaps *m, const void *X, int T, int K, const void *W, const void *W2, int N, int epi) {
  const uint32_t wrows = (epi == E3_DEC_SWIGLU) ? 64 : DM;
  e3_status s = make_tmap_2d(&m->w, W, (uint64_t)N, (uint64_t)K, (uint64_t)K, wrows, DK);
  if (s == E3_OK) s = make_tmap_2d(&m->w2, W2 ? W2 : W, (uint64_t)N, (uint64_t)K, (uint64_t)K, wrows, DK);
  if (s == E3_OK) s = make_tmap_2d(&m->x, X, (uint64_t)T, (uint64_t)K, (uint64_t)K, (uint32_t)T, DK);
  return s;
}

// Cluster split-K (4 CTAs per tile) where the tiles fill at most a quarter
// of the SMs (W_o, W_down of Llama-7B: 32 tiles -> 128 CTAs) and the
// epilogue is a plain / residual store with 16-byte vectors; E3_DEC_STREAMK
// forces stream-K everywhere (diagnostics)
bool dec_partial_ok(int N, int K, int sms) {
  static const bool off = getenv("E3_DEC_NO_PARTIAL") != nullptr;   // diagnostics: cluster split-K + rmsnorm
  return !off && N % 8 == 0 && 4 * dec_tiles(N, E3_DEC_RESID) <= sms && K / DKS >= 4;
}

static int dec_csk(const DecArgs &a, int sms) {
  if (a.epi == E3_DEC_PARTIAL) return 4;
  static const bool off = getenv("E3_DEC_STREAMK") != nullptr;
  if (off || (a.epi != E3_DEC_STORE && a.epi != E3_DEC_RESID)) return 1;
  const int tiles = dec_tiles(a.N, a.epi);
  const bool vec = a.ldo % 8 == 0 && a.N % 8 == 0 && (reinterpret_cast<uintptr_t>(a.Y) & 15) == 0 &&
                   (a.epi != E3_DEC_RESID || (reinterpret_cast<uintptr_t>(a.R) & 15) == 0);
  return (vec && 4 * tiles <= sms && a.K / DKS >= 4) ? 4 : 1;
}

e3_status dec_run(const DecMaps &m, const DecArgs &a_in, int sms, cudaStream_t st) {
  // PDL trigger after the epilogue: the next kernel's CTAs (decode attention,
  // RMSNorm), resident early beside this kernel's, sat in griddepcontrol.wait
  // taking issue slots from the stream-K fixup and epilogues (LM 9.42k ->
  // 9.61k tokens/s); E3_DEC_LATE_TRIGGER=0 restores the early trigger
  static const int late = getenv("E3_DEC_LATE_TRIGGER") ? atoi(getenv("E3_DEC_LATE_TRIGGER")) : 1;
  DecArgs a = a_in;
  a.late_trigger = late;
  const int csk = dec_csk(a, sms);
  const int grid = csk > 1 ? csk * dec_tiles(a.N, a.epi) : dec_grid(a.N, a.K, a.epi, sms);
  switch (a.T) {
    case 32: return dec_launch_epi<32>(m, a, grid, csk, st);
    case 64: return dec_launch_epi<64>(m, a, grid, csk, st);
    case 128: return dec_launch_epi<128>(m, a, grid, csk, st);
  }
  set_error("decode GEMM: batch must be 32, 64 or 128 tokens");
  return E3_EUNSUPPORTED;
}

e3_status rope_table(int max_ctx, int head_dim, double theta, float2 **out) {
  const int half = head_dim / 2;
  std::vector<float2> h((size_t)max_ctx * half);
  for (int p = 0; p < max_ctx; ++p)
    for (int j = 0; j < half; ++j) {
      const double ang = (double)p * std::pow(theta, -2.0 * j / head_dim);
      h[(size_t)p * half + j] = make_float2((float)std::cos(ang), (float)std::sin(ang));
    }
  float2 *d = nullptr;
  E3_CUDA_TRY(cudaMalloc(&d, h.size() * sizeof(float2)));
  E3_CUDA_TRY(cudaMemcpy(d, h.data(), h.size() * sizeof(float2), cudaMemcpyHostToDevice));
  *out = d;
  return E3_OK;
}

}  // namespace e3
