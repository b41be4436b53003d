// Self-attention of the split's encoder layers on the
// sm_100a tensor cores.  S <= 256 fits one KV tile, so there is no online
// rescaling.  A work item is (input b, head h, 128-query tile):
//
//   TMA   Q [128x64], K [SKVx64], V [SKVx64] (128B swizzle, OOB rows -> 0)
//   MMA1  S = Q K^T          tcgen05 128 x SKV x 64, fp32 in TMEM
//   soft  query row r = TMEM lane r is shared by two threads (warps w and
//         w+4 own lane quarter w and one half of the keys each): row max and
//         sum l of p = 2^((s-m) log2e / 8) combined through smem; l is fp32 of
//         the UNROUNDED p; bf16(p) -> smem in the K-major SW128 layout the
//         next MMA reads as its A operand
//   MMA2  O = P V            tcgen05 128 x 64 x SKV, V read MN-major; O reuses
//         the S columns of TMEM (S is dead once the softmax has read it)
//   out   ctx = bf16(O / l)  (rounding contract), staged in smem
//         with the 128B swizzle and written by one TMA store of the
//         [128 q x 64 d] box (rows >= S clipped by the 3-D tensor map)
//
// Persistent CTAs (2 per SM for SKV = 128) walk the items with the Q/K/V
// tiles double buffered: the next item's loads fly while the current item
// runs.  P overwrites the current item's dead Q|K tiles and the output tile is
// staged in the dead V tile, so a CTA needs 96 KB of smem and 128 TMEM columns.
// Keys >= S are masked to -inf; query rows >= S are not stored.
#include "common.cuh"
#include "kernels.h"
#include "prof.h"

namespace e3 {

namespace {

constexpr int D = 64;          // head dim
constexpr int QT = 128;        // query rows per item
// KP = 2 threads per query row: warps w and w+4 own TMEM lane quarter w % 4
// and one of two key ranges each (256 threads, two CTAs per SM)
template <int SKV>
struct AThr {
  static constexpr int KP = 2;
  static constexpr int kThreads = 128 * KP;
};

// SKV = keys per tile: S rounded up to 128 or, above 128, to a multiple of 32
// (S = 197 -> 224: 12 % fewer masked exponentials than 256).
//
// r02: P lives in TMEM (tcgen05.st over the thread's own dead S columns) and
// MMA2 reads it as its A operand (tcgen05.mma [d], [a_tmem], b_desc), so the
// smem holds only Q, K and V: above 128 keys the next item's Q | K land
// during this item's softmax (Q | K are dead once MMA1 completed) and V is
// double-buffered; at 128 keys whole Q | K | V buffers are double-buffered.
// Before (P in smem over the dead Q | K): the next item's loads could only
// start after MMA2, 2.3 us exposed per item at S = 197 (attn_trace).
template <int SKV>
struct ACfg {
  static constexpr int kQ = QT * D * 2;                  // 16 KB
  static constexpr int kKV = SKV * D * 2;                // 16 .. 32 KB
  static constexpr int kExtra = 1024 + 128 + 2 * 2 * AThr<SKV>::KP * QT * 4;
  static constexpr int kSmemMax = 232448 / 2 - 2048;     // two CTAs per SM
  // slots: Q|K pairs and V tiles
  static constexpr int kNQK = SKV <= 128 ? 2 : 1;
  static constexpr int kNV = (kNQK * (kQ + kKV) + 2 * kKV + kExtra <= kSmemMax) ? 2 : 1;
  static constexpr int kQKBytes = kNQK * (kQ + kKV);
  static constexpr int kSmem = kQKBytes + kNV * kKV + kExtra;
  static_assert(kSmem <= kSmemMax + 2048, "attention smem");
  static constexpr int NCH = SKV / 32;                   // 32-key chunks
  static constexpr int NCH0 = (NCH + 1) / 2;             // chunks of key part 0
  static constexpr int kBeginB = NCH0 * 32;              // first key of part 1
  // TMEM: S at columns [0, SKV); P of key k of part p at column
  // begin_p + (k - begin_p) / 2 (two bf16 per column, inside the part's own
  // S columns, already read); O (64 columns) past S, or between the parts
  static constexpr int kTmemCols = 256;
  static constexpr int kOCol = (((SKV + 31) / 32) * 32 + 64 <= kTmemCols) ? ((SKV + 31) / 32) * 32 : NCH0 * 16;
  static_assert(kOCol + 64 <= kTmemCols, "O columns");
  static_assert(kOCol >= SKV || kOCol + 64 <= kBeginB, "O overlaps part 1's P");
};

// Diagnostics (e3_debug_gemm_trace): per CTA and item (<= 8), globaltimer
// stamps: [0] MMA1 issued (Q | K landed), [1] S in TMEM, [2] P in TMEM
// (MMA2 issued), [3] O in TMEM, [4] output staged (store issued)
__device__ unsigned long long *g_attn_trace = nullptr;
__device__ __forceinline__ void atrace(int j, int kind) {
  unsigned long long *b = g_attn_trace;
  if (b && j < 8) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    b[((size_t)blockIdx.x * 8 + j) * 6 + kind] = t;
  }
}

// kMask: S < SKV, keys >= S are masked; without it (S == SKV, BB) the
// softmax loops carry no per-element compare / select
template <int SKV, bool kMask>
__global__ void __launch_bounds__(AThr<SKV>::kThreads, 2)
    attn_tc_kernel(const __grid_constant__ CUtensorMap tq, const __grid_constant__ CUtensorMap tkv,
                   const __grid_constant__ CUtensorMap tctx, int S, int H, int heads, int n_items,
                   unsigned *__restrict__ ctr) {
  using CF = ACfg<SKV>;
  constexpr int KP = AThr<SKV>::KP;
  constexpr int NCH = CF::NCH;
  constexpr int NCH0 = CF::NCH0;
  extern __shared__ uint8_t smem_raw[];
  // 1024-B aligned by offset arithmetic on the __shared__ array, so the
  // compiler keeps the shared address space (LDS / STS, not generic LD / ST)
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t *sVbase = smem + CF::kQKBytes;
  float *xch = reinterpret_cast<float *>(sVbase + CF::kNV * CF::kKV);   // [2][2][KP][QT]
  uint64_t *bars = reinterpret_cast<uint64_t *>(xch + 2 * 2 * KP * QT);
  uint64_t *bar_qk = bars;          // [2]
  uint64_t *bar_v = bars + 2;       // [2]
  uint64_t *bar_s = bars + 4;
  uint64_t *bar_o = bars + 5;
  uint32_t *tslot = reinterpret_cast<uint32_t *>(bars + 6);

  const int warp = warp_id(), lane = lane_id();
  const int tid = threadIdx.x;
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  const int qtiles = (S + QT - 1) / QT;
  const int quarter = warp & 3;
  const int khalf = warp >> 2;                            // which key part (and half of D for the output)
  const int row = quarter * 32 + lane;                    // query row within tile == TMEM lane
  const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
  const float sl2 = 1.4426950408889634f * 0.125f;         // log2(e) / sqrt(64)

  if (tid == 0) {
    tma_prefetch(&tq);
    tma_prefetch(&tkv);
    tma_prefetch(&tctx);
    for (int i = 0; i < 6; ++i) mbar_init(&bars[i], 1);
    fence_barrier_init();
  }
  // Items are handed out by an atomic counter (ctr[0]) instead of a static
  // stride: a CTA that becomes resident late (the SMs held by the previous
  // run's ramp and compaction on the tail stream) takes only what is left,
  // instead of its fixed share finishing last.  The last CTA to leave
  // (ctr[1]) zeroes both words for the next launch.  Every item is computed
  // the same way wherever it runs, so results do not depend on the schedule.
  // The counter is taken before the PDL wait: consecutive launches on one
  // counter set alternate between its two pairs (attn_run), and the launch
  // that last used (and zeroed) this pair completed before the previous
  // kernel in the stream -- the other pair's launch -- passed its own wait.
  // Thread 0 holds one ticket ahead (nreg), so the atomic's round trip is
  // off the critical path: the ticket taken in iteration j is used in j + 1.
  // (ctr == NULL: the static stride, E3_ATTN_STATIC=1 diagnostics)
  __shared__ int s_item[2];
  int nreg = 0;
  if (tid == 0) {
    s_item[0] = ctr ? (int)atomicAdd(&ctr[0], 1u) : (int)blockIdx.x;
    if (s_item[0] < n_items) nreg = ctr ? (int)atomicAdd(&ctr[0], 1u) : s_item[0] + (int)gridDim.x;
  }
  if (warp == 0) tmem_alloc(tslot, CF::kTmemCols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tslot;
  pdl_wait();                       // qkv of the previous kernel now visible
  pdl_trigger();
  const unsigned long long tl1 = tl_now();

  auto coords = [&](int it, int &b, int &h, int &qt) {
    const int bh = it / qtiles;
    qt = it % qtiles;
    b = bh / heads;
    h = bh % heads;
  };
  auto issue_qk = [&](int it, int slot) {
    int b, h, qt;
    coords(it, b, h, qt);
    uint8_t *base = smem + slot * (CF::kQ + CF::kKV);
    mbar_expect_tx(&bar_qk[slot], CF::kQ + CF::kKV);
    tma_load_3d(base, &tq, &bar_qk[slot], h * D, qt * QT, b);
    tma_load_3d(base + CF::kQ, &tkv, &bar_qk[slot], H + h * D, 0, b);
  };
  auto issue_v = [&](int it, int slot) {
    int b, h, qt;
    coords(it, b, h, qt);
    mbar_expect_tx(&bar_v[slot], CF::kKV);
    tma_load_3d(sVbase + slot * CF::kKV, &tkv, &bar_v[slot], 2 * H + h * D, 0, b);
  };
  uint32_t phases = 0;                                    // bit i: parity of bars[i] (thread 0)
  auto wait_bar = [&](int i) {
    mbar_wait(&bars[i], (phases >> i) & 1u);
    phases ^= 1u << i;
  };

  int item = s_item[0];
  if (tid == 0 && item < n_items) {
    issue_qk(item, 0);
    issue_v(item, 0);
  }
  uint32_t sphase = 0, ophase = 0;

  for (int j = 0; item < n_items; ++j) {
    const int qs = (CF::kNQK == 2) ? (j & 1) : 0;
    const int vs = (CF::kNV == 2) ? (j & 1) : 0;
    uint8_t *sQ = smem + qs * (CF::kQ + CF::kKV);
    uint8_t *sV = sVbase + vs * CF::kKV;
    int b, h, qt;
    coords(item, b, h, qt);
    const int q0 = qt * QT;
    int next = n_items;
    if (tid == 0) {                 // read by the other threads after the softmax exchange barrier
      next = nreg;
      s_item[(j + 1) & 1] = next;
      if (next < n_items) nreg = ctr ? (int)atomicAdd(&ctr[0], 1u) : next + (int)gridDim.x;
    }

    if (tid == 0) {
      // MMA1: S = Q K^T
      wait_bar(qs);
      tc_fence_after();
      atrace(j, 0);
      const uint32_t idesc = idesc_bf16_f32(QT, SKV, 0);
      const uint64_t dq = smem_desc_sw128(smem_u32(sQ), 16, 1024);
      const uint64_t dk = smem_desc_sw128(smem_u32(sQ + CF::kQ), 16, 1024);
#pragma unroll
      for (int k = 0; k < D / 16; ++k) tc_mma_f16(tbase, dq + 2 * k, dk + 2 * k, idesc, k != 0);
      tc_commit(bar_s);
      if (next < n_items) {
        // the other slots' last readers: MMA1 / MMA2 of item j-1 (done: waited
        // before its output) and the TMA store of its output from its V tile
        bulk_wait_read<0>();
        if (CF::kNQK == 2) issue_qk(next, qs ^ 1);
        if (CF::kNV == 2) issue_v(next, vs ^ 1);
      }
    }
    __syncwarp();

    // ------------------------------------------------------------ softmax
    mbar_wait(bar_s, sphase);
    sphase ^= 1;
    tc_fence_after();
    if (tid == 0) {
      atrace(j, 1);
      if (CF::kNQK == 1 && next < n_items) issue_qk(next, 0);   // Q | K dead once MMA1 completed
    }
    // S = 128: S is read from TMEM once, this thread's 64 keys stay in
    // registers between the max pass and the exponentiation pass (-6 %);
    // longer rows would spill, so they are read twice
    constexpr bool kKeep = NCH0 <= 2;                     // <= 64 registers; longer rows reload
    const int c_begin = khalf * NCH0 * 32;
    // a lane quarter whose 32 query rows all lie past S (the second query
    // tile of S = 197) skips its softmax and output: those rows are never
    // stored, and P / O rows are independent in both MMAs
    const bool qvalid = !kMask || q0 + quarter * 32 < S;
    const int nch = qvalid ? min(NCH0, NCH - khalf * NCH0) : 0;
    float sv[kKeep ? NCH0 * 32 : 32];
    float mx = -INFINITY;
#pragma unroll
    for (int ci = 0; ci < NCH0; ++ci) {
      if (ci < nch) {
        const int c = c_begin + ci * 32;
        uint32_t r[32];
        tmem_ld32(tbase + lane_off + c, r);
        tmem_wait_ld();
        float m4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
        if (kMask && c + 32 > S) {        // the chunk holding key S: masked keys become -inf (p = 0)
#pragma unroll
          for (int jj = 0; jj < 32; ++jj) {
            const float v = (c + jj < S) ? __uint_as_float(r[jj]) : -INFINITY;
            if (kKeep) sv[ci * 32 + jj] = v;
            m4[jj & 3] = fmaxf(m4[jj & 3], v);
          }
        } else {                           // full chunks: no per-key test
#pragma unroll
          for (int jj = 0; jj < 32; ++jj) {
            const float v = __uint_as_float(r[jj]);
            if (kKeep) sv[ci * 32 + jj] = v;
            m4[jj & 3] = fmaxf(m4[jj & 3], v);
          }
        }
        mx = fmaxf(mx, fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3])));
      }
    }
    float *xmax = xch + (j & 1) * 2 * KP * QT;             // double-buffered exchange slots [KP][QT]
    float *xsum = xmax + KP * QT;
    xmax[khalf * QT + row] = mx;
    __syncthreads();
    mx = xmax[row];
#pragma unroll
    for (int q = 1; q < KP; ++q) mx = fmaxf(mx, xmax[q * QT + row]);
    const float mb = mx * sl2;
    float l4[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int ci = 0; ci < NCH0; ++ci) {
      if (ci < nch) {
        const int c = c_begin + ci * 32;
        if (!kKeep) {
          uint32_t r[32];
          tmem_ld32(tbase + lane_off + c, r);
          tmem_wait_ld();
#pragma unroll
          for (int jj = 0; jj < 32; ++jj) sv[jj] = __uint_as_float(r[jj]);
        }
        // p = 2^(s log2e / 8 - m log2e / 8): packed fp32x2 FMAs and sums (the
        // same roundings and summation order as the scalar form)
        float p[32];
#pragma unroll
        for (int jj = 0; jj < 32; jj += 4) {
          const float *sp = sv + (kKeep ? ci * 32 : 0) + jj;
          const float2 t0 = __ffma2_rn(make_float2(sp[0], sp[1]), make_float2(sl2, sl2), make_float2(-mb, -mb));
          const float2 t1 = __ffma2_rn(make_float2(sp[2], sp[3]), make_float2(sl2, sl2), make_float2(-mb, -mb));
          p[jj] = ex2_approx(t0.x);
          p[jj + 1] = ex2_approx(t0.y);
          p[jj + 2] = ex2_approx(t1.x);
          p[jj + 3] = ex2_approx(t1.y);
          if (kMask && !kKeep) {           // kept scores are already -inf past S
#pragma unroll
            for (int e = 0; e < 4; ++e)
              if (c + jj + e >= S) p[jj + e] = 0.f;
          }
          const float2 a0 = __fadd2_rn(make_float2(l4[0], l4[1]), make_float2(p[jj], p[jj + 1]));
          const float2 a1 = __fadd2_rn(make_float2(l4[2], l4[3]), make_float2(p[jj + 2], p[jj + 3]));
          l4[0] = a0.x;
          l4[1] = a0.y;
          l4[2] = a1.x;
          l4[3] = a1.y;
        }
        // bf16(p) of keys c..c+31 -> 16 TMEM columns of this row, inside this
        // part's own S columns (keys <= c + 15: already read)
        uint32_t pk[16];
#pragma unroll
        for (int jj = 0; jj < 16; ++jj) pk[jj] = pack_bf16(p[2 * jj], p[2 * jj + 1]);
        tmem_st16(tbase + lane_off + c_begin + (c - c_begin) / 2, pk);
      }
    }
    const float lpart = (l4[0] + l4[1]) + (l4[2] + l4[3]);
    xsum[khalf * QT + row] = lpart;
    tmem_wait_st();
    tc_fence_before();            // P in TMEM before MMA2 reads it
    __syncthreads();

    if (tid == 0) {
      wait_bar(2 + vs);           // this item's V
      tc_fence_after();
      atrace(j, 2);
      const uint32_t idesc = idesc_bf16_f32(QT, D, 1);   // B (= V) is MN-major, A (= P) K-major in TMEM
#pragma unroll
      for (int kk = 0; kk < SKV / 16; ++kk) {
        const int k = kk * 16;
        const int cb = k < CF::kBeginB ? 0 : CF::kBeginB;
        const uint32_t ap = tbase + (uint32_t)(cb + (k - cb) / 2);
        const uint64_t dv = smem_desc_sw128(smem_u32(sV + kk * 16 * 128), SKV * 128, 1024);
        tc_mma_f16_ts(tbase + CF::kOCol, ap, dv, idesc, kk != 0);
      }
      tc_commit(bar_o);
    }
    __syncwarp();
    mbar_wait(bar_o, ophase);     // MMA2 done: V tile is dead -> output staging
    ophase ^= 1;
    tc_fence_after();
    if (tid == 0) atrace(j, 3);
    float l = xsum[row];          // key parts summed in order (written before the last barrier)
#pragma unroll
    for (int q = 1; q < KP; ++q) l += xsum[q * QT + row];
    const float inv_l = 1.0f / l;
    if (qvalid) {                 // part k writes output columns 32k .. 32k + 31
      uint32_t r[32];
      tmem_ld32(tbase + lane_off + CF::kOCol + khalf * 32, r);   // this thread's 32 of the 64 d columns
      tmem_wait_ld();
      uint8_t *orow = sV + row * 128;                     // [128 q x 128 B], 128B swizzle
#pragma unroll
      for (int jj = 0; jj < 4; ++jj) {
        uint4 o;
        o.x = pack_bf16(__uint_as_float(r[8 * jj + 0]) * inv_l, __uint_as_float(r[8 * jj + 1]) * inv_l);
        o.y = pack_bf16(__uint_as_float(r[8 * jj + 2]) * inv_l, __uint_as_float(r[8 * jj + 3]) * inv_l);
        o.z = pack_bf16(__uint_as_float(r[8 * jj + 4]) * inv_l, __uint_as_float(r[8 * jj + 5]) * inv_l);
        o.w = pack_bf16(__uint_as_float(r[8 * jj + 6]) * inv_l, __uint_as_float(r[8 * jj + 7]) * inv_l);
        *reinterpret_cast<uint4 *>(orow + (((khalf * 4 + jj) ^ (row & 7)) << 4)) = o;
      }
    }
    fence_proxy_async_smem();
    tc_fence_before();            // O read before the next MMA1 / P writes reuse TMEM
    __syncthreads();
    if (tid == 0) {
      atrace(j, 4);
      tma_store_3d(&tctx, sV, h * D, q0, b);
      bulk_commit();
      if (CF::kNV == 1 && next < n_items) {               // the store reads the only V tile first
        bulk_wait_read<0>();
        issue_v(next, 0);
      }
    }
    item = s_item[(j + 1) & 1];   // written by thread 0 before this iteration's first barrier
  }
  if (tid == 0 && ctr) {
    __threadfence();
    if (atomicAdd(&ctr[1], 1u) == gridDim.x - 1) {   // every CTA has taken its last item
      atomicExch(&ctr[0], 0u);
      atomicExch(&ctr[1], 0u);
    }
  }
  if (tid == 0) bulk_wait_read<0>();   // smem read before exit; the global writes complete with the grid
  __syncthreads();
  if (warp == 0) tmem_dealloc(tbase, CF::kTmemCols);
  if (tid == 0) tl_rec(tlb, 2000 + SKV + (kMask ? 500 : 0), tl0, tl1);
}

template <int SKV, bool kMask>
e3_status launch_attn(const AttnMaps &m, int B, int S, int H, int heads, unsigned *ctr, cudaStream_t st) {
  auto kern = attn_tc_kernel<SKV, kMask>;
  static bool attr_done = false;
  static int sms = 0, per_sm = 0;
  if (!attr_done) {
    E3_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, ACfg<SKV>::kSmem));
    // without the max-shared carveout the occupancy query (and the launch) may
    // settle on one 101 KB CTA per SM although two fit (r01: grid 148, 18.5 us)
    E3_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
    int dev = 0;
    E3_CUDA_TRY(cudaGetDevice(&dev));
    sms = num_sms(dev);
    // resident CTAs per SM from the resources themselves: the occupancy API
    // answers 1 for SKV = 128 (r01: grid 148, 18.6 us) although two fit
    // (ncu: block limit registers 2, shared memory 2; forced 2: 13.8 us)
    cudaFuncAttributes fa;
    E3_CUDA_TRY(cudaFuncGetAttributes(&fa, kern));
    const int by_regs = 65536 / (fa.numRegs * AThr<SKV>::kThreads);
    const int by_smem = 233472 / (ACfg<SKV>::kSmem + (int)fa.sharedSizeBytes + 1024);
    per_sm = by_regs < by_smem ? by_regs : by_smem;
    if (per_sm < 1) per_sm = 1;
    if (const char *e = getenv("E3_ATTN_PER_SM")) per_sm = atoi(e);
    if (getenv("E3_VERBOSE")) fprintf(stderr, "[e3] attn_tc_kernel<%d>: %d CTAs per SM\n", SKV, per_sm);
    attr_done = true;
  }
  const int n_items = B * heads * ((S + QT - 1) / QT);
  const int grid = n_items < per_sm * sms ? n_items : per_sm * sms;
  static const bool stat = getenv("E3_ATTN_STATIC") != nullptr;
  if (stat) ctr = nullptr;
  E3_CUDA_TRY(launch_k(kern, dim3(grid), dim3(AThr<SKV>::kThreads), ACfg<SKV>::kSmem, st, m.q, m.kv, m.ctx, S, H, heads,
                       n_items, ctr));
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace

E3_TL_SETTER(tl_set_attn)

e3_status attn_set_trace(void *buf) {
  E3_CUDA_TRY(cudaMemcpyToSymbol(g_attn_trace, &buf, sizeof(buf)));
  return E3_OK;
}

e3_status attn_tmaps(AttnMaps *m, const void *qkv, const void *ctx, int B, int S, int H) {
  m->skv = S <= 128 ? 128 : ((S + 31) / 32) * 32;
  const uint64_t W3 = 3ull * H;
  e3_status s = make_tmap_3d(&m->q, qkv, W3, (uint64_t)S, (uint64_t)B, W3, W3 * S, D, QT, 1);
  if (s == E3_OK) s = make_tmap_3d(&m->kv, qkv, W3, (uint64_t)S, (uint64_t)B, W3, W3 * S, D, (uint32_t)m->skv, 1);
  if (s == E3_OK)
    s = make_tmap_3d(&m->ctx, ctx, (uint64_t)H, (uint64_t)S, (uint64_t)B, (uint64_t)H, (uint64_t)H * S, D, QT, 1);
  return s;
}

e3_status attn_run(const AttnMaps &m, int B, int S, int H, int heads, unsigned *ctr4, int *parity,
                   cudaStream_t st) {
  unsigned *ctr = ctr4 + 2 * (*parity & 1);
  *parity ^= 1;
  switch (m.skv) {
    case 128: return S == 128 ? launch_attn<128, false>(m, B, S, H, heads, ctr, st) : launch_attn<128, true>(m, B, S, H, heads, ctr, st);
    case 160: return S == 160 ? launch_attn<160, false>(m, B, S, H, heads, ctr, st) : launch_attn<160, true>(m, B, S, H, heads, ctr, st);
    case 192: return S == 192 ? launch_attn<192, false>(m, B, S, H, heads, ctr, st) : launch_attn<192, true>(m, B, S, H, heads, ctr, st);
    case 224: return S == 224 ? launch_attn<224, false>(m, B, S, H, heads, ctr, st) : launch_attn<224, true>(m, B, S, H, heads, ctr, st);
    case 256: return S == 256 ? launch_attn<256, false>(m, B, S, H, heads, ctr, st) : launch_attn<256, true>(m, B, S, H, heads, ctr, st);
  }
  set_error("attention: S > 256");
  return E3_EUNSUPPORTED;
}

}  // namespace e3
