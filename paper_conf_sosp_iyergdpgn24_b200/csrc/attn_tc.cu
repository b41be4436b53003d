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
// KP threads per query row (warps w, w+4, ... own TMEM lane quarter w % 4 and
// one of KP key ranges): 2 for S <= 128 (256 threads, 2 CTAs per SM), 4 above
// (512 threads, one CTA per SM: each thread keeps its <= 64 scores in
// registers instead of re-reading TMEM, and twice the warps hide the MUFU
// and TMEM latencies)
template <int SKV>
struct AThr {
  // r02: 2 threads per query row at every SKV (above 128 keys the second CTA
  // per SM, below, replaces the r01 layout of 4 threads per row in one CTA)
  static constexpr int KP = 2;
  static constexpr int kThreads = 128 * KP;
};

// SKV = keys per tile: S rounded up to 128 or, above 128, to a multiple of 32
// (S = 197 -> 224: 12 % fewer masked exponentials than 256 and small enough
// K/V tiles to double-buffer the next item's loads)
template <int SKV>
struct ACfg {
  static constexpr int kQ = QT * D * 2;                  // 16 KB
  static constexpr int kKV = SKV * D * 2;                // 16 .. 32 KB
  static constexpr int kP = ((SKV + 63) / 64) * QT * 128;   // bf16 P in 64-key SW128 blocks
  // above 128 keys (S = 197 -> 224, r02): TWO CTAs per SM instead of one
  // double-buffered CTA -- one CTA's softmax overlaps the other's loads and
  // MMAs (r01 trace: 3.6 us per item, strictly serial load -> S -> softmax
  // -> PV -> store).  To fit two 256-thread CTAs, P (64 KB) overwrites the
  // dead Q | K tiles plus a pad placed before V: [Q | K | pad | V].
  static constexpr bool kTwoPerSm = SKV > 128;
  static constexpr int kPad = (kTwoPerSm && kP > kQ + kKV) ? kP - kQ - kKV : 0;
  static constexpr int kVOff = kQ + kKV + kPad;          // V tile offset in a buffer
  static constexpr int kBuf = kVOff + kKV;               // Q | K | (pad) | V
  static constexpr bool kPInQK = (kP <= kQ + kKV + kPad);   // P overwrites the dead Q|K(|pad) tiles
  static constexpr int kExtra = 1024 + 64 + 2 * 2 * AThr<SKV>::KP * QT * 4;
#ifdef E3_ATTN_SINGLE_BUF   // diagnostics: occupancy instead of double buffering
  static constexpr int kNBuf = 1;
#else
  static constexpr int kNBuf = kTwoPerSm ? 1 : ((2 * kBuf + (kPInQK ? 0 : kP) + kExtra <= 232448) ? 2 : 1);
#endif
  static constexpr int kSmem = kNBuf * kBuf + (kPInQK ? 0 : kP) + kExtra;
  static constexpr int kSCols = SKV <= 128 ? 128 : 256;      // one S (later O, 64 columns) accumulator
  // above 128 keys (one CTA per SM) two accumulators: MMA1 of item j+1 runs
  // while item j's output is written
  static constexpr bool kPipe = SKV > 128 && kNBuf == 2;
  static constexpr int kTmemCols = kPipe ? 2 * kSCols : kSCols;
};

// Diagnostics (e3_debug_gemm_trace): per CTA and item (<= 8), globaltimer
// stamps: [0] loads landed, [1] S in TMEM, [2] P in smem (MMA2 issued),
// [3] O in TMEM, [4] output staged (store issued)
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
                   const __grid_constant__ CUtensorMap tctx, int S, int H, int heads, int n_items) {
  using CF = ACfg<SKV>;
  constexpr int KP = AThr<SKV>::KP;
  constexpr int NCH = SKV / 32;     // 32-key chunks; key part p takes chunks [p NCHP, (p + 1) NCHP)
  constexpr int NCHP = (NCH + KP - 1) / KP;
  extern __shared__ uint8_t smem_raw[];
  // 1024-B aligned by offset arithmetic on the __shared__ array, so the
  // compiler keeps the shared address space (LDS / STS, not generic LD / ST)
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t *pbuf_sep = smem + CF::kNBuf * CF::kBuf;      // only when !kPInQK
  float *xch = reinterpret_cast<float *>(smem + CF::kNBuf * CF::kBuf + (CF::kPInQK ? 0 : CF::kP));  // [2][2][KP][QT]
  uint64_t *bars = reinterpret_cast<uint64_t *>(xch + 2 * 2 * KP * QT);
  uint64_t *bar_load = bars;        // [2]
  uint64_t *bar_s = bars + 2;
  uint64_t *bar_o = bars + 3;
  uint32_t *tslot = reinterpret_cast<uint32_t *>(bars + 4);

  const int warp = warp_id(), lane = lane_id();
  const int tid = threadIdx.x;
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  const int qtiles = (S + QT - 1) / QT;
  const int quarter = warp & 3;
  const int khalf = warp >> 2;                            // which key part (and, for parts 0-1, half of D)
  const int row = quarter * 32 + lane;                    // query row within tile == TMEM lane
  const uint32_t lane_off = (uint32_t)(quarter * 32) << 16;
  const float sl2 = 1.4426950408889634f * 0.125f;         // log2(e) / sqrt(64)

  if (tid == 0) {
    tma_prefetch(&tq);
    tma_prefetch(&tkv);
    tma_prefetch(&tctx);
    mbar_init(&bar_load[0], 1);
    mbar_init(&bar_load[1], 1);
    mbar_init(bar_s, 1);
    mbar_init(bar_o, 1);
    fence_barrier_init();
  }
  if (warp == 0) tmem_alloc(tslot, CF::kTmemCols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tslot;
  pdl_wait();                       // qkv of the previous kernel now visible
  pdl_trigger();
  const unsigned long long tl1 = tl_now();

  auto issue_load = [&](int item, int buf) {
    const int bh = item / qtiles, qt = item % qtiles;
    const int b = bh / heads, h = bh % heads;
    uint8_t *base = smem + buf * CF::kBuf;
    mbar_expect_tx(&bar_load[buf], CF::kQ + 2 * CF::kKV);   // the pad is not loaded
    tma_load_3d(base, &tq, &bar_load[buf], h * D, qt * QT, b);
    tma_load_3d(base + CF::kQ, &tkv, &bar_load[buf], H + h * D, 0, b);
    tma_load_3d(base + CF::kVOff, &tkv, &bar_load[buf], 2 * H + h * D, 0, b);
  };

  uint32_t load_phases = 0;                               // bit i: parity of bar_load[i] (thread 0)
  // S = Q K^T of the item in buffer `bf` into S accumulator `acc`
  auto issue_mma1 = [&](int bf, int acc) {
    mbar_wait(&bar_load[bf], (load_phases >> bf) & 1u);
    load_phases ^= 1u << bf;
    tc_fence_after();
    uint8_t *q = smem + bf * CF::kBuf;
    const uint32_t idesc = idesc_bf16_f32(QT, SKV, 0);
    const uint64_t dq = smem_desc_sw128(smem_u32(q), 16, 1024);
    const uint64_t dk = smem_desc_sw128(smem_u32(q + CF::kQ), 16, 1024);
#pragma unroll
    for (int k = 0; k < D / 16; ++k) tc_mma_f16(tbase + acc * CF::kSCols, dq + 2 * k, dk + 2 * k, idesc, k != 0);
    tc_commit(bar_s);
  };

  int item = blockIdx.x;
  if (tid == 0 && item < n_items) {
    issue_load(item, 0);
    if (CF::kPipe) issue_mma1(0, 0);
  }
  uint32_t sphase = 0, ophase = 0;

  for (int j = 0; item < n_items; ++j, item += gridDim.x) {
    const int buf = (CF::kNBuf == 2) ? (j & 1) : 0;
    uint8_t *sQ = smem + buf * CF::kBuf;
    uint8_t *sK = sQ + CF::kQ;
    uint8_t *sV = sQ + CF::kVOff;
    uint8_t *sP = CF::kPInQK ? sQ : pbuf_sep;
    const int bh = item / qtiles, qt = item % qtiles;
    const int b = bh / heads, h = bh % heads;
    const int q0 = qt * QT;
    const int next = item + gridDim.x;

    const uint32_t tS = tbase + (CF::kPipe ? (j & 1) * CF::kSCols : 0);   // this item's S, later O
    (void)sK;
    if (tid == 0) {
      if (!CF::kPipe) issue_mma1(buf, 0);               // kPipe: issued during the previous item
      atrace(j, 0);
      if (CF::kNBuf == 2 && next < n_items) {
        // the other buffer's last readers: MMA2 of item j-1 (done: waited before
        // its epilogue) and the TMA store of its output from the V tile
        bulk_wait_read<0>();
        issue_load(next, buf ^ 1);
      }
    }
    __syncwarp();

    // ------------------------------------------------------------ softmax
    mbar_wait(bar_s, sphase);
    sphase ^= 1;
    tc_fence_after();
    if (tid == 0) atrace(j, 1);
    // S = 128: S is read from TMEM once, this thread's 64 keys stay in
    // registers between the max pass and the exponentiation pass (-6 %);
    // longer rows would spill, so they are read twice
    constexpr int NCH0 = NCHP;                            // chunks per key part (the last may have fewer)
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
        tmem_ld32(tS + lane_off + c, r);
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
    uint8_t *prow = sP + row * 128;
#pragma unroll
    for (int ci = 0; ci < NCH0; ++ci) {
      if (ci < nch) {
        const int c = c_begin + ci * 32;
        if (!kKeep) {
          uint32_t r[32];
          tmem_ld32(tS + lane_off + c, r);
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
        // columns c..c+31 -> block c/64, 16-byte chunks (c%64)/8 .. +3, XOR-swizzled by row%8
        uint8_t *blk = prow + (c / 64) * (QT * 128);
        const int ch0 = (c % 64) / 8;
#pragma unroll
        for (int jj = 0; jj < 4; ++jj) {
          uint4 o;
          o.x = pack_bf16(p[8 * jj + 0], p[8 * jj + 1]);
          o.y = pack_bf16(p[8 * jj + 2], p[8 * jj + 3]);
          o.z = pack_bf16(p[8 * jj + 4], p[8 * jj + 5]);
          o.w = pack_bf16(p[8 * jj + 6], p[8 * jj + 7]);
          *reinterpret_cast<uint4 *>(blk + (((ch0 + jj) ^ (row & 7)) << 4)) = o;
        }
      }
    }
    const float lpart = (l4[0] + l4[1]) + (l4[2] + l4[3]);
    xsum[khalf * QT + row] = lpart;
    fence_proxy_async_smem();     // generic-proxy smem writes -> visible to the tensor core
    tc_fence_before();            // S fully read before MMA2 overwrites it with O
    __syncthreads();

    if (tid == 0) {
      tc_fence_after();
      atrace(j, 2);
      const uint32_t idesc = idesc_bf16_f32(QT, D, 1);   // B (= V) is MN-major
#pragma unroll
      for (int kk = 0; kk < SKV / 16; ++kk) {
        const uint64_t dp = smem_desc_sw128(smem_u32(sP + (kk / 4) * (QT * 128) + (kk % 4) * 32), 16, 1024);
        const uint64_t dv = smem_desc_sw128(smem_u32(sV + kk * 16 * 128), SKV * 128, 1024);
        tc_mma_f16(tS, dp, dv, idesc, kk != 0);
      }
      tc_commit(bar_o);
      if (CF::kPipe && next < n_items) issue_mma1(buf ^ 1, (j + 1) & 1);   // overlaps this item's output
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
    if (khalf < 2 && qvalid) {    // parts 0 and 1 write the 2 x 32 output columns
      uint32_t r[32];
      tmem_ld32(tS + lane_off + khalf * 32, r);           // this thread's 32 of the 64 d columns
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
    tc_fence_before();            // O read before the next MMA1 overwrites TMEM
    __syncthreads();
    if (tid == 0) {
      atrace(j, 4);
      tma_store_3d(&tctx, sV, h * D, q0, b);
      bulk_commit();
      if (CF::kNBuf == 1 && next < n_items) {
        bulk_wait_read<0>();
        issue_load(next, 0);
      }
    }
  }
  if (tid == 0) bulk_wait<0>();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tbase, CF::kTmemCols);
  if (tid == 0) tl_rec(tlb, 2000 + SKV + (kMask ? 500 : 0), tl0, tl1);
}

template <int SKV, bool kMask>
e3_status launch_attn(const AttnMaps &m, int B, int S, int H, int heads, cudaStream_t st) {
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
  E3_CUDA_TRY(launch_k(kern, dim3(grid), dim3(AThr<SKV>::kThreads), ACfg<SKV>::kSmem, st, m.q, m.kv, m.ctx, S, H, heads,
                       n_items));
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

e3_status attn_run(const AttnMaps &m, int B, int S, int H, int heads, cudaStream_t st) {
  switch (m.skv) {
    case 128: return S == 128 ? launch_attn<128, false>(m, B, S, H, heads, st) : launch_attn<128, true>(m, B, S, H, heads, st);
    case 160: return S == 160 ? launch_attn<160, false>(m, B, S, H, heads, st) : launch_attn<160, true>(m, B, S, H, heads, st);
    case 192: return S == 192 ? launch_attn<192, false>(m, B, S, H, heads, st) : launch_attn<192, true>(m, B, S, H, heads, st);
    case 224: return S == 224 ? launch_attn<224, false>(m, B, S, H, heads, st) : launch_attn<224, true>(m, B, S, H, heads, st);
    case 256: return S == 256 ? launch_attn<256, false>(m, B, S, H, heads, st) : launch_attn<256, true>(m, B, S, H, heads, st);
  }
  set_error("attention: S > 256");
  return E3_EUNSUPPORTED;
}

}  // namespace e3
