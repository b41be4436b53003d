// BERT exit ramp without clusters, and the ramp FUSED with the stable
// compaction of the split's survivors (SURVEY.md §8(a) a3 + a4; DESIGN.md §6
// K4/K5, r02).
//
// Ramp (DeeBERT; R1): c = LN2(y[b, 0, :]) (at a split's last
// layer the rows arrive pre-LN), p = tanh(W_p c + b_p), z = W_c p + b_c, exit
// test (R3/R4/R6/R12).  Work unit = (group g of 16 rows,
// slice j of TN = H / kSl pooler outputs): the CTA stages its TN W_p rows
// (cp.async, before the PDL wait), LayerNorms the group's 16 CLS rows
// (ln_row.cuh: bit-identical to the compaction's LN), runs the 16 x TN x H
// pooler on mma.sync with K split over the 8 warps (partials summed in warp
// order), tanh, and writes its partial logits sum_{o in slice} p W_c to
// global memory.  The LAST slice CTA of a group to arrive (ticket) sums the
// kSl partials in slice order -- deterministic, no float atomics -- and
// decides.  No clusters: the r01 kernel's 16-CTA clusters could not be
// placed until the FFN2 CTAs left whole GPCs (timeline: 2.5 us from FFN2's
// end to the ramp's release, 8 us to the decision).
//
// Fused ramp + compaction (the split's last ramp): ONE cooperative launch
// (every CTA co-resident) whose first R = groups x kSl CTAs also run the ramp
// slices; every CTA first loads its share of the token rows (warp per row, 4
// rows in flight) and LayerNorms them, then waits for the groups' decisions
// (device counter, acquire), scans the alive flags (ballot / popc, every CTA
// itself) and stores only the survivors at their compacted position straight
// into the next split's queue ring.  The row loads and the LayerNorm overlap
// the ramp; one kernel boundary less than ramp -> compaction.
#include "common.cuh"
#include "exitrule.cuh"
#include "kernels.h"
#include "ln_row.cuh"
#include "prof.h"

namespace e3 {

namespace {

constexpr int kT = 256;                 // threads
constexpr int kNW = kT / 32;
constexpr int kGRows = 16;              // rows per group (mma M)
constexpr int kMaxCl = 16;              // classes
constexpr int kMaxBc = 4096;
constexpr int kRowsFly = 4;             // token rows in flight per warp (compaction)

__device__ __forceinline__ void cp_async16(void *smem, const void *gmem) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

__device__ __forceinline__ void mma16816(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0, %1, %2, %3}, {%4, %5, %6, %7}, {%8, %9}, "
      "{%0, %1, %2, %3};"
      : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ bool row_ok(const RampArgs &a, int b, int n_valid) {
  return b < a.B && (a.init_alive ? (b < n_valid) : (__ldcg(a.alive + b) != 0));
}

// slices per group: TN = H / kSl pooler outputs per CTA, a multiple of 8
__host__ __device__ inline int ramp_slices(int H) { return H >= 512 ? 32 : 16; }

// dynamic smem: W tile [TN][P] bf16 | CLS [16][P] bf16 | partials [8][16][TN] f32
// | p [16][TN] f32 | W_c slice [C][TN] f32 | b_p slice [TN] f32
__host__ __device__ inline int rslice_smem_bytes(int H, int C) {
  const int TN = H / ramp_slices(H), P = H + 8;
  return (TN + kGRows) * P * 2 + kNW * kGRows * TN * 4 + kGRows * TN * 4 + C * TN * 4 + TN * 4;
}

// Counters in the workspace (zero between launches): tickets [groups],
// groups_done, exit ticket.
struct RCtr {
  unsigned *tickets;
  unsigned *groups_done;
  unsigned *exit_ctr;
};

template <int VPL>
struct RampSlice {
  const RampArgs &a;
  uint8_t *smem;
  int g, j, TN, NT, P, kSl;
  __nv_bfloat16 *sW, *sC;
  float *sRed, *sP, *sWc, *sBp;

  __device__ RampSlice(const RampArgs &a_, uint8_t *smem_, int g_, int j_) : a(a_), smem(smem_), g(g_), j(j_) {
    kSl = ramp_slices(a.H);
    TN = a.H / kSl;
    NT = TN / 8;
    P = a.H + 8;
    sW = reinterpret_cast<__nv_bfloat16 *>(smem);
    sC = sW + TN * P;
    sRed = reinterpret_cast<float *>(sC + kGRows * P);
    sP = sRed + kNW * kGRows * TN;
    sWc = sP + kGRows * TN;
    sBp = sWc + a.C * TN;
  }

  // weights only: before the dependency wait
  __device__ void prefetch() {
    const int H = a.H, nvec = H / 8, o0 = j * TN;
    const uint4 *wp = reinterpret_cast<const uint4 *>(a.w.w_p);
    for (int i = threadIdx.x; i < TN * nvec; i += kT) {
      const int r = i / nvec, k = i - r * nvec;
      cp_async16(reinterpret_cast<uint4 *>(sW + r * P) + k, wp + (size_t)(o0 + r) * nvec + k);
    }
    const __nv_bfloat16 *wc = reinterpret_cast<const __nv_bfloat16 *>(a.w.w_c);
    const __nv_bfloat16 *bp = reinterpret_cast<const __nv_bfloat16 *>(a.w.b_p);
    for (int i = threadIdx.x; i < a.C * TN; i += kT) {
      const int c = i / TN, o = i - c * TN;
      sWc[i] = bf2f(wc[(size_t)c * H + o0 + o]);
    }
    for (int i = threadIdx.x; i < TN; i += kT) sBp[i] = bf2f(bp[o0 + i]);
  }

  // CLS rows -> LN -> pooler -> partial logits of this slice -> part (global)
  __device__ void compute(const LnParams<VPL> &lp, int n_valid, float *part) {
    const int H = a.H, C = a.C, nvec = H / 8;
    const int warp = warp_id(), lane = lane_id();
    const int b0 = g * kGRows;
    const __nv_bfloat16 *x = reinterpret_cast<const __nv_bfloat16 *>(a.x);
    const size_t row_stride = (size_t)a.S * H;
    {
      uint4 v[2][VPL];
      bool ok[2];
#pragma unroll
      for (int jj = 0; jj < 2; ++jj) {
        const int r = warp + jj * kNW;
        ok[jj] = row_ok(a, b0 + r, n_valid);
        if (ok[jj]) ln_load_row<VPL>(v[jj], x + (size_t)(b0 + r) * row_stride, H, lane);
      }
#pragma unroll
      for (int jj = 0; jj < 2; ++jj) {
        const int r = warp + jj * kNW;
        if (ok[jj]) {
          if (a.ln_g) ln_apply<VPL>(v[jj], lp, H, a.eps, lane);
        } else {
#pragma unroll
          for (int i = 0; i < VPL; ++i) v[jj][i] = make_uint4(0, 0, 0, 0);
        }
        uint4 *dst = reinterpret_cast<uint4 *>(sC + r * P);
#pragma unroll
        for (int i = 0; i < VPL; ++i)
          if (lane + 32 * i < nvec) dst[lane + 32 * i] = v[jj][i];
      }
    }
    cp_async_wait_all();
    __syncthreads();
    {   // pooler: warp w takes the k16 steps w, w + 8, ...; NT independent chains
      constexpr int kMaxNT = 4;
      float acc[kMaxNT][4];
#pragma unroll
      for (int t = 0; t < kMaxNT; ++t) acc[t][0] = acc[t][1] = acc[t][2] = acc[t][3] = 0.f;
      const int gq = lane >> 2, tq = lane & 3;
      const __nv_bfloat16 *a_lo = sC + gq * P + 2 * tq;
      const __nv_bfloat16 *a_hi = sC + (gq + 8) * P + 2 * tq;
      const __nv_bfloat16 *bw = sW + gq * P + 2 * tq;
      for (int k = 16 * warp; k < H; k += 16 * kNW) {
        uint32_t af[4];
        af[0] = *reinterpret_cast<const uint32_t *>(a_lo + k);
        af[1] = *reinterpret_cast<const uint32_t *>(a_hi + k);
        af[2] = *reinterpret_cast<const uint32_t *>(a_lo + k + 8);
        af[3] = *reinterpret_cast<const uint32_t *>(a_hi + k + 8);
#pragma unroll
        for (int t = 0; t < kMaxNT; ++t)
          if (t < NT) {
            const uint32_t bf0 = *reinterpret_cast<const uint32_t *>(bw + t * 8 * P + k);
            const uint32_t bf1 = *reinterpret_cast<const uint32_t *>(bw + t * 8 * P + k + 8);
            mma16816(acc[t], af, bf0, bf1);
          }
      }
      float *red = sRed + warp * kGRows * TN;
#pragma unroll
      for (int t = 0; t < kMaxNT; ++t)
        if (t < NT) {
          const int col = t * 8 + 2 * tq;
          *reinterpret_cast<float2 *>(red + gq * TN + col) = make_float2(acc[t][0], acc[t][1]);
          *reinterpret_cast<float2 *>(red + (gq + 8) * TN + col) = make_float2(acc[t][2], acc[t][3]);
        }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < kGRows * TN; i += kT) {
      float s = sRed[i];
#pragma unroll
      for (int w = 1; w < kNW; ++w) s += sRed[w * kGRows * TN + i];
      sP[i] = tanhf(s + sBp[i % TN]);              // p = tanh(W_p c + b_p)
    }
    __syncthreads();
    // partial logits of this slice: warp w, rows w and w + 8 (lane-strided, shuffle-reduced)
    for (int jj = 0; jj < 2; ++jj) {
      const int r = warp + jj * kNW;
      for (int c = 0; c < C; ++c) {
        float z = 0.f;
        for (int o = lane; o < TN; o += 32) z = fmaf(sP[r * TN + o], sWc[c * TN + o], z);
#pragma unroll
        for (int off = 16; off; off >>= 1) z += __shfl_xor_sync(0xffffffffu, z, off);
        if (lane == 0) __stcg(part + ((size_t)(g * kSl + j) * kGRows + r) * C + c, z);
      }
    }
  }

  // ticket: the group's last slice CTA decides (returns true in that CTA)
  __device__ bool arrive(const RCtr &ctr, int *s_flag) {
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      const unsigned t = atomicAdd(ctr.tickets + g, 1u);
      *s_flag = (t == (unsigned)kSl - 1);
      if (*s_flag) {
        __threadfence();
        ctr.tickets[g] = 0;     // every slice of the group has arrived: reset for the next launch
      }
    }
    __syncthreads();
    return *s_flag != 0;
  }

  // rows of group g: sum the kSl partials in slice order, decide, exit record
  __device__ void decide(int n_valid, const float *part) {
    const int C = a.C;
    const int warp = warp_id(), lane = lane_id();
    // the group's kSl x 16 x C partials -> smem with every thread's loads in
    // flight at once (a lane summing them straight from L2 serialised kSl x C
    // round trips: r02 timeline, ~23 us to the decision), then summed per row
    // in slice order below (deterministic)
    float *sPart = sRed;   // [kSl][16][C] <= 8 x 16 x TN floats (kSl C <= H)
    const int np = kSl * kGRows * C;
    const float *gp = part + (size_t)g * kSl * kGRows * C;
    for (int i = threadIdx.x; i < np; i += kT) sPart[i] = __ldcg(gp + i);
    __syncthreads();
    if (warp != 0) return;
    const int r = lane, b = g * kGRows + r;
    bool exit_now = false;
    if (r < kGRows && b < a.B) {
      if (!row_ok(a, b, n_valid)) {
        if (a.init_alive) a.alive[b] = 0;
      } else {
        float z[kMaxCl];
#pragma unroll
        for (int c = 0; c < kMaxCl; ++c) {
          z[c] = 0.f;
          if (c < C) {
            float s = 0.f;
            for (int q = 0; q < kSl; ++q) s += sPart[(q * kGRows + r) * C + c];
            z[c] = s + bf2f(reinterpret_cast<const __nv_bfloat16 *>(a.w.b_c)[c]);
          }
        }
        float m = z[0];
        int label = 0;
#pragma unroll
        for (int c = 1; c < kMaxCl; ++c)
          if (c < C && z[c] > m) { m = z[c]; label = c; }   // lowest index on ties
        float sum = 0.f, qz = 0.f;
#pragma unroll
        for (int c = 0; c < kMaxCl; ++c)
          if (c < C) {
            const float e = expf(z[c] - m);
            sum += e;
            qz += e * (z[c] - m);
          }
        float metric;
        bool pass;
        if (a.test == E3_TEST_PATIENCE) {
          pass = patience_step(a.ex.state, a.id[b], a.ex.capacity, label, a.tau, &metric);
        } else if (a.test == E3_TEST_MAXPROB) {
          metric = 1.0f / sum;
          pass = metric > a.tau;
        } else {
          metric = logf(sum) - qz / sum;
          pass = metric < a.tau;
        }
        exit_now = pass || a.final_ramp;
        if (a.ex.ramp_metric && a.id[b] >= 0 && a.id[b] < a.ex.capacity)
          a.ex.ramp_metric[a.id[b] * a.ex.ramp_metric_stride + a.ramp_index] = metric;
        if (exit_now) {
          const int64_t id = a.id[b];
          if (id >= 0 && id < a.ex.capacity) {
            if (a.ex.exit_layer) a.ex.exit_layer[id] = a.layer;
            if (a.ex.label) a.ex.label[id] = label;
            if (a.ex.conf) a.ex.conf[id] = metric;
            if (a.ex.logits)
#pragma unroll
              for (int c = 0; c < kMaxCl; ++c)
                if (c < C) a.ex.logits[id * C + c] = z[c];
          }
        }
        a.alive[b] = exit_now ? 0 : 1;
      }
    }
    const int n_ex = __popc(__ballot_sync(0xffffffffu, exit_now));
    if (lane == 0 && n_ex) {
      if (a.ex.n_exit) atomicAdd(a.ex.n_exit, n_ex);
      if (a.ex.ramp_count) atomicAdd(a.ex.ramp_count + a.ramp_index, n_ex);
    }
  }
};

template <int VPL>
__global__ void __launch_bounds__(kT, 2) ramp_bert2_kernel(RampArgs a, float *part, RCtr ctr) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  __shared__ int s_flag;
  const int kSl = ramp_slices(a.H);
  RampSlice<VPL> rs(a, smem_raw, blockIdx.x / kSl, blockIdx.x % kSl);
  rs.prefetch();
  LnParams<VPL> lp;
  if (a.ln_g)
    ln_load_params<VPL>(lp, reinterpret_cast<const __nv_bfloat16 *>(a.ln_g),
                        reinterpret_cast<const __nv_bfloat16 *>(a.ln_b), a.H, lane_id());
  const unsigned long long tl0 = tl_now();
  pdl_wait();
  const unsigned long long tl1 = tl_now();
  const int n_valid = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  rs.compute(lp, n_valid, part);
  const unsigned long long tl2 = tl_now();
  const bool dec = rs.arrive(ctr, &s_flag);
  if (dec) rs.decide(n_valid, part);
  __syncthreads();
  pdl_trigger();
  if (threadIdx.x == 0) {
    tl_rec(g_tl, 74, tl0, tl1);                          // ramp2: entry | release | end
    tl_rec(g_tl, dec ? 76 : 75, tl1, tl2);               // slice computed (75) / decider (76): release | partials | end
  }
}

// block scan of the alive flags (ballot / popc per 32, serial over words)
__device__ __forceinline__ int scan_flags(const uint8_t *alive, int B, int16_t *src_of, int16_t *pos_of,
                                          int *word_cnt) {
  const int warp = warp_id(), lane = lane_id();
  const int nwords = (B + 31) / 32;
  for (int w = warp; w < nwords; w += kNW) {
    const int i = w * 32 + lane;
    const unsigned bal = __ballot_sync(0xffffffffu, i < B && __ldcg(alive + i) != 0);
    if (lane == 0) word_cnt[w] = __popc(bal);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int run = 0;
    for (int w = 0; w < nwords; ++w) {
      const int c = word_cnt[w];
      word_cnt[w] = run;
      run += c;
    }
    word_cnt[nwords] = run;
  }
  __syncthreads();
  for (int w = warp; w < nwords; w += kNW) {
    const int i = w * 32 + lane;
    const bool f = i < B && __ldcg(alive + i) != 0;
    const unsigned bal = __ballot_sync(0xffffffffu, f);
    const int pos = word_cnt[w] + __popc(bal & ((1u << lane) - 1u));
    if (f) src_of[pos] = (int16_t)i;
    if (i < B) pos_of[i] = f ? (int16_t)pos : (int16_t)-1;
  }
  __syncthreads();
  return word_cnt[nwords];
}

// cooperative launch: every CTA co-resident (the compaction role waits for the
// ramp role of other CTAs)
template <int VPL>
__global__ void __launch_bounds__(kT, 2)
    ramp_compact_kernel(RampArgs a, float *part, RCtr ctr, RingDst dst, int32_t *n_surv_dev, int n_ramp_ctas) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  __shared__ int16_t src_of[kMaxBc];
  __shared__ int16_t pos_of[kMaxBc];
  __shared__ int word_cnt[kMaxBc / 32 + 1];
  __shared__ int s_flag;
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  const int warp = warp_id(), lane = lane_id();
  const int H = a.H, S = a.S, B = a.B;
  const int kSl = ramp_slices(H);
  const bool ramp_cta = (int)blockIdx.x < n_ramp_ctas;
  RampSlice<VPL> rs(a, smem_raw, blockIdx.x / kSl, blockIdx.x % kSl);
  if (ramp_cta) rs.prefetch();
  LnParams<VPL> lp;
  ln_load_params<VPL>(lp, reinterpret_cast<const __nv_bfloat16 *>(a.ln_g),
                      reinterpret_cast<const __nv_bfloat16 *>(a.ln_b), H, lane);
  pdl_wait();
  const unsigned long long tl1 = tl_now();
  const int n_valid = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  // this CTA's token rows (pre-LN y): loads in flight before any ramp work
  const __nv_bfloat16 *y = reinterpret_cast<const __nv_bfloat16 *>(a.x);
  const int stride = gridDim.x * kNW;
  const int all_units = B * S;
  uint4 v[kRowsFly][VPL];
#pragma unroll
  for (int jj = 0; jj < kRowsFly; ++jj) {
    const int u = blockIdx.x * kNW + warp + jj * stride;
    if (u < all_units) ln_load_row<VPL>(v[jj], y + (size_t)u * H, H, lane);
  }
  const unsigned long long tlr0 = tl_now();
  if (ramp_cta) {
    rs.compute(lp, n_valid, part);
    if (threadIdx.x == 0) tl_rec(tlb, 72, tl1, tlr0);     // ramp slice: release | rows issued | computed
    if (rs.arrive(ctr, &s_flag)) {
      if (threadIdx.x == 0) tl_rec(tlb, 73, tl1, tl1);    // decider start
      rs.decide(n_valid, part);
      __syncthreads();
      if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(ctr.groups_done, 1u);
      }
    }
  }
#pragma unroll
  for (int jj = 0; jj < kRowsFly; ++jj) {   // LayerNorm while the decisions are pending
    const int u = blockIdx.x * kNW + warp + jj * stride;
    if (u < all_units) ln_apply<VPL>(v[jj], lp, H, a.eps, lane);
  }
  const unsigned groups = (unsigned)((B + kGRows - 1) / kGRows);
  if (threadIdx.x == 0)
    while (ld_acquire(ctr.groups_done) < groups) __nanosleep(64);
  __syncthreads();
  pdl_trigger();
  const unsigned long long tl2 = tl_now();
  const int64_t tail = dst.tail_dev ? *dst.tail_dev : 0;
  const int n = scan_flags(a.alive, B, src_of, pos_of, word_cnt);
  const bool fits = (tail - dst.head) + n <= dst.cap;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    const int out = fits ? n : 0;
    if (!fits && dst.overflow_dev) *dst.overflow_dev = 1;
    if (dst.tail_out) *dst.tail_out = fits ? tail + n : tail;
    if (n_surv_dev) *n_surv_dev = out;
    if (dst.mailbox) *dst.mailbox = fits ? out : -1;
  }
  if (fits && n > 0) {
    __nv_bfloat16 *ring = reinterpret_cast<__nv_bfloat16 *>(dst.rows);
    const size_t row_elems = (size_t)S * H;
#pragma unroll
    for (int jj = 0; jj < kRowsFly; ++jj) {
      const int u = blockIdx.x * kNW + warp + jj * stride;
      if (u < all_units) {
        const int b = u / S, t = u - b * S;
        const int k = pos_of[b];
        if (k >= 0) ln_store_row<VPL>(v[jj], ring + ((tail + k) % dst.cap) * row_elems + (size_t)t * H, H, lane);
      }
    }
    if (blockIdx.x == 0)
      for (int k = threadIdx.x; k < n; k += kT) dst.ids[(tail + k) % dst.cap] = a.id[src_of[k]];
  }
  // the last CTA out resets the decision counter for the next launch
  __syncthreads();
  if (threadIdx.x == 0) {
    if (atomicAdd(ctr.exit_ctr, 1u) == gridDim.x - 1) {
      *ctr.groups_done = 0;
      *ctr.exit_ctr = 0;
    }
    tl_rec(tlb, 70, tl0, tl1);
    tl_rec(tlb, 71, tl1, tl2);
  }
}

template <int VPL>
e3_status rc_occupancy(int smem, int *occ) {
  static int cache[2] = {0, 0};
  static int cached_smem = -1;
  if (cached_smem != smem) {
    E3_CUDA_TRY(cudaFuncSetAttribute(ramp_compact_kernel<VPL>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    E3_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&cache[0], ramp_compact_kernel<VPL>, kT, smem));
    cached_smem = smem;
  }
  *occ = cache[0];
  return E3_OK;
}

}  // namespace

E3_TL_SETTER(tl_set_rampc)

bool ramp_ticket_mode() {
  static const bool on = getenv("E3_RAMP_TICKET") != nullptr || getenv("E3_FUSED_RC") != nullptr;
  return on;
}

bool ramp_bert2_supported(int H, int C) {
  const int kSl = ramp_slices(H);
  // partials [groups][kSl][16][C] f32 live in the [B, H] f32 pool workspace
  // (and their smem copy in the decider, [kSl][16][C] in the [8][16][TN] partial-sum buffer)
  return C >= 1 && C <= kMaxCl && H % (8 * kSl) == 0 && H <= 1024 && H / kSl <= 32 && kSl * C <= H &&
         kSl * kSl * C <= 8 * H;
}

static RCtr make_ctr(unsigned *ctr_words) {
  RCtr c;
  c.tickets = ctr_words + 1;
  c.groups_done = ctr_words + kRampCtrGroupsDone;
  c.exit_ctr = ctr_words + kRampCtrExit;
  return c;
}

e3_status ramp_bert2_run(const RampArgs &a, unsigned *ctr_words, cudaStream_t st) {
  if (!ramp_bert2_supported(a.H, a.C) || a.B > kMaxBc) {
    set_error("ramp: need 1 <= C <= 16, H % (8 slices) == 0, H <= 1024");
    return E3_EUNSUPPORTED;
  }
  const int kSl = ramp_slices(a.H);
  const int groups = (a.B + kGRows - 1) / kGRows;
  const int smem = rslice_smem_bytes(a.H, a.C);
  const int vpl = (a.H / 8 + 31) / 32;
  const RCtr c = make_ctr(ctr_words);
#define E3_R2(V)                                                                                                \
  do {                                                                                                          \
    static int done = 0;                                                                                        \
    if (done != smem) {                                                                                         \
      E3_CUDA_TRY(cudaFuncSetAttribute(ramp_bert2_kernel<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)); \
      done = smem;                                                                                              \
    }                                                                                                           \
    E3_CUDA_TRY(launch_k(ramp_bert2_kernel<V>, dim3(groups * kSl), dim3(kT), (size_t)smem, st, a, a.pool_ws, c)); \
  } while (0)
  if (vpl <= 1) E3_R2(1);
  else if (vpl <= 3) E3_R2(3);
  else E3_R2(4);
#undef E3_R2
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

e3_status ramp_compact_run(const RampArgs &a, unsigned *ctr_words, const RingDst &dst, int32_t *n_surv_dev, int sms,
                           cudaStream_t st, bool *done) {
  *done = false;
  // Off by default (E3_FUSED_RC=1 enables it): measured on B200 (scripts/timeline.py bb, r02) the fused
  // launch took 21.8 us per BB split run from FFN2's end to the next QKV GEMM against 20.5 us for the
  // ticketed ramp + ln_compact pair (154.1 vs 148.8 us per run): its decision chain (slice partials,
  // ticket, partial reload, decision) slows while 296 CTAs stream the 12.6 MB of token rows beside it,
  // which outweighs the saved kernel boundary.
  static const bool on = getenv("E3_FUSED_RC") != nullptr;
  if (!on || !ramp_bert2_supported(a.H, a.C) || a.B > kMaxBc || !a.ln_g) return E3_OK;
  const int kSl = ramp_slices(a.H);
  const int groups = (a.B + kGRows - 1) / kGRows;
  const int n_ramp = groups * kSl;
  const int smem = rslice_smem_bytes(a.H, a.C);
  const int vpl = (a.H / 8 + 31) / 32;
  int occ = 0;
  e3_status r = E3_OK;
  if (vpl <= 1) r = rc_occupancy<1>(smem, &occ);
  else if (vpl <= 3) r = rc_occupancy<3>(smem, &occ);
  else r = rc_occupancy<4>(smem, &occ);
  if (r != E3_OK) return r;
  const int grid = occ * sms;
  // every token row must have a slot (rows are held in registers across the
  // wait) and every ramp slice a CTA; otherwise the two-kernel path runs
  if (occ < 1 || n_ramp > grid || (int64_t)a.B * a.S > (int64_t)kRowsFly * kNW * grid) return E3_OK;
  const RCtr c = make_ctr(ctr_words);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kT);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  auto go = [&]() {
    if (vpl <= 1) return cudaLaunchKernelEx(&cfg, ramp_compact_kernel<1>, a, a.pool_ws, c, dst, n_surv_dev, n_ramp);
    if (vpl <= 3) return cudaLaunchKernelEx(&cfg, ramp_compact_kernel<3>, a, a.pool_ws, c, dst, n_surv_dev, n_ramp);
    return cudaLaunchKernelEx(&cfg, ramp_compact_kernel<4>, a, a.pool_ws, c, dst, n_surv_dev, n_ramp);
  };
  static bool coop_pdl_ok = true;   // cooperative + programmatic serialization, if the driver takes both
  if (!coop_pdl_ok) cfg.numAttrs = 1;
  cudaError_t e = go();
  if (e != cudaSuccess && cfg.numAttrs == 2) {
    cudaGetLastError();
    coop_pdl_ok = false;
    cfg.numAttrs = 1;
    e = go();
  }
  E3_CUDA_TRY(e);
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  *done = true;
  return E3_OK;
}

}  // namespace e3
