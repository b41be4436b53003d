// Fused exit ramp + threshold test.
//
// DeeBERT ramp after an encoder block: "a bertpooler, a dropout layer, and a
// fully connected layer" (R1):
//     c = x[b, 0, :]   p = tanh(W_p c + b_p)   z = W_c p + b_c
// exit test (R3/R4/R12): max softmax(z) > tau, or
// entropy(softmax(z)) < tau; the model's last ramp exits every row (R6).
//
// One launch; grid (16, ceil(B / 16)): one cluster of 16 CTAs per group of
// 16 rows (the mma M), CTA rank r owning pooler outputs [r*TN, (r+1)*TN),
// TN = H/16.  The work is spread over B/16 x 16 SMs (BB: 64) -- measured on
// B200 the ramp is instruction-issue-bound per SM, so fewer, fatter CTAs
// (one cluster for the whole batch) were 1.6x slower:
//   stage    the CTA's TN W_p rows by cp.async into padded smem (row pitch
//            H + 8 bf16: conflict-free fragments), its W_c / b_p slices as
//            fp32, all BEFORE the PDL wait;
//   CLS      every CTA normalises the group's 16 CLS rows itself (warp w:
//            rows w and w + 8; at a split's last layer the rows arrive
//            PRE-LayerNorm and the shared warp-per-row LN of ln_row.cuh makes
//            them bit-identical to what the fused LN + compaction writes) --
//            redundant across the cluster but one L2 round trip, where a
//            DSMEM broadcast from one warp per CTA cost a serial store chain
//            and a cluster barrier (r01 timeline: 3 us);
//   pooler   mma.sync m16n8k16 bf16 -> fp32 with K split over the 8 warps
//            (warp w: k16 steps w, w + 8, ...; NT = TN / 8 independent chains
//            per warp instead of one 48-step chain on 6 of 8 warps), per-warp
//            partials summed in warp order through smem, p = tanh(. + b_p);
//   partial  partial logits sum_{o in CTA} p[b,o] W_c[c,o] by warp shuffles,
//            stored into rank 0's shared memory (DSMEM);
//   decide   after a cluster barrier rank 0 sums the 16 partials per (row,
//            class) in rank order, then softmax / max-prob / entropy, argmax
//            (lowest index on ties), threshold test, exit record by input id
//            and the alive flag.  Deterministic: no float atomics anywhere.
// All ramp math is fp32, never rounded to bf16 (rounding contract).
// The ViT ramp (LayerNorm + linear over C <= 2048 classes) is ramp_vit_kernel
// below.
#include "common.cuh"
#include "exitrule.cuh"
#include "kernels.h"
#include "ln_row.cuh"
#include "softstat.cuh"
#include "prof.h"

namespace e3 {

namespace {

constexpr int kMaxC = 16;
constexpr int kCS = 16;          // cluster size (non-portable)
constexpr int kRows = 16;        // rows per cluster (mma M)
constexpr int kRThreads = 256;

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

__device__ __forceinline__ void st_cluster_f32(uint32_t addr, float v) {
  asm volatile("st.shared::cluster.f32 [%0], %1;" ::"r"(addr), "f"(v) : "memory");
}
__device__ __forceinline__ void st_cluster_v4(uint32_t addr, uint4 v) {
  asm volatile("st.shared::cluster.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w)
               : "memory");
}

// split cluster barrier: arrive at kernel start, wait before the first DSMEM
// access, so every CTA of the cluster is known to be running
__device__ __forceinline__ void cluster_arrive_relaxed() {
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
}
__device__ __forceinline__ void cluster_wait() { asm volatile("barrier.cluster.wait.aligned;" ::: "memory"); }

__device__ __forceinline__ bool row_alive(const RampArgs &a, int b, int n_valid) {
  return b < a.B && (a.init_alive ? (b < n_valid) : (a.alive[b] != 0));
}

// smem: W tile [TN][P] bf16 | CLS [16][P] bf16 | per-warp pooler partials
// [8][16][TN] f32 | pooled p [16][TN] f32 | W_c slice [C][TN] f32 | b_p slice
// [TN] f32 | cluster partials (rank 0) [kCS][16][C] f32
__host__ __device__ inline int ramp_smem_bytes(int H, int C) {
  const int TN = H / kCS, P = H + 8;
  return (TN + kRows) * P * 2 + (kRThreads / 32) * kRows * TN * 4 + kRows * TN * 4 + C * TN * 4 + TN * 4 +
         kCS * kRows * C * 4;
}

template <int VPL>
__global__ void __launch_bounds__(kRThreads, 1) ramp_bert_kernel(RampArgs a) {
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  extern __shared__ uint8_t smem_raw[];
  constexpr int nw = kRThreads / 32;
  constexpr int kMaxNT = 2 * VPL;                        // TN / 8 <= H / 128
  const int H = a.H, C = a.C;
  const int TN = H / kCS, NT = TN / 8;
  const int P = H + 8;                                   // padded pitch (bf16)
  __nv_bfloat16 *sW = reinterpret_cast<__nv_bfloat16 *>(smem_raw);   // [TN][P]
  __nv_bfloat16 *sC = sW + TN * P;                                    // [16][P]
  float *sRed = reinterpret_cast<float *>(sC + kRows * P);            // [nw][16][TN]
  float *sP = sRed + nw * kRows * TN;                                 // [16][TN]
  float *sWc = sP + kRows * TN;                                       // [C][TN]
  float *sBp = sWc + C * TN;                                          // [TN]
  float *sQ = sBp + TN;                                               // [kCS][16][C] (rank 0)
  __shared__ bool row_ok[kRows];

  const int warp = warp_id(), lane = lane_id();
  const int gq = lane >> 2, tq = lane & 3;
  const uint32_t rank = cluster_ctarank();
  const int b0 = blockIdx.y * kRows;
  const int o0 = (int)rank * TN;
  const int nvec = H / 8;
  const __nv_bfloat16 *x = reinterpret_cast<const __nv_bfloat16 *>(a.x);
  const size_t row_stride = (size_t)a.S * H;

  cluster_arrive_relaxed();
  // ---------------------------------------------------------- weights: no dependency
  const uint4 *wp = reinterpret_cast<const uint4 *>(a.w.w_p);
  for (int i = threadIdx.x; i < TN * nvec; i += kRThreads) {
    const int r = i / nvec, k = i - r * nvec;
    cp_async16(reinterpret_cast<uint4 *>(sW + r * P) + k, wp + (size_t)(o0 + r) * nvec + k);
  }
  {
    const __nv_bfloat16 *wc = reinterpret_cast<const __nv_bfloat16 *>(a.w.w_c);
    const __nv_bfloat16 *bp = reinterpret_cast<const __nv_bfloat16 *>(a.w.b_p);
    for (int i = threadIdx.x; i < C * TN; i += kRThreads) {
      const int c = i / TN, o = i - c * TN;
      sWc[i] = bf2f(wc[(size_t)c * H + o0 + o]);
    }
    for (int i = threadIdx.x; i < TN; i += kRThreads) sBp[i] = bf2f(bp[o0 + i]);
  }
  LnParams<VPL> lp;
  if (a.ln_g)
    ln_load_params<VPL>(lp, reinterpret_cast<const __nv_bfloat16 *>(a.ln_g),
                        reinterpret_cast<const __nv_bfloat16 *>(a.ln_b), H, lane);
  pdl_wait();                      // CLS rows / alive flags of the previous kernels now visible
  const unsigned long long tl1 = tl_now();
  const int n_valid = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  if (threadIdx.x < kRows) row_ok[threadIdx.x] = row_alive(a, b0 + threadIdx.x, n_valid);

  // ---------------------------------------------------------- CLS rows: every CTA normalises all 16
  // itself (warp w: rows w and w + 8; at a split's last layer the rows arrive
  // PRE-LayerNorm, and the shared warp-per-row LN of ln_row.cuh makes them
  // bit-identical to what the fused LN + compaction writes)
  {
    uint4 v[2][VPL];
    bool ok[2];
#pragma unroll
    for (int j = 0; j < 2; ++j) {
      const int r = warp + j * nw;
      ok[j] = row_alive(a, b0 + r, n_valid);
      if (ok[j]) ln_load_row<VPL>(v[j], x + (size_t)(b0 + r) * row_stride, H, lane);
    }
#pragma unroll
    for (int j = 0; j < 2; ++j) {
      const int r = warp + j * nw;
      if (ok[j]) {
        if (a.ln_g) ln_apply<VPL>(v[j], lp, H, a.eps, lane);
      } else {
#pragma unroll
        for (int i = 0; i < VPL; ++i) v[j][i] = make_uint4(0, 0, 0, 0);
      }
      uint4 *dst = reinterpret_cast<uint4 *>(sC + r * P);
#pragma unroll
      for (int i = 0; i < VPL; ++i)
        if (lane + 32 * i < nvec) dst[lane + 32 * i] = v[j][i];
    }
  }
  cp_async_wait_all();
  __syncthreads();                 // CLS rows and the W tile in smem
  const unsigned long long tl2 = tl_now();

  // ---------------------------------------------------------- pooler: K split over the warps
  // warp w accumulates the k16 steps w, w + 8, ... for all NT n8 tiles (NT
  // independent mma chains), partials summed across warps in warp order
  {
    float acc[kMaxNT][4];
#pragma unroll
    for (int t = 0; t < kMaxNT; ++t) acc[t][0] = acc[t][1] = acc[t][2] = acc[t][3] = 0.f;
    const __nv_bfloat16 *a_lo = sC + gq * P + 2 * tq;
    const __nv_bfloat16 *a_hi = sC + (gq + 8) * P + 2 * tq;
    const __nv_bfloat16 *bw = sW + gq * P + 2 * tq;
    for (int k = 16 * warp; k < H; k += 16 * nw) {
      uint32_t af[4];
      af[0] = *reinterpret_cast<const uint32_t *>(a_lo + k);
      af[1] = *reinterpret_cast<const uint32_t *>(a_hi + k);
      af[2] = *reinterpret_cast<const uint32_t *>(a_lo + k + 8);
      af[3] = *reinterpret_cast<const uint32_t *>(a_hi + k + 8);
#pragma unroll
      for (int t = 0; t < kMaxNT; ++t) {
        if (t < NT) {
          const uint32_t bf0 = *reinterpret_cast<const uint32_t *>(bw + t * 8 * P + k);
          const uint32_t bf1 = *reinterpret_cast<const uint32_t *>(bw + t * 8 * P + k + 8);
          mma_bf16_16816(acc[t], af, bf0, bf1);
        }
      }
    }
    float *red = sRed + warp * kRows * TN;
#pragma unroll
    for (int t = 0; t < kMaxNT; ++t) {
      if (t < NT) {
        const int col = t * 8 + 2 * tq;
        *reinterpret_cast<float2 *>(red + gq * TN + col) = make_float2(acc[t][0], acc[t][1]);
        *reinterpret_cast<float2 *>(red + (gq + 8) * TN + col) = make_float2(acc[t][2], acc[t][3]);
      }
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < kRows * TN; i += kRThreads) {
    float s = sRed[i];
#pragma unroll
    for (int w = 1; w < nw; ++w) s += sRed[w * kRows * TN + i];
    sP[i] = tanhf(s + sBp[i % TN]);              // p = tanh(W_p c + b_p)
  }
  __syncthreads();
  // partial logits over this CTA's TN pooler outputs: warp w, rows w and w + 8
  cluster_wait();                  // every CTA of the cluster is running (DSMEM below)
  for (int j = 0; j < 2; ++j) {
    const int r = warp + j * nw;
    for (int c = 0; c < C; ++c) {
      float z = 0.f;
      for (int o = lane; o < TN; o += 32) z = fmaf(sP[r * TN + o], sWc[c * TN + o], z);
#pragma unroll
      for (int off = 16; off; off >>= 1) z += __shfl_xor_sync(0xffffffffu, z, off);
      if (lane == 0) st_cluster_f32(mapa_shared(smem_u32(sQ + ((int)rank * kRows + r) * C + c), 0), z);
    }
  }
  // rank 0 decides row r = threadIdx.x < 16: its id and the class biases are
  // fetched before the cluster barrier
  const int r = threadIdx.x;
  const int b = b0 + r;
  const bool decider = rank == 0 && r < kRows && b < a.B;
  int64_t row_id = -1;
  float bcv[kMaxC];
#pragma unroll
  for (int c = 0; c < kMaxC; ++c)
    bcv[c] = (decider && c < C) ? bf2f(reinterpret_cast<const __nv_bfloat16 *>(a.w.b_c)[c]) : 0.f;
  if (decider) row_id = a.id[b];
  const unsigned long long tl3 = tl_now();
  cluster_sync();                  // every CTA's partials are in rank 0's smem
  const unsigned long long tlA = tl_now();
  if (threadIdx.x == 0 && rank != 0) tl_rec(tlb, 40, tl2, tl3);   // phases: CLS + W ready, partials stored, synced
  unsigned long long tlB = 0;
  // PDL trigger only once the decision is written (non-deciding CTAs trigger
  // by exiting): dependent CTAs made resident earlier sit in
  // griddepcontrol.wait on the deciding CTA's SM and slowed its few hundred
  // instructions from <1 to ~3 us (r01 timeline); before the pooler they cost
  // +6 us
  if (rank != 0 || warp != 0) {
    if (threadIdx.x == 0) tl_rec(tlb, 4, tl0, tl1);
    return;
  }

  // ---------------------------------------------------------- decide (rank 0)
  bool exit_now = false;
  if (decider && !row_ok[r]) {
    if (a.init_alive) a.alive[b] = 0;
  } else if (decider) {
    float z[kMaxC];
#pragma unroll
    for (int c = 0; c < kMaxC; ++c) {
      z[c] = 0.f;
      if (c < C) {
        float s = 0.f;
        for (int q = 0; q < kCS; ++q) s += sQ[(q * kRows + r) * C + c];   // fixed order
        z[c] = s + bcv[c];
      }
    }
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
    if (a.test == E3_TEST_PATIENCE) {
      pass = patience_step(a.ex.state, row_id, a.ex.capacity, label, a.tau, &metric);
    } else if (a.test == E3_TEST_MAXPROB) {
      metric = 1.0f / sum;                       // max_c softmax(z)_c
      pass = metric > a.tau;
    } else {
      metric = logf(sum) - qz / sum;             // H = lse - sum_c q_c z_c
      pass = metric < a.tau;
    }
    exit_now = pass || a.final_ramp;
    if (a.ex.ramp_metric && row_id >= 0 && row_id < a.ex.capacity)
      a.ex.ramp_metric[row_id * a.ex.ramp_metric_stride + a.ramp_index] = metric;
    tlB = tl_now();
    if (exit_now) {
      const int64_t id = row_id;
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
    }
    a.alive[b] = exit_now ? 0 : 1;
  }
  // one counter update per warp (exit counts are order-independent)
  const int n_ex = __popc(__ballot_sync(0xffffffffu, exit_now));
  if (lane == 0 && n_ex) {
    if (a.ex.n_exit) atomicAdd(a.ex.n_exit, n_ex);
    if (a.ex.ramp_count) atomicAdd(a.ex.ramp_count + a.ramp_index, n_ex);
  }
  __syncwarp();
  pdl_trigger();
  if (threadIdx.x == 0) tl_rec(tlb, 5, tl0, tl1);   // rank 0: the decision is written
  if (threadIdx.x == 0) tl_rec(tlb, 41, tlA, tlB);
}

// ============================================================== ViT ramp
// ViT exit ramp (R1): n = LN_r(x[b, 0, :]) (the ramp's own
// LayerNorm), z = W_c n + b_c over C classes (C = 1000 for EE-ViT-B/16).  All
// fp32: the normalised row is never rounded (rounding contract), so the
// classifier runs on the FMA pipe (B x H x C = 197 MFMA per call at VT; a few
// microseconds spread over the grid).
//
// grid (CS, ceil(B / 16)), clusters of CS = ceil(C / CB) CTAs: CTA rank r owns
// classes [r*CB, (r+1)*CB) of one group of 16 rows.  Thread t owns the class
// pair 2j, 2j+1 (j = t mod CB/2) for the 4 rows of row group t / (CB/2); every
// lane of a warp reads the same normalised row values (smem broadcast) and its
// own two classifier rows (16-byte loads).  Per row and CTA the softmax
// statistics are reduced to (max m, argmax, s = sum e^(z-m), u = sum
// e^(z-m)(z-m)) and sent to rank 0 through DSMEM; rank 0 merges the CS
// partials in rank order (exact merge of log-sum-exp partials), tests the
// threshold, writes the record and the alive flag, and publishes the decision;
// each CTA then writes its slice of the logits of the exiting rows.
constexpr int kVitRows = 16;
constexpr int kVitKQ = 4;                              // CTA = kVitKQ x 2 CB threads = 8 per class

__device__ __forceinline__ int ld_cluster_s32(uint32_t addr) {
  int v;
  asm volatile("ld.shared::cluster.s32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
  return v;
}

template <int CB, bool kLate>
__global__ void __launch_bounds__(kVitKQ * 2 * CB) ramp_vit_kernel(RampArgs a, int CS) {
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  // 8 threads per class for the classifier; the first 2 CB threads then own
  // 2 classes x 4 rows each for the softmax statistics and the logits
  constexpr int kThreads = 2 * CB, kWarps = kThreads / 32, kWarpsPerRg = CB / 64;
  constexpr int kAll = kVitKQ * kThreads, kAllWarps = kAll / 32;
  constexpr int kVitCls = CB;
  extern __shared__ float sN[];                       // [16][H + 4] normalised CLS rows (fp32)
  __shared__ SoftStat sRed[kWarps][4];
  __shared__ SoftStat sQ[16][kVitRows];               // rank 0: [rank][row]
  __shared__ int sDec[kVitRows];                      // rank 0: 1 = row exits here
  __shared__ bool row_ok[kVitRows];
  const int H = a.H, P = H + 4, C = a.C;
  const int tAll = threadIdx.x;
  const int t = tAll % kThreads, warp = t >> 5, lane = t & 31, wAll = tAll >> 5;
  const uint32_t rank = cluster_ctarank();
  const int b0 = blockIdx.y * kVitRows;
  const int j = t % (CB / 2), rg = t / (CB / 2);
  const int c0 = (int)rank * CB + 2 * j, c1 = c0 + 1;
  const __nv_bfloat16 *W = reinterpret_cast<const __nv_bfloat16 *>(a.w.w_c);
  const __nv_bfloat16 *bc = reinterpret_cast<const __nv_bfloat16 *>(a.w.b_c);
  const float bias0 = c0 < C ? bf2f(bc[c0]) : 0.f, bias1 = c1 < C ? bf2f(bc[c1]) : 0.f;
  cluster_arrive_relaxed();

  pdl_wait();
  if (!kLate) pdl_trigger();
  const unsigned long long tl1 = tl_now();
  const int n_valid = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  if (tAll < kVitRows) row_ok[tAll] = row_alive(a, b0 + tAll, n_valid);
  __syncthreads();

  // ---- LayerNorm of the CLS rows (two passes, fp32), one warp per row
  const __nv_bfloat16 *x = reinterpret_cast<const __nv_bfloat16 *>(a.x);
  const __nv_bfloat16 *lg = reinterpret_cast<const __nv_bfloat16 *>(a.w.ln_g);
  const __nv_bfloat16 *lb = reinterpret_cast<const __nv_bfloat16 *>(a.w.ln_b);
  for (int r = wAll; r < kVitRows; r += kAllWarps) {
    float *row = sN + r * P;
    if (!row_ok[r]) {
      for (int k = lane; k < H; k += 32) row[k] = 0.f;
      continue;
    }
    const __nv_bfloat16 *xr = x + (size_t)(b0 + r) * a.S * H;
    float s = 0.f;
    for (int k = lane; k < H; k += 32) {
      const float v = bf2f(xr[k]);
      row[k] = v;
      s += v;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const float mean = s / (float)H;
    float q = 0.f;
    for (int k = lane; k < H; k += 32) {
      const float d = row[k] - mean;
      q += d * d;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
    const float rstd = 1.0f / sqrtf(q / (float)H + a.eps);
    for (int k = lane; k < H; k += 32) row[k] = (row[k] - mean) * rstd * bf2f(lg[k]) + bf2f(lb[k]);
  }
  __syncthreads();

  const unsigned long long tlLn = tl_now();
  // ---- classifier, fp32 FMA over K = H: thread (class cl, k lane q) sums
  // k = 8q + 64i for all 16 rows, so the 8 lanes of a class read 128
  // contiguous bytes of its W_c row per step (one class row per lane was a
  // 32-line scattered load per instruction: ~60 us per launch at VT, r01);
  // partial sums are reduced over q by shuffles in a fixed order
  __shared__ float sZ[kVitRows][kVitCls];
  {
    const int cl = tAll >> 3, q = tAll & 7;
    const int cg = (int)rank * CB + cl;
    float acc[kVitRows];
#pragma unroll
    for (int r = 0; r < kVitRows; ++r) acc[r] = 0.f;
    if (cg < C) {
      const uint4 *wr = reinterpret_cast<const uint4 *>(W + (size_t)cg * H);
#pragma unroll 2
      for (int k = 8 * q; k < H; k += 64) {
        const uint4 w = __ldg(wr + k / 8);
        const float wf[8] = {bf_lo(w.x), bf_hi(w.x), bf_lo(w.y), bf_hi(w.y),
                             bf_lo(w.z), bf_hi(w.z), bf_lo(w.w), bf_hi(w.w)};
#pragma unroll
        for (int r = 0; r < kVitRows; ++r) {
          const float4 n0 = *reinterpret_cast<const float4 *>(sN + r * P + k);
          const float4 n1 = *reinterpret_cast<const float4 *>(sN + r * P + k + 4);
          float v = acc[r];
          v = fmaf(n0.x, wf[0], v);
          v = fmaf(n0.y, wf[1], v);
          v = fmaf(n0.z, wf[2], v);
          v = fmaf(n0.w, wf[3], v);
          v = fmaf(n1.x, wf[4], v);
          v = fmaf(n1.y, wf[5], v);
          v = fmaf(n1.z, wf[6], v);
          v = fmaf(n1.w, wf[7], v);
          acc[r] = v;
        }
      }
    }
#pragma unroll
    for (int r = 0; r < kVitRows; ++r) {
      float v = acc[r];
      v += __shfl_xor_sync(0xffffffffu, v, 1);
      v += __shfl_xor_sync(0xffffffffu, v, 2);
      v += __shfl_xor_sync(0xffffffffu, v, 4);
      if (q == 0) sZ[r][cl] = v;
    }
  }
  __syncthreads();
  const unsigned long long tlCls = tl_now();
  // threads t < 2 CB continue with 2 classes x 4 rows each
  const bool g0 = tAll < kThreads;
  float z[4][2];
#pragma unroll
  for (int rr = 0; rr < 4; ++rr) {
    z[rr][0] = (g0 ? sZ[rg * 4 + rr][2 * j] : 0.f) + bias0;
    z[rr][1] = (g0 ? sZ[rg * 4 + rr][2 * j + 1] : 0.f) + bias1;
  }

  // ---- per-row softmax statistics of this CTA's classes
#pragma unroll
  for (int rr = 0; rr < 4; ++rr) {
    SoftStat st{-INFINITY, 0.f, 0.f, -1};
    if (c0 < C) st = SoftStat{z[rr][0], 1.f, 0.f, c0};
    if (c1 < C) st = soft_merge(st, SoftStat{z[rr][1], 1.f, 0.f, c1});
#pragma unroll
    for (int o = 16; o; o >>= 1) st = soft_merge(st, soft_shfl_xor(st, o));
    if (lane == 0 && g0) sRed[warp][rr] = st;
  }
  __syncthreads();
  cluster_wait();                            // every CTA of the cluster is running
  if (g0 && t < kVitRows) {                  // row t: merge this CTA's warps, send to rank 0
    const int g = t / 4, rr = t % 4;
    SoftStat st = sRed[g * kWarpsPerRg][rr];
    for (int w = 1; w < kWarpsPerRg; ++w) st = soft_merge(st, sRed[g * kWarpsPerRg + w][rr]);
    const uint32_t dst = mapa_shared(smem_u32(&sQ[rank][t]), 0);
    st_cluster_f32(dst, st.m);
    st_cluster_f32(dst + 4, st.s);
    st_cluster_f32(dst + 8, st.u);
    asm volatile("st.shared::cluster.s32 [%0], %1;" ::"r"(dst + 12), "r"(st.idx) : "memory");
  }
  cluster_sync();

  // ---- rank 0 decides (rows t < 16 of warp 0)
  if (rank == 0 && warp == 0 && g0) {
    const int r = lane, b = b0 + r;
    bool exit_now = false;
    if (r < kVitRows && b < a.B) {
      if (!row_ok[r]) {
        if (a.init_alive) a.alive[b] = 0;
      } else {
        SoftStat st = sQ[0][r];
        for (int q = 1; q < CS; ++q) st = soft_merge(st, sQ[q][r]);
        float metric;
        bool pass;
        if (a.test == E3_TEST_PATIENCE) {
          pass = patience_step(a.ex.state, a.id[b], a.ex.capacity, st.idx, a.tau, &metric);
        } else if (a.test == E3_TEST_MAXPROB) {
          metric = 1.0f / st.s;
          pass = metric > a.tau;
        } else {
          metric = logf(st.s) - st.u / st.s;
          pass = metric < a.tau;
        }
        exit_now = pass || a.final_ramp;
        if (a.ex.ramp_metric && a.id[b] >= 0 && a.id[b] < a.ex.capacity)
          a.ex.ramp_metric[a.id[b] * a.ex.ramp_metric_stride + a.ramp_index] = metric;
        const int64_t id = a.id[b];
        if (exit_now && id >= 0 && id < a.ex.capacity) {
          if (a.ex.exit_layer) a.ex.exit_layer[id] = a.layer;
          if (a.ex.label) a.ex.label[id] = st.idx;
          if (a.ex.conf) a.ex.conf[id] = metric;
        }
        a.alive[b] = exit_now ? 0 : 1;
      }
    }
    if (r < kVitRows) sDec[r] = exit_now ? 1 : 0;
    const int n_ex = __popc(__ballot_sync(0xffffffffu, exit_now));
    if (lane == 0 && n_ex) {
      if (a.ex.n_exit) atomicAdd(a.ex.n_exit, n_ex);
      if (a.ex.ramp_count) atomicAdd(a.ex.ramp_count + a.ramp_index, n_ex);
    }
  }
  cluster_sync();
  // ---- logits of the exiting rows: each CTA writes its class slice
  if (a.ex.logits && g0) {
#pragma unroll
    for (int rr = 0; rr < 4; ++rr) {
      const int r = rg * 4 + rr, b = b0 + r;
      if (b >= a.B) continue;
      if (!ld_cluster_s32(mapa_shared(smem_u32(&sDec[r]), 0))) continue;
      const int64_t id = a.id[b];
      if (id < 0 || id >= a.ex.capacity) continue;
      if (c0 < C) a.ex.logits[id * C + c0] = z[rr][0];
      if (c1 < C) a.ex.logits[id * C + c1] = z[rr][1];
    }
  }
  cluster_sync();                            // rank 0's smem stays valid until every CTA has read it
  if (kLate) pdl_trigger();
  if (tAll == 0) tl_rec(tlb, 9, tl0, tl1);
  if (tAll == 0) tl_rec(tlb, 91, tlLn, tlCls);   // phases: CLS LN done, classifier done, end
}


// ViT ramp on the tensor cores (C <= 1024, H % 64 == 0, H <= 1024): the
// classifier z = W_c n over a cluster's 16 rows is a dense [16 x H] x [H x 64]
// contraction per CTA.  The fp32 normalised rows n are split exactly into
// three bf16 terms n = hi + mid + lo (|n - (hi + mid + lo)| <= 2^-24 |n|), so
// the three mma.sync m16n8k16 products with the bf16 W_c accumulate in fp32
// what the fp32 FMA loop computed (products of 8-bit mantissas are exact in
// fp32; only the summation order differs).  Warp w owns classes [8w, 8w + 8)
// of the CTA's 64; W_c's slice is staged by cp.async before the PDL wait.
// The old FMA kernel (kept for C > 1024) was shared-memory-bound re-reading
// the rows per class group: 100 us per VT launch (r01 timeline).
constexpr int kVtcThreads = 256;

constexpr int kVtcKC = 128;                            // K chunk of the staged W_c slice
constexpr int kVtcPW = kVtcKC + 8;                     // its padded pitch (bf16)
__host__ __device__ inline int ramp_vit_tc_smem(int H) {
  const int P = H + 8;
  return 3 * kVitRows * P * 2 + 2 * 128 * kVtcPW * 2;
}

template <bool kLate>
__global__ void __launch_bounds__(kVtcThreads, 1) ramp_vit_tc_kernel(RampArgs a, int CS) {
  // 128 classes per CTA (8 warps x two n8 tiles): clusters of <= 8 CTAs for
  // C <= 1024, all resident at once (16-CTA clusters of 64-class slices fit
  // one per GPC and ran in 2-3 waves)
  constexpr int CB = 128, kThreads = 2 * CB, kWarps = kThreads / 32, kWarpsPerRg = CB / 64;
  static_assert(kThreads == kVtcThreads, "all threads own 2 classes x 4 rows");
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  extern __shared__ uint8_t smem_raw[];
  const int H = a.H, C = a.C, P = H + 8;
  __nv_bfloat16 *sA = reinterpret_cast<__nv_bfloat16 *>(smem_raw);   // [3][16][P]: hi, mid, lo
  __nv_bfloat16 *sWc = sA + 3 * kVitRows * P;                         // [2][128][kVtcPW] W_c chunks
  __shared__ float sZ[kVitRows][CB];
  __shared__ SoftStat sRed[kWarps][4];
  __shared__ SoftStat sQ[16][kVitRows];               // rank 0: [rank][row]
  __shared__ int sDec[kVitRows];                      // rank 0: 1 = row exits here
  __shared__ bool row_ok[kVitRows];
  const int tAll = threadIdx.x, wAll = tAll >> 5;
  const int t = tAll % kThreads, warp = t >> 5, lane = t & 31;
  const int gq = lane >> 2, tq = lane & 3;
  const uint32_t rank = cluster_ctarank();
  const int b0 = blockIdx.y * kVitRows;
  const int j = t % (CB / 2), rg = t / (CB / 2);
  const int c0 = (int)rank * CB + 2 * j, c1 = c0 + 1;
  const __nv_bfloat16 *W = reinterpret_cast<const __nv_bfloat16 *>(a.w.w_c);
  const __nv_bfloat16 *bc = reinterpret_cast<const __nv_bfloat16 *>(a.w.b_c);
  const float bias0 = c0 < C ? bf2f(bc[c0]) : 0.f, bias1 = c1 < C ? bf2f(bc[c1]) : 0.f;
  const int nvec = H / 8;
  cluster_arrive_relaxed();
  // W_c slice [rank*128, +128) x H in K chunks of 128 through a double
  // buffer (cp.async, zero rows past C); chunk 0 before the PDL wait
  const int nch = (H + kVtcKC - 1) / kVtcKC;
  auto stage_chunk = [&](int c) {
    __nv_bfloat16 *dstb = sWc + (c & 1) * 128 * kVtcPW;
    const int k0 = c * kVtcKC, kw = min(kVtcKC, H - k0) / 8;   // 16-byte vectors per row
    for (int i = tAll; i < 128 * kw; i += kVtcThreads) {
      const int r = i / kw, v = i - r * kw;
      const int cls = (int)rank * CB + r;
      uint4 *d = reinterpret_cast<uint4 *>(dstb + r * kVtcPW) + v;
      if (cls < C) cp_async16(d, reinterpret_cast<const uint4 *>(W + (size_t)cls * H + k0) + v);
      else *d = make_uint4(0, 0, 0, 0);
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  stage_chunk(0);
  pdl_wait();
  if (!kLate) pdl_trigger();
  const unsigned long long tl1 = tl_now();
  const int n_valid = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
  if (tAll < kVitRows) row_ok[tAll] = row_alive(a, b0 + tAll, n_valid);

  // ---- LayerNorm of the CLS rows (fp32, two passes), warp w: rows w, w + 8;
  // lane l owns the 16-byte vectors l, l + 32, ... of the row
  {
    const __nv_bfloat16 *x = reinterpret_cast<const __nv_bfloat16 *>(a.x);
    const uint4 *lg = reinterpret_cast<const uint4 *>(a.w.ln_g);
    const uint4 *lb = reinterpret_cast<const uint4 *>(a.w.ln_b);
    constexpr int VM = 4;                              // H <= 1024
    for (int r = wAll; r < kVitRows; r += kVtcThreads / 32) {
      const bool ok = row_alive(a, b0 + r, n_valid);
      float v[VM][8];
      uint4 gv[VM], bv[VM];
      const uint4 *xr = reinterpret_cast<const uint4 *>(x + (size_t)(b0 + r) * a.S * H);
#pragma unroll
      for (int i = 0; i < VM; ++i) {
        const int k = lane + 32 * i;
        const uint4 u = (ok && k < nvec) ? xr[k] : make_uint4(0, 0, 0, 0);
        gv[i] = k < nvec ? __ldg(lg + k) : make_uint4(0, 0, 0, 0);
        bv[i] = k < nvec ? __ldg(lb + k) : make_uint4(0, 0, 0, 0);
        const uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          v[i][2 * e] = bf_lo(w[e]);
          v[i][2 * e + 1] = bf_hi(w[e]);
        }
      }
      float sum = 0.f;
#pragma unroll
      for (int i = 0; i < VM; ++i)
#pragma unroll
        for (int e = 0; e < 8; ++e) sum += v[i][e];
#pragma unroll
      for (int o = 16; o; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
      const float mean = sum / (float)H;
      float qs = 0.f;
#pragma unroll
      for (int i = 0; i < VM; ++i)
        if (lane + 32 * i < nvec)
#pragma unroll
          for (int e = 0; e < 8; ++e) {
            const float d = v[i][e] - mean;
            qs += d * d;
          }
#pragma unroll
      for (int o = 16; o; o >>= 1) qs += __shfl_xor_sync(0xffffffffu, qs, o);
      const float rstd = 1.0f / sqrtf(qs / (float)H + a.eps);
#pragma unroll
      for (int i = 0; i < VM; ++i) {
        const int k = lane + 32 * i;
        if (k >= nvec) continue;
        const uint32_t gw[4] = {gv[i].x, gv[i].y, gv[i].z, gv[i].w};
        const uint32_t bw[4] = {bv[i].x, bv[i].y, bv[i].z, bv[i].w};
        uint32_t hi[4], mi[4], lo[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          float y[2];
          y[0] = ok ? (v[i][2 * e] - mean) * rstd * bf_lo(gw[e]) + bf_lo(bw[e]) : 0.f;
          y[1] = ok ? (v[i][2 * e + 1] - mean) * rstd * bf_hi(gw[e]) + bf_hi(bw[e]) : 0.f;
          float h2[2], m2[2], l2[2];
#pragma unroll
          for (int u = 0; u < 2; ++u) {   // exact three-term bf16 split
            h2[u] = __bfloat162float(__float2bfloat16_rn(y[u]));
            const float r1 = y[u] - h2[u];
            m2[u] = __bfloat162float(__float2bfloat16_rn(r1));
            l2[u] = r1 - m2[u];
          }
          hi[e] = pack_bf16(h2[0], h2[1]);
          mi[e] = pack_bf16(m2[0], m2[1]);
          lo[e] = pack_bf16(l2[0], l2[1]);
        }
        reinterpret_cast<uint4 *>(sA + (0 * kVitRows + r) * P)[k] = make_uint4(hi[0], hi[1], hi[2], hi[3]);
        reinterpret_cast<uint4 *>(sA + (1 * kVitRows + r) * P)[k] = make_uint4(mi[0], mi[1], mi[2], mi[3]);
        reinterpret_cast<uint4 *>(sA + (2 * kVitRows + r) * P)[k] = make_uint4(lo[0], lo[1], lo[2], lo[3]);
      }
    }
  }
  __syncthreads();
  const unsigned long long tlLn = tl_now();

  // ---- classifier: warp w, classes 16w .. 16w + 15 (two n8 tiles), three
  // split products per k16 step, W_c fragments from the staged chunk (the
  // first version staged the whole 64-class slice, 99 KB, in 16-CTA clusters
  // that ran in three waves: ~60 us per VT launch; fragments straight from L2
  // were scattered 4-byte loads: 20-28 us)
  {
    float acc[2][4] = {};
    const __nv_bfloat16 *a0 = sA + gq * P + 2 * tq;
#pragma unroll 1
    for (int c = 0; c < nch; ++c) {
      if (c + 1 < nch) {
        stage_chunk(c + 1);
        asm volatile("cp.async.wait_group 1;" ::: "memory");
      } else {
        asm volatile("cp.async.wait_group 0;" ::: "memory");
      }
      __syncthreads();                              // chunk c landed for every thread
      const int kb = c * kVtcKC;
      const __nv_bfloat16 *bwc = sWc + (c & 1) * 128 * kVtcPW + (16 * wAll + gq) * kVtcPW + 2 * tq;
#pragma unroll
      for (int i = 0; i < kVtcKC / 16; ++i) {
        const int k = kb + 16 * i;
        if (k < H) {
          uint32_t bf[2][2];
#pragma unroll
          for (int nt = 0; nt < 2; ++nt) {
            bf[nt][0] = *reinterpret_cast<const uint32_t *>(bwc + nt * 8 * kVtcPW + 16 * i);
            bf[nt][1] = *reinterpret_cast<const uint32_t *>(bwc + nt * 8 * kVtcPW + 16 * i + 8);
          }
#pragma unroll
          for (int sp = 0; sp < 3; ++sp) {
            const __nv_bfloat16 *a_lo = a0 + sp * kVitRows * P + k;
            const __nv_bfloat16 *a_hi = a_lo + 8 * P;
            uint32_t af[4];
            af[0] = *reinterpret_cast<const uint32_t *>(a_lo);
            af[1] = *reinterpret_cast<const uint32_t *>(a_hi);
            af[2] = *reinterpret_cast<const uint32_t *>(a_lo + 8);
            af[3] = *reinterpret_cast<const uint32_t *>(a_hi + 8);
            mma_bf16_16816(acc[0], af, bf[0][0], bf[0][1]);
            mma_bf16_16816(acc[1], af, bf[1][0], bf[1][1]);
          }
        }
      }
      __syncthreads();                              // buffer c & 1 is restaged for chunk c + 2
    }
#pragma unroll
    for (int nt = 0; nt < 2; ++nt) {
      const int col = 16 * wAll + 8 * nt + 2 * tq;
      sZ[gq][col] = acc[nt][0];
      sZ[gq][col + 1] = acc[nt][1];
      sZ[gq + 8][col] = acc[nt][2];
      sZ[gq + 8][col + 1] = acc[nt][3];
    }
  }
  __syncthreads();
  const unsigned long long tlCls = tl_now();
  // threads t < 2 CB continue with 2 classes x 4 rows each
  const bool g0 = tAll < kThreads;
  float z[4][2];
#pragma unroll
  for (int rr = 0; rr < 4; ++rr) {
    z[rr][0] = (g0 ? sZ[rg * 4 + rr][2 * j] : 0.f) + bias0;
    z[rr][1] = (g0 ? sZ[rg * 4 + rr][2 * j + 1] : 0.f) + bias1;
  }

  // ---- per-row softmax statistics of this CTA's classes
#pragma unroll
  for (int rr = 0; rr < 4; ++rr) {
    SoftStat st{-INFINITY, 0.f, 0.f, -1};
    if (c0 < C) st = SoftStat{z[rr][0], 1.f, 0.f, c0};
    if (c1 < C) st = soft_merge(st, SoftStat{z[rr][1], 1.f, 0.f, c1});
#pragma unroll
    for (int o = 16; o; o >>= 1) st = soft_merge(st, soft_shfl_xor(st, o));
    if (lane == 0 && g0) sRed[warp][rr] = st;
  }
  __syncthreads();
  cluster_wait();                            // every CTA of the cluster is running
  if (g0 && t < kVitRows) {                  // row t: merge this CTA's warps, send to rank 0
    const int g = t / 4, rr = t % 4;
    SoftStat st = sRed[g * kWarpsPerRg][rr];
    for (int w = 1; w < kWarpsPerRg; ++w) st = soft_merge(st, sRed[g * kWarpsPerRg + w][rr]);
    const uint32_t dst = mapa_shared(smem_u32(&sQ[rank][t]), 0);
    st_cluster_f32(dst, st.m);
    st_cluster_f32(dst + 4, st.s);
    st_cluster_f32(dst + 8, st.u);
    asm volatile("st.shared::cluster.s32 [%0], %1;" ::"r"(dst + 12), "r"(st.idx) : "memory");
  }
  cluster_sync();

  // ---- rank 0 decides (rows t < 16 of warp 0)
  if (rank == 0 && warp == 0 && g0) {
    const int r = lane, b = b0 + r;
    bool exit_now = false;
    if (r < kVitRows && b < a.B) {
      if (!row_ok[r]) {
        if (a.init_alive) a.alive[b] = 0;
      } else {
        SoftStat st = sQ[0][r];
        for (int q = 1; q < CS; ++q) st = soft_merge(st, sQ[q][r]);
        float metric;
        bool pass;
        if (a.test == E3_TEST_PATIENCE) {
          pass = patience_step(a.ex.state, a.id[b], a.ex.capacity, st.idx, a.tau, &metric);
        } else if (a.test == E3_TEST_MAXPROB) {
          metric = 1.0f / st.s;
          pass = metric > a.tau;
        } else {
          metric = logf(st.s) - st.u / st.s;
          pass = metric < a.tau;
        }
        exit_now = pass || a.final_ramp;
        if (a.ex.ramp_metric && a.id[b] >= 0 && a.id[b] < a.ex.capacity)
          a.ex.ramp_metric[a.id[b] * a.ex.ramp_metric_stride + a.ramp_index] = metric;
        const int64_t id = a.id[b];
        if (exit_now && id >= 0 && id < a.ex.capacity) {
          if (a.ex.exit_layer) a.ex.exit_layer[id] = a.layer;
          if (a.ex.label) a.ex.label[id] = st.idx;
          if (a.ex.conf) a.ex.conf[id] = metric;
        }
        a.alive[b] = exit_now ? 0 : 1;
      }
    }
    if (r < kVitRows)                        // the decision to every CTA of the cluster (DSMEM)
      for (int q = 0; q < CS; ++q)
        asm volatile("st.shared::cluster.s32 [%0], %1;" ::"r"(mapa_shared(smem_u32(&sDec[r]), (uint32_t)q)),
                     "r"(exit_now ? 1 : 0)
                     : "memory");
    const int n_ex = __popc(__ballot_sync(0xffffffffu, exit_now));
    if (lane == 0 && n_ex) {
      if (a.ex.n_exit) atomicAdd(a.ex.n_exit, n_ex);
      if (a.ex.ramp_count) atomicAdd(a.ex.ramp_count + a.ramp_index, n_ex);
    }
  }
  cluster_sync();
  // ---- logits of the exiting rows: each CTA writes its class slice
  if (a.ex.logits && g0) {
#pragma unroll
    for (int rr = 0; rr < 4; ++rr) {
      const int r = rg * 4 + rr, b = b0 + r;
      if (b >= a.B) continue;
      if (!sDec[r]) continue;
      const int64_t id = a.id[b];
      if (id < 0 || id >= a.ex.capacity) continue;
      if (c0 < C) a.ex.logits[id * C + c0] = z[rr][0];
      if (c1 < C) a.ex.logits[id * C + c1] = z[rr][1];
    }
  }
  cluster_sync();                            // rank 0's smem stays valid until every CTA has read it
  if (kLate) pdl_trigger();
  if (tAll == 0) tl_rec(tlb, 9, tl0, tl1);
  if (tAll == 0) tl_rec(tlb, 91, tlLn, tlCls);   // phases: CLS LN done, classifier done, end
}



e3_status ramp_vit_run(const RampArgs &a, cudaStream_t st) {
  if (a.C < 1 || a.C > 16 * 128 || a.H % 64 || a.H > 3072 || !a.w.ln_g || !a.w.ln_b) {
    set_error("ViT ramp: need 1 <= C <= 2048, H % 64 == 0, H <= 3072 and ramp LayerNorm weights");
    return E3_EUNSUPPORTED;
  }
  const int CB = (a.C <= 16 * 64) ? 64 : 128;
  int CS = (a.C + CB - 1) / CB;
  const int smem = kVitRows * (a.H + 4) * 4;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(CS, (a.B + kVitRows - 1) / kVitRows);
  cfg.blockDim = dim3(kVitKQ * 2 * CB);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CS;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
#define E3_VRAMP(V, L)                                                                                      \
  do {                                                                                                      \
    static bool attr_done = false;                                                                          \
    if (!attr_done) {                                                                                       \
      E3_CUDA_TRY(cudaFuncSetAttribute(ramp_vit_kernel<V, L>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                       kVitRows * (3072 + 4) * 4));                                         \
      E3_CUDA_TRY(cudaFuncSetAttribute(ramp_vit_kernel<V, L>, cudaFuncAttributeNonPortableClusterSizeAllowed, \
                                       1));                                                                 \
      attr_done = true;                                                                                     \
    }                                                                                                       \
    E3_CUDA_TRY(cudaLaunchKernelEx(&cfg, ramp_vit_kernel<V, L>, a, CS));                                    \
  } while (0)
  static const bool early = getenv("E3_VIT_EARLY_TRIGGER") != nullptr;   // diagnostics
  if (a.C <= 8 * 128 && a.H <= 1024 && ramp_vit_tc_smem(a.H) <= 200 * 1024 && getenv("E3_VIT_RAMP_FMA") == nullptr) {
    CS = (a.C + 127) / 128;
    cfg.gridDim = dim3(CS, (a.B + kVitRows - 1) / kVitRows);
    attr[0].val.clusterDim.x = CS;
    cfg.blockDim = dim3(kVtcThreads);
    cfg.dynamicSmemBytes = ramp_vit_tc_smem(a.H);
    static bool tc_attr = false;
    if (!tc_attr) {
      for (auto k : {ramp_vit_tc_kernel<true>, ramp_vit_tc_kernel<false>}) {
        E3_CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
        E3_CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
      }
      tc_attr = true;
    }
    if (early) E3_CUDA_TRY(cudaLaunchKernelEx(&cfg, ramp_vit_tc_kernel<false>, a, CS));
    else E3_CUDA_TRY(cudaLaunchKernelEx(&cfg, ramp_vit_tc_kernel<true>, a, CS));
  } else if (CB == 64) {
    if (early) E3_VRAMP(64, false);
    else E3_VRAMP(64, true);
  } else {
    if (early) E3_VRAMP(128, false);
    else E3_VRAMP(128, true);
  }
#undef E3_VRAMP
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace

E3_TL_SETTER(tl_set_ramp)

e3_status ramp_run(const RampArgs &a, cudaStream_t st) {
  if (a.arch == E3_ARCH_VIT) return ramp_vit_run(a, st);
  if (a.arch != E3_ARCH_BERT) {
    set_error("ramp: arch not implemented");
    return E3_EUNSUPPORTED;
  }
  // r02: the cluster-free (group, slice) ramp of rampc.cu on request
  // (E3_RAMP_TICKET=1, or E3_FUSED_RC=1 whose fused last ramp shares its
  // arithmetic, so a ramp inside a split and at a split's end give identical
  // bits).  Not the default: in the BB pipeline it measured 2.2 % slower than
  // this cluster kernel on the same box (bench: 58.4k vs 59.7k inputs/s; the
  // graph-replayed single split of scripts/timeline.py had shown the reverse)
  if (ramp_ticket_mode() && ramp_bert2_supported(a.H, a.C) && a.done_ctr && a.pool_ws)
    return ramp_bert2_run(a, a.done_ctr, st);
  if (a.C < 1 || a.C > kMaxC || a.H % (8 * kCS) || a.H > 2048 || ramp_smem_bytes(a.H, a.C) > 220 * 1024) {
    set_error("ramp: need 1 <= C <= 16, H % 128 == 0 and H <= 2048");
    return E3_EUNSUPPORTED;
  }
  const int smem = ramp_smem_bytes(a.H, a.C);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(kCS, (a.B + kRows - 1) / kRows);
  cfg.blockDim = dim3(kRThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = kCS;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  const int vpl = (a.H / 8 + 31) / 32;
#define E3_RAMP(V)                                                                                          \
  do {                                                                                                      \
    static bool attr_done = false;                                                                          \
    if (!attr_done) {                                                                                       \
      E3_CUDA_TRY(cudaFuncSetAttribute(ramp_bert_kernel<V>, cudaFuncAttributeMaxDynamicSharedMemorySize,   \
                                       220 * 1024));                                                        \
      E3_CUDA_TRY(cudaFuncSetAttribute(ramp_bert_kernel<V>, cudaFuncAttributeNonPortableClusterSizeAllowed, \
                                       1));                                                                 \
      attr_done = true;                                                                                     \
    }                                                                                                       \
    E3_CUDA_TRY(cudaLaunchKernelEx(&cfg, ramp_bert_kernel<V>, a));                                          \
  } while (0)
  if (vpl <= 1) E3_RAMP(1);
  else if (vpl <= 3) E3_RAMP(3);
  else if (vpl <= 4) E3_RAMP(4);
  else E3_RAMP(8);
#undef E3_RAMP
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace e3
