// Internal launchers of the split path (host side).  Product code only.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/e3.h"
#include "../../include/e3_ops.h"

namespace e3 {

// ---- K1 layer GEMM (gemm_tc.cu)
struct GemmMaps {
  CUtensorMap a;   // A [M,K], box 128 (64 when A is multicast) x 64, 128-B swizzle
  CUtensorMap b;   // W [N,K], box BN/2 (/2 again when W is multicast) x 64, 128-B swizzle
  CUtensorMap c;   // C [M,N], box 32 x 32, 64-B swizzle (epilogue TMA store)
  int bn;          // tile code: N tile | multicast mode << 12 (gemm_pick_bn)
};
// Multicast modes of the layer GEMM (a cluster of two CTA pairs):
//   GEMM_MC_NONE  one pair per cluster
//   GEMM_MC_A     the pairs own N-neighbour tiles of one M block: each A box is
//                 loaded half by each pair and multicast to both
//   GEMM_MC_B     the pairs own M-neighbour tiles of one N block: W multicast
enum { GEMM_MC_NONE = 0, GEMM_MC_A = 1, GEMM_MC_B = 2 };
// returns a tile code (N tile | mode << 12) for gemm_tmaps / gemm_run
int gemm_pick_bn(int M, int N, int K, int sms, int epi);
e3_status gemm_set_trace(void *buf);   // diagnostics (e3_debug_gemm_trace)
e3_status attn_set_trace(void *buf);   // diagnostics (e3_debug_gemm_trace)
// diagnostics (e3_debug_timeline): per translation unit
e3_status tl_set_gemm(void *buf);
e3_status tl_set_attn(void *buf);
e3_status tl_set_ln(void *buf);
e3_status tl_set_ramp(void *buf);
e3_status tl_set_compact(void *buf);
e3_status tl_set_gemm_ln(void *buf);
e3_status tl_set_dec(void *buf);
e3_status tl_set_llama(void *buf);
e3_status gemm_tmaps(GemmMaps *g, const void *A, int64_t lda, const void *W, const void *C, int M, int N, int K,
                     int bn);
e3_status gemm_run(const GemmMaps &g, const void *bias, const void *R, int M, int N, int K, int epi, int sms,
                   cudaStream_t st);

// ---- K1b projection + bias + residual + LayerNorm (gemm_ln.cu): cluster of
// 2 CTAs per 128 rows, each owning N/2 columns; pre (optional) receives
// y = bf16(A W^T + bias + R), out = bf16(LN(y) * g + b)
struct LnGemmMaps {
  CUtensorMap a, w, w2, r, pre, out;   // w2: W boxes of the CTA-pair variant (half the MMA N)
};
struct LnGemmArgs {
  const __nv_bfloat16 *bias, *R, *g, *b;
  float eps;
  int M, N, K;
  int store_pre;
};
bool ln_gemm_supported(int N, int K);
e3_status ln_gemm_tmaps(LnGemmMaps *m, const void *A, const void *W, const void *R, const void *pre, const void *out,
                        int M, int N, int K);
e3_status ln_gemm_run(const LnGemmMaps &m, const LnGemmArgs &a, cudaStream_t st);

// ---- K2 attention (attn_tc.cu)
struct AttnMaps {
  CUtensorMap q;    // qkv [B][S][3H], box 64 x 128 x 1
  CUtensorMap kv;   // qkv [B][S][3H], box 64 x SKV x 1
  CUtensorMap ctx;  // ctx [B][S][H],  box 64 x 128 x 1 (TMA store)
  int skv;
};
e3_status attn_tmaps(AttnMaps *m, const void *qkv, const void *ctx, int B, int S, int H);
// ctr: four device words, zero before the first launch (the kernel leaves
// them zero): two (item counter, CTA exit count) pairs, used alternately by
// consecutive launches (*parity flips per call), so a launch never takes
// items from the pair its still-running predecessor uses
e3_status attn_run(const AttnMaps &m, int B, int S, int H, int heads, unsigned *ctr, int *parity, cudaStream_t st);

// ---- K3 LayerNorm (layernorm.cu)
e3_status layernorm_run(const void *x, const void *g, const void *b, void *y, int rows, int H, float eps,
                        cudaStream_t st);

// ---- K4 exit ramp (ramp.cu)
constexpr int kRampRowsPerCta = 16;   // rows per ramp row group (one ticket each)
// workspace counter words: [0] compaction ticket, [1 .. 256] ramp group
// tickets, then the fused ramp + compaction's decision and exit counters
constexpr int kRampCtrGroupsDone = 1 + 4096 / kRampRowsPerCta;
constexpr int kRampCtrExit = kRampCtrGroupsDone + 1;
constexpr int kAttnCtr = kRampCtrExit + 1;   // [2][2]: attention item counter, CTA exits (two pairs)
constexpr int kCtrWordsAll = kAttnCtr + 4;
struct RampArgs {
  int arch;
  const void *x;            // [B,S,H] bf16 (pre-LN rows when ln_g != NULL)
  const void *ln_g, *ln_b;  // optional LayerNorm applied to the CLS rows first
  const int64_t *id;        // [B]
  int B, S, H, C;
  e3_ramp_weights w;
  int test;
  float tau;
  int final_ramp;
  int layer, ramp_index;
  float eps;
  uint8_t *alive;           // [B]
  int init_alive;
  const int32_t *n_valid_dev;   // NULL: n_valid_host
  int n_valid_host;
  e3_exits ex;
  float *pool_ws;           // [B,H] fp32 workspace (BERT: the slices' partial logits)
  unsigned *done_ctr;       // device counters [kCtrWordsAll] (zero between launches)
  // LLAMA: per-128-class-tile softmax statistics from the LM-head GEMM
  // (gemm_dec.cu, E3_DEC_LOGITS, which also wrote the logits to the exit
  // records); the decide kernel merges them
  const float4 *lm_stats;   // [tiles][B] (max, sum e, sum e*(z-max), argmax bits)
  int lm_tiles;
};
e3_status ramp_run(const RampArgs &a, cudaStream_t st);
// BERT ramp on (group, slice) CTAs without clusters (rampc.cu); ctr_words =
// the workspace counters (RampArgs.done_ctr)
bool ramp_bert2_supported(int H, int C);
bool ramp_ticket_mode();   // E3_RAMP_TICKET / E3_FUSED_RC: the ticketed ramp for every BERT ramp
e3_status ramp_bert2_run(const RampArgs &a, unsigned *ctr_words, cudaStream_t st);
// the split's last BERT ramp (pre-LN rows, a.ln_g set) fused with the stable
// LN + compaction of the survivors into dst; *done = false when the shape
// does not fit one cooperative wave (the caller then runs ramp + ln_compact)
e3_status ramp_compact_run(const RampArgs &a, unsigned *ctr_words, const struct RingDst &dst, int32_t *n_surv_dev,
                           int sms, cudaStream_t st, bool *done);
e3_status tl_set_rampc(void *buf);

// ---- K7 decode GEMM (gemm_dec.cu): Y[T,N] = epi(X[T,K] W[N,K]^T), swap-AB tcgen05
// PARTIAL: split-K by 4 (CSK) without a cluster; each CTA writes its fp32
// partial tile to part_out[k][t][n] and the reduction (+ residual, + the
// following RMSNorm) is done by reduce_rmsnorm_run
enum { E3_DEC_STORE = 0, E3_DEC_RESID = 1, E3_DEC_SWIGLU = 2, E3_DEC_QKV_ROPE = 3, E3_DEC_LOGITS = 4, E3_DEC_PARTIAL = 5 };
struct DecMaps {
  CUtensorMap w;    // W [N,K], box 128 (SWIGLU: 64) x 64, 128-B swizzle
  CUtensorMap w2;   // SWIGLU: W_up, same box
  CUtensorMap x;    // X [T,K], box T x 64
};
struct DecArgs {
  int T, N, K, epi;
  int max_contrib;          // partial slots per tile (dec_max_contrib)
  const __nv_bfloat16 *R;   // RESID: residual [T, ldo]
  __nv_bfloat16 *Y;         // STORE / RESID / SWIGLU / QKV (q): [T, ldo]
  int ldo;
  float *Z;                 // LOGITS: exit-record logits [id_cap, N] (NULL: not recorded)
  const uint8_t *alive;     // LOGITS: rows alive at this ramp (unless init_alive)
  int init_alive;
  float4 *stats;            // LOGITS: [tiles][T]
  float *part;              // stream-K partials [tiles][max_contrib][T/4][128 rows] of float4
  unsigned *tickets;        // stream-K tickets [tiles], zero between launches
  // QKV_ROPE: this layer's cache and the tokens' slots / positions
  int nh, kvh, max_ctx;
  __nv_bfloat16 *kc, *vc;
  const float2 *rope;       // [max_ctx][64] (cos, sin) of exact angles
  const int64_t *ids;
  const int32_t *n_valid_dev;
  int n_valid_host;
  const int32_t *slot_of_id;
  int64_t id_cap;
  const int32_t *pos_of_slot;
  int n_slots;              // QKV_ROPE: slots of the cache; slot / pos outside it -> *err, row skipped
  int *err;                 // device error flag (E3_EINVAL reported by the pipeline), may be NULL
  int late_trigger;         // PDL trigger at the end instead of after the dependency wait
  float *part_out;          // PARTIAL: [4][T][N] fp32 split-K partials
};
int dec_tiles(int N, int epi);
int dec_max_contrib(int N, int K, int epi, int sms);
e3_status dec_tmaps(DecMaps *m, const void *X, int T, int K, const void *W, const void *W2, int N, int epi);
e3_status dec_run(const DecMaps &m, const DecArgs &a, int sms, cudaStream_t st);
e3_status rope_table(int max_ctx, int head_dim, double theta, float2 **out);

// ---- K8 LLaMA decode helpers (llama.cu)
e3_status rmsnorm_run(const void *x, const void *g, void *y, int rows, int H, float eps, cudaStream_t st);
// h = bf16((((0 + p0) + p1) + p2) + p3 + resid) from 4 split-K partials
// [4][rows][H] (the cluster split-K's rank-order sum + RESID epilogue, bit for
// bit), stored to h_out; then y = RMSNorm(h) * g exactly as rmsnorm_run
// (g == nullptr: no norm)
e3_status reduce_rmsnorm_run(const float *part, const void *resid, void *h_out, const void *g, void *y, int rows,
                             int H, float eps, cudaStream_t st);
// the split-K-by-4 partial mode is available for this GEMM shape (else RESID + rmsnorm_run)
bool dec_partial_ok(int N, int K, int sms);
// ctx[t, h*128 + :] = softmax(q_t,h . K[slot, g(h), 0..pos]^T / sqrt 128) V[...]
e3_status attn_dec_run(const void *q, void *ctx, const void *kc, const void *vc, const int64_t *ids,
                       const int32_t *n_valid_dev, int n_valid_host, const int32_t *slot_of_id, int64_t id_cap,
                       const int32_t *pos_of_slot, int n_slots, int T, int nh, int kvh, int max_ctx,
                       cudaStream_t st);
// merge the LM-head statistics, threshold test, exit records (RampArgs with lm_*);
// a.x (the rows) is copied into ex.hidden for the exiting tokens when both are set
e3_status lm_decide_run(const RampArgs &a, cudaStream_t st);
// multi-step decode helpers (llama.cu; e3_decode_run)
e3_status fill_prep_run(const int64_t *ids, int nv, int B, const void *hidden, int64_t cap, const int32_t *exit_layer,
                        int layer, int64_t row_bytes, void *x, int64_t *ids_out, uint8_t *mask, cudaStream_t st);
e3_status decode_advance_run(const int64_t *ids, int64_t n, const int32_t *label, int64_t cap, int32_t *tokens_out,
                             const void *embed, int32_t vocab, int64_t row_bytes, void *x, const int32_t *slot_of_id,
                             int32_t *pos_of_slot, int n_slots, int *err, cudaStream_t st);

// ---- K5 compaction (compact.cu)
struct RingDst {
  uint8_t *rows;            // [cap, row_bytes]
  int64_t *ids;             // [cap]
  int64_t cap;
  int64_t *tail_dev;        // current tail (read); NULL: contiguous output at row 0
  int64_t *tail_out;        // next tail slot (written by ln_compact; NULL: none)
  int64_t head;             // host-known head (rows) at launch
  int *overflow_dev;        // may be NULL
  volatile int *mailbox;    // host-mapped slot for n_surv (may be NULL)
};
e3_status compact_run(const void *x, const int64_t *id, const uint8_t *alive, int B, int64_t row_bytes,
                      const RingDst &dst, int32_t *n_surv_dev, unsigned *done_ctr, int sms, cudaStream_t st);

// fused LN2 + compaction: survivors of the PRE-LN rows y [B,S,H] are
// LayerNorm-ed (g, b, eps) and written to dst; g == NULL: copied unchanged
// (pre-LN ViT, whose layer output needs no normalisation)
e3_status ln_compact_run(const void *y, const int64_t *id, const uint8_t *alive, int B, int S, int H, const void *g,
                         const void *b, float eps, const RingDst &dst, int32_t *n_surv_dev, int sms,
                         cudaStream_t st);

// ---- K6 queue pop (compact.cu): rows [head, head+n) of a ring -> contiguous
// dst, zero-padding rows n..B-1 (ids -1).
e3_status ring_pop_copy(const uint8_t *ring, const int64_t *ring_ids, int64_t cap, int64_t head, int n, int B,
                        int64_t row_bytes, void *dst, int64_t *dst_ids, int sms, cudaStream_t st);
// device-count push (e3_queue_push): rows [0, *n_dev) appended at *tail_dev
e3_status ring_push_copy(const void *rows, const int64_t *ids, const int32_t *n_dev, int max_rows, uint8_t *ring,
                         int64_t *ring_ids, int64_t cap, int64_t *tail_dev, const int64_t *head_dev,
                         int *overflow_dev, int64_t row_bytes, cudaStream_t st);
e3_status fill_valid(int32_t *dst, int value, cudaStream_t st);

}  // namespace e3
