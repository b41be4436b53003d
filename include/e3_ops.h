/*
 * e3_ops.h — kernel-level entry points of the E3 split path (C ABI).
 *
 * These are the individual steps e3_split_run chains (SURVEY.md §8(a)
 * a2-a4), exported so that tests/ can check each kernel against the oracle
 * and profiles can time each one.  Same conventions as e3.h: status return,
 * e3_last_error(), stream as void*, ASYNC (no host sync), bf16 row-major
 * activations, weights in nn.Linear layout [out, in], caller-owned device
 * buffers.  Shape limits are checked before launch (E3_EUNSUPPORTED).
 */
#ifndef E3_OPS_H_
#define E3_OPS_H_

#include "e3.h"

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  E3_EPI_BIAS = 0,        /* C = bf16(A W^T + b)                        */
  E3_EPI_BIAS_GELU = 1,   /* C = bf16(GELU_erf(A W^T + b))              */
  E3_EPI_BIAS_RESID = 2   /* C = bf16(A W^T + b + R)                    */
} e3_epilogue;

/* Layer GEMM on tcgen05 tensor cores (a2): C[M,N] = epi(A[M,K] W[N,K]^T).
 * A row pitch lda (elements), C / R row pitch N.  K % 128 == 0, N % 64 == 0,
 * 16-byte aligned pointers.  fp32 accumulation in TMEM; one rounding to bf16. */
e3_status e3_op_gemm(void *stream, const void *A, int64_t lda, const void *W, const void *bias,
                     const void *resid, void *C, int32_t M, int32_t N, int32_t K, int32_t epilogue);

/* Decode-shaped GEMM of the LLaMA split (a8; gemm_dec.cu): Y[T,N] =
 * epi(X[T,K] W[N,K]^T), bf16 in, fp32 accumulate, bf16 out, T in {32, 64,
 * 128} tokens, K % 128 == 0.  epilogue: 0 plain, 1 + R[T,N] (residual),
 * 2 SwiGLU: Y[T,N] = SiLU(X W^T) * (X W2^T) with W = W_gate, W2 = W_up [N,K]
 * (N % 64 == 0).  Stream-K scratch is allocated on the stream per call. */
e3_status e3_op_dec_gemm(void *stream, const void *X, int32_t T, const void *W, const void *W2, int32_t N,
                         int32_t K, int32_t epilogue, const void *R, void *Y);

/* Attention output projection with the LayerNorm fused (a2; gemm_ln.cu):
 *   y   = bf16(A[M,K] W[N,K]^T + bias + R[M,N])     (written to pre if non-NULL)
 *   out = bf16(LN(y) * g + b), fp32 statistics of the rounded y, eps.
 * N in {128, 256, 384, 512, 640, 768, 1024} (a cluster of 2 CTAs holds a
 * whole row), K % 64 == 0, any M. */
e3_status e3_op_gemm_ln(void *stream, const void *A, const void *W, const void *bias, const void *R, const void *g,
                        const void *b, float eps, void *pre, void *out, int32_t M, int32_t N, int32_t K);

/* Self-attention (a2) on tcgen05: qkv [B*S, 3H] (q | k | v, head h owning
 * columns h*64..h*64+63 of each third) -> ctx [B*S, H].  head_dim 64,
 * S <= 256, no mask.  softmax(q k^T / sqrt(64)) v with the rounding contract
 * p_bf16 = bf16(exp(s - max)), ctx = bf16((p_bf16 v) / sum(exp(s - max))).
 * Work items are handed out through one device counter per GPU (allocated on
 * the first call): calls on one device must be ordered on one stream. */
e3_status e3_op_attention(void *stream, const void *qkv, void *ctx, int32_t B, int32_t S, int32_t H,
                          int32_t heads);

/* Row LayerNorm (a2): y = bf16(LN(x) * g + b), fp32 statistics, biased
 * variance.  x, y [rows, H]; H % 8 == 0, H <= 4096. */
e3_status e3_op_layernorm(void *stream, const void *x, const void *g, const void *b, void *y, int32_t rows,
                          int32_t H, float eps);

/* Fused exit ramp + threshold test (a3) for one ramp of a BERT/VIT model.
 *   x      [B,S,H] bf16 (CLS = token 0 of each row)
 *   alive  [B] uint8 device, in/out.  If init_alive, rows < n_valid are set
 *          alive first (n_valid from n_valid_dev, or B when NULL).
 *   A row that is alive and passes (or final != 0) is recorded in `ex` with
 *   exit layer `layer`, model ramp number `ramp_index`, and marked dead. */
e3_status e3_op_ramp(void *stream, int32_t arch, const void *x, const int64_t *id, int32_t B, int32_t S,
                     int32_t H, int32_t C, const e3_ramp_weights *rw, int32_t test, float tau, int32_t final,
                     int32_t layer, int32_t ramp_index, float norm_eps, uint8_t *alive, int32_t init_alive,
                     const int32_t *n_valid_dev, const e3_exits *ex);

/* Stable compaction (a4): survivors (alive[i] != 0) of x [B, row_bytes] and
 * id [B] gathered, in order, into x_out / id_out; *n_surv_dev = count.
 * row_bytes % 16 == 0. */
e3_status e3_op_compact(void *stream, const void *x, const int64_t *id, const uint8_t *alive, int32_t B,
                        int64_t row_bytes, void *x_out, int64_t *id_out, int32_t *n_surv_dev);

/* ---------------------------------------------------------- diagnostics --- */

/* Number of kernels this library has launched since load (all devices). */
long long e3_kernel_launches(void);

/* Per-kernel CUDA-event profiling.  When enabled, every kernel of the split
 * path is bracketed by an event pair on its own stream (small host cost);
 * e3_profile_read synchronises and returns, for kind k in
 * 0..8 (gemm_qkv, attention, gemm_o, layernorm, gemm_ffn1, gemm_ffn2, ramp,
 * compact, queue_copy): total ms, ALGORITHMIC flops and bytes (valid rows
 * only), launch count and name.  E3_EINVAL for k outside that range. */
e3_status e3_profile_enable(int32_t on);
e3_status e3_profile_reset(void);
e3_status e3_profile_read(int32_t kind, double *ms, double *flops, double *bytes, long long *launches,
                          const char **name);

/* Kernel timelines (diagnostics).  dev_buf: NULL (off, the default) or a
 * caller-owned device buffer of 148 x 16 x 6 + 296 x 8 x 6 uint64.  Every
 * later layer-GEMM launch fills the first part with globaltimer stamps (ns)
 * per CTA and per tile (<= 16 tiles): MMA start, last MMA commit, epilogue
 * warp 4 start / end, epilogue warp 11 start / end; every attention launch
 * fills the second part per CTA and item (<= 8): loads landed, S ready, P
 * ready, O ready, output stored.  Not thread-safe; E3_ECUDA if the symbol
 * copy fails. */
e3_status e3_debug_gemm_trace(void *dev_buf);

/* Diagnostics: kernel timeline of the encoder split path.  dev_buf = NULL
 * disables it; otherwise a zeroed device buffer of 1 + 4 * 32768 uint64:
 * buf[0] counts records, and thread 0 of every CTA of the layer GEMMs,
 * attention, LayerNorm, BERT ramp and fused LN + compaction kernels appends
 * {kernel id | blockIdx.x << 16, entry, released from griddepcontrol.wait,
 * end} globaltimer stamps (ns).  Kernel ids: 1000 + BN + epilogue (GEMM),
 * 2000 + key tile (+500 with the key mask; attention), 3 LayerNorm, 4 ramp
 * CTA, 5 ramp decision CTA, 6 compaction, 7 fused O + LayerNorm, 9 ViT ramp,
 * 8100 + epilogue decode GEMM; sub-phase records reuse the three stamps:
 * 40 ramp (CLS ready, partials stored, synced), 41 ramp decision (synced,
 * decided, recorded), 60 compaction scan done, 91 ViT ramp (LN done,
 * classifier done, end), 8000 + epilogue decode GEMM (first / last
 * accumulator ready, end), 8200 + epilogue stream-K tile reduction.  Not
 * thread-safe; E3_ECUDA if a symbol copy fails. */
e3_status e3_debug_timeline(void *dev_buf);

#ifdef __cplusplus
}
#endif
#endif /* E3_OPS_H_ */
