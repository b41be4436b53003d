// FP32 mode launchers (fp32_path.cu; E3_DTYPE_FP32).  Product code only.
#pragma once

#include "kernels.h"

namespace e3 {

// Y[M,N] = epi(A[M,K] W[N,K]^T + bias): A, R, Y fp32 row-major (R, Y leading
// dimension N); W, bias bf16; epi = E3_EPI_BIAS | _GELU | _RESID
e3_status f32_gemm_run(const float *A, int lda, const void *W, const void *bias, const float *R, float *Y, int M,
                       int N, int K, int epi, cudaStream_t st);
// ctx [B,S,H] from qkv [B,S,3H] (head_dim 64)
e3_status f32_attn_run(const float *qkv, float *ctx, int B, int S, int H, cudaStream_t st);
e3_status f32_ln_run(const float *x, const void *g, const void *b, float *y, int rows, int H, float eps,
                     cudaStream_t st);
// LLaMA decode pieces (DecArgs carries ids, n_valid, slots, positions, alive)
e3_status f32_rms_run(const float *x, const void *g, float *y, int rows, int H, float eps, cudaStream_t st);
e3_status f32_swiglu_run(const float *g, const float *u, float *a, size_t n, cudaStream_t st);
e3_status f32_rope_kv_run(const float *qkv, float *qo, float *kc, float *vc, const float2 *rope, const DecArgs &a,
                          cudaStream_t st);
e3_status f32_attn_dec_run(const float *q, float *ctx, const float *kc, const float *vc, const DecArgs &a,
                           cudaStream_t st);
// RampArgs with x = fp32 rows [B,S,H] (post-LN for BERT; the ViT ramp applies its own LN)
e3_status f32_ramp_run(const RampArgs &a, cudaStream_t st);

}  // namespace e3
