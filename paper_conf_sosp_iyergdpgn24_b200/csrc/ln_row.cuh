// Warp-per-row LayerNorm core shared by every kernel that normalises a row
// (layernorm.cu, the ramp's CLS rows, the fused LN2 + compaction).  One
// implementation, one lane mapping and one reduction order, so a row
// normalised in two kernels gives bit-identical bf16 results.
//
// y = bf16((x - mean) * rsqrt(var + eps) * g + b), fp32 statistics, biased
// variance (two passes over registers).  Lane l owns the 16-byte vectors
// l, l+32, ... of the row (H % 8 == 0, H <= 256 * VPL).
#pragma once

#include "common.cuh"

namespace e3 {

template <int VPL>
struct LnParams {
  uint4 g[VPL], b[VPL];
};

template <int VPL>
__device__ __forceinline__ void ln_load_params(LnParams<VPL> &p, const __nv_bfloat16 *g, const __nv_bfloat16 *b,
                                               int H, int lane) {
  const uint4 *gp = reinterpret_cast<const uint4 *>(g);
  const uint4 *bp = reinterpret_cast<const uint4 *>(b);
  const int nvec = H / 8;
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int k = lane + 32 * i;
    p.g[i] = (k < nvec) ? __ldg(gp + k) : make_uint4(0, 0, 0, 0);
    p.b[i] = (k < nvec) ? __ldg(bp + k) : make_uint4(0, 0, 0, 0);
  }
}

template <int VPL>
__device__ __forceinline__ void ln_load_row(uint4 (&v)[VPL], const __nv_bfloat16 *x, int H, int lane) {
  const uint4 *xr = reinterpret_cast<const uint4 *>(x);
  const int nvec = H / 8;
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int k = lane + 32 * i;
    v[i] = (k < nvec) ? xr[k] : make_uint4(0, 0, 0, 0);
  }
}

// normalise the row held in v (in place, bf16-packed)
template <int VPL>
__device__ __forceinline__ void ln_apply(uint4 (&v)[VPL], const LnParams<VPL> &p, int H, float eps, int lane) {
  const int nvec = H / 8;
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const uint32_t w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
#pragma unroll
    for (int e = 0; e < 4; ++e) s += bf_lo(w[e]) + bf_hi(w[e]);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  const float mean = s / (float)H;
  float q = 0.f;
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    if (lane + 32 * i < nvec) {
      const uint32_t w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float a = bf_lo(w[e]) - mean, c = bf_hi(w[e]) - mean;
        q += a * a + c * c;
      }
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
  const float rstd = 1.0f / sqrtf(q / (float)H + eps);
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const uint32_t w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
    const uint32_t gw[4] = {p.g[i].x, p.g[i].y, p.g[i].z, p.g[i].w};
    const uint32_t bw[4] = {p.b[i].x, p.b[i].y, p.b[i].z, p.b[i].w};
    uint32_t o[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const float a = (bf_lo(w[e]) - mean) * rstd * bf_lo(gw[e]) + bf_lo(bw[e]);
      const float c = (bf_hi(w[e]) - mean) * rstd * bf_hi(gw[e]) + bf_hi(bw[e]);
      o[e] = pack_bf16(a, c);
    }
    v[i] = make_uint4(o[0], o[1], o[2], o[3]);
  }
}

template <int VPL>
__device__ __forceinline__ void ln_store_row(const uint4 (&v)[VPL], __nv_bfloat16 *y, int H, int lane) {
  uint4 *yr = reinterpret_cast<uint4 *>(y);
  const int nvec = H / 8;
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int k = lane + 32 * i;
    if (k < nvec) yr[k] = v[i];
  }
}

}  // namespace e3
