// Row LayerNorm of the post-LN encoder layer:
// y = bf16((x - mean) / sqrt(var + eps) * g + b), fp32 statistics, biased
// variance, two passes over registers.  One warp per row, 16-byte loads; the
// row (H <= 4096 bf16) stays in registers.  HBM-bound: 2 * H * 2 bytes/row.
#include "common.cuh"
#include "kernels.h"
#include "prof.h"

namespace e3 {

namespace {

template <int VPL>   // 16-byte vectors per lane
__global__ void __launch_bounds__(256)
    layernorm_kernel(const __nv_bfloat16 *__restrict__ x, const __nv_bfloat16 *__restrict__ g,
                     const __nv_bfloat16 *__restrict__ bb, __nv_bfloat16 *__restrict__ y, int rows, int H,
                     float eps) {
  const int row = blockIdx.x * 8 + warp_id();
  if (row >= rows) return;
  const int lane = lane_id();
  const int nvec = H / 8;
  const uint4 *xr = reinterpret_cast<const uint4 *>(x + (size_t)row * H);
  uint4 v[VPL];
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int k = lane + 32 * i;
    if (k < nvec) {
      v[i] = __ldg(xr + k);
      const uint32_t w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
#pragma unroll
      for (int e = 0; e < 4; ++e) s += bf_lo(w[e]) + bf_hi(w[e]);
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  const float mean = s / (float)H;
  float q = 0.f;
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int k = lane + 32 * i;
    if (k < nvec) {
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
  uint4 *yr = reinterpret_cast<uint4 *>(y + (size_t)row * H);
  const uint4 *gp = reinterpret_cast<const uint4 *>(g);
  const uint4 *bp = reinterpret_cast<const uint4 *>(bb);
#pragma unroll
  for (int i = 0; i < VPL; ++i) {
    const int k = lane + 32 * i;
    if (k < nvec) {
      const uint4 g4 = __ldg(gp + k), b4 = __ldg(bp + k);
      const uint32_t w[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
      const uint32_t gw[4] = {g4.x, g4.y, g4.z, g4.w};
      const uint32_t bw[4] = {b4.x, b4.y, b4.z, b4.w};
      uint32_t o[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float a = (bf_lo(w[e]) - mean) * rstd * bf_lo(gw[e]) + bf_lo(bw[e]);
        const float c = (bf_hi(w[e]) - mean) * rstd * bf_hi(gw[e]) + bf_hi(bw[e]);
        o[e] = pack_bf16(a, c);
      }
      yr[k] = make_uint4(o[0], o[1], o[2], o[3]);
    }
  }
}

}  // namespace

e3_status layernorm_run(const void *x, const void *g, const void *b, void *y, int rows, int H, float eps,
                        cudaStream_t st) {
  const int grid = (rows + 7) / 8;
  auto *xp = reinterpret_cast<const __nv_bfloat16 *>(x);
  auto *gp = reinterpret_cast<const __nv_bfloat16 *>(g);
  auto *bp = reinterpret_cast<const __nv_bfloat16 *>(b);
  auto *yp = reinterpret_cast<__nv_bfloat16 *>(y);
  const int vpl = (H / 8 + 31) / 32;
  if (vpl <= 1) layernorm_kernel<1><<<grid, 256, 0, st>>>(xp, gp, bp, yp, rows, H, eps);
  else if (vpl <= 3) layernorm_kernel<3><<<grid, 256, 0, st>>>(xp, gp, bp, yp, rows, H, eps);
  else if (vpl <= 4) layernorm_kernel<4><<<grid, 256, 0, st>>>(xp, gp, bp, yp, rows, H, eps);
  else if (vpl <= 8) layernorm_kernel<8><<<grid, 256, 0, st>>>(xp, gp, bp, yp, rows, H, eps);
  else if (vpl <= 16) layernorm_kernel<16><<<grid, 256, 0, st>>>(xp, gp, bp, yp, rows, H, eps);
  else {
    set_error("LayerNorm: H > 4096 unsupported");
    return E3_EUNSUPPORTED;
  }
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace e3
