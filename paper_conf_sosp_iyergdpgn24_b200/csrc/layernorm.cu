// Row LayerNorm of the post-LN encoder layer:
// y = bf16((x - mean) / sqrt(var + eps) * g + b), fp32 statistics, biased
// variance, two passes over registers (ln_row.cuh).  One warp per row, 16-byte
// loads, the row and gamma/beta loaded together (one memory round trip).
// HBM/L2-bound: 2 * H * 2 bytes per row.
#include "common.cuh"
#include "kernels.h"
#include "ln_row.cuh"
#include "prof.h"

namespace e3 {

namespace {

template <int VPL>   // 16-byte vectors per lane
__global__ void __launch_bounds__(256)
    layernorm_kernel(const __nv_bfloat16 *__restrict__ x, const __nv_bfloat16 *__restrict__ g,
                     const __nv_bfloat16 *__restrict__ bb, __nv_bfloat16 *__restrict__ y, int rows, int H,
                     float eps) {
  const int row = blockIdx.x * 8 + warp_id();
  const int lane = lane_id();
  uint4 v[VPL];
  LnParams<VPL> p;
  ln_load_params<VPL>(p, g, bb, H, lane);   // weights: before the dependency wait
  pdl_wait();
  pdl_trigger();
  if (row >= rows) return;
  ln_load_row<VPL>(v, x + (size_t)row * H, H, lane);
  ln_apply<VPL>(v, p, H, eps, lane);
  ln_store_row<VPL>(v, y + (size_t)row * H, H, lane);
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
  if (vpl <= 1) E3_CUDA_TRY(launch_k(layernorm_kernel<1>, dim3(grid), dim3(256), 0, st, xp, gp, bp, yp, rows, H, eps));
  else if (vpl <= 3) E3_CUDA_TRY(launch_k(layernorm_kernel<3>, dim3(grid), dim3(256), 0, st, xp, gp, bp, yp, rows, H, eps));
  else if (vpl <= 4) E3_CUDA_TRY(launch_k(layernorm_kernel<4>, dim3(grid), dim3(256), 0, st, xp, gp, bp, yp, rows, H, eps));
  else if (vpl <= 8) E3_CUDA_TRY(launch_k(layernorm_kernel<8>, dim3(grid), dim3(256), 0, st, xp, gp, bp, yp, rows, H, eps));
  else if (vpl <= 16) E3_CUDA_TRY(launch_k(layernorm_kernel<16>, dim3(grid), dim3(256), 0, st, xp, gp, bp, yp, rows, H, eps));
  else {
    set_error("LayerNorm: H > 4096 unsupported");
    return E3_EUNSUPPORTED;
  }
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace e3
