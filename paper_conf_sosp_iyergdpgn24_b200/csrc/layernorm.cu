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

// RPW rows per warp, all loads issued before any arithmetic: with one row per
// warp BB's 8192 rows needed 1024 CTAs, 1.7 waves of the 4 resident per SM
// (64 registers x 256 threads), and every second-wave CTA repeated the whole
// load latency (r01 timeline: 7.0 us for 25 MB).
template <int VPL, int RPW>
__global__ void __launch_bounds__(256)
    layernorm_kernel(const __nv_bfloat16 *__restrict__ x, const __nv_bfloat16 *__restrict__ g,
                     const __nv_bfloat16 *__restrict__ bb, __nv_bfloat16 *__restrict__ y, int rows, int H,
                     float eps) {
  const unsigned long long tl0 = tl_now();
  unsigned long long *const tlb = g_tl;
  const int lane = lane_id();
  const int warps = gridDim.x * 8;
  const int row0 = blockIdx.x * 8 + warp_id();
  uint4 v[RPW][VPL];
  LnParams<VPL> p;
  ln_load_params<VPL>(p, g, bb, H, lane);   // weights: before the dependency wait
  pdl_wait();
  pdl_trigger();
  const unsigned long long tl1 = tl_now();
  // persistent: the grid is at most one wave; each warp walks its rows RPW at
  // a time (loads of a batch first).  RPW == 1: the next row's loads are
  // issued before the current row is normalised (VT, H = 768: 3.37 -> 4.16
  // TB/s, VT 37.7 -> 38.2 k inputs/s; at H = 1024 two rows per warp without
  // the prefetch stay ahead: 3.36 vs 3.22 TB/s)
  const int stride = RPW * warps;
  if (RPW == 1) {
    uint4 w[VPL];
    int base = row0;
    if (base < rows) ln_load_row<VPL>(v[0], x + (size_t)base * H, H, lane);
    while (base < rows) {
      const int nb = base + stride;
      if (nb < rows) ln_load_row<VPL>(w, x + (size_t)nb * H, H, lane);
      ln_apply<VPL>(v[0], p, H, eps, lane);
      ln_store_row<VPL>(v[0], y + (size_t)base * H, H, lane);
#pragma unroll
      for (int i = 0; i < VPL; ++i) v[0][i] = w[i];
      base = nb;
    }
  } else {
    for (int base = row0; base < rows; base += stride) {
#pragma unroll
      for (int j = 0; j < RPW; ++j) {
        const int row = base + j * warps;
        if (row < rows) ln_load_row<VPL>(v[j], x + (size_t)row * H, H, lane);
      }
#pragma unroll
      for (int j = 0; j < RPW; ++j) {
        const int row = base + j * warps;
        if (row < rows) {
          ln_apply<VPL>(v[j], p, H, eps, lane);
          ln_store_row<VPL>(v[j], y + (size_t)row * H, H, lane);
        }
      }
    }
  }
  if (threadIdx.x == 0) tl_rec(tlb, 3, tl0, tl1);
}

}  // namespace

E3_TL_SETTER(tl_set_ln)

e3_status layernorm_run(const void *x, const void *g, const void *b, void *y, int rows, int H, float eps,
                        cudaStream_t st) {
  // rows per warp: 2 when one row per warp would exceed one wave of resident
  // CTAs; the grid is capped at one wave and the warps walk the rest
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    E3_CUDA_TRY(cudaGetDevice(&dev));
    E3_CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  }
  const int vpl = (H / 8 + 31) / 32;
  if (vpl > 16) {
    set_error("LayerNorm: H > 4096 unsupported");
    return E3_EUNSUPPORTED;
  }
  // rows per warp: 1 with the next row prefetched up to H = 768, else 2
  // when one row per warp would exceed one wave of resident CTAs
  const bool two = rows > 8 * 4 * sms && H <= 1024 && H > 768;   // registers: 2 rows of <= 4 vectors per lane
  using Kern = void (*)(const __nv_bfloat16 *, const __nv_bfloat16 *, const __nv_bfloat16 *, __nv_bfloat16 *, int,
                        int, float);
  const int vi = vpl <= 1 ? 0 : vpl <= 3 ? 1 : vpl <= 4 ? 2 : vpl <= 8 ? 3 : 4;
  static const Kern kerns[5][2] = {{layernorm_kernel<1, 1>, layernorm_kernel<1, 2>},
                                   {layernorm_kernel<3, 1>, layernorm_kernel<3, 2>},
                                   {layernorm_kernel<4, 1>, layernorm_kernel<4, 2>},
                                   {layernorm_kernel<8, 1>, layernorm_kernel<8, 2>},
                                   {layernorm_kernel<16, 1>, layernorm_kernel<16, 2>}};
  static int occ[5][2] = {};
  const Kern kern = kerns[vi][two ? 1 : 0];
  int &o = occ[vi][two ? 1 : 0];
  if (!o) E3_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, kern, 256, 0));
  if (o < 1) o = 1;
  int grid = two ? (rows + 15) / 16 : (rows + 7) / 8;
  if (grid > o * sms) grid = o * sms;
  E3_CUDA_TRY(launch_k(kern, dim3(grid), dim3(256), 0, st, reinterpret_cast<const __nv_bfloat16 *>(x),
                       reinterpret_cast<const __nv_bfloat16 *>(g), reinterpret_cast<const __nv_bfloat16 *>(b),
                       reinterpret_cast<__nv_bfloat16 *>(y), rows, H, eps));
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

}  // namespace e3
