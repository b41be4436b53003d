// Shared device helpers for the E3 split path on sm_100a: bf16 conversion,
// mbarrier / TMA / tcgen05 PTX wrappers, error plumbing.
// Product code only: nothing here is shared with oracle/ (DESIGN.md "Boundary").
#pragma once

#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include <string>

#include "../../include/e3.h"

namespace e3 {

// ----------------------------------------------------------------- errors --
void set_error(const std::string &msg);
e3_status cuda_fail(cudaError_t e, const char *what);

#define E3_CUDA_TRY(expr)                                      \
  do {                                                         \
    cudaError_t _e = (expr);                                   \
    if (_e != cudaSuccess) return ::e3::cuda_fail(_e, #expr);  \
  } while (0)

#define E3_CHECK_ARG(cond, msg)                                \
  do {                                                         \
    if (!(cond)) {                                             \
      ::e3::set_error(std::string("invalid argument: ") + msg); \
      return E3_EINVAL;                                        \
    }                                                          \
  } while (0)

// Resolve cuTensorMapEncodeTiled through the runtime (no libcuda link).
typedef CUresult (*PFN_encodeTiled)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                    const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                    const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                    CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
PFN_encodeTiled encode_tiled_fn();

// 2-D bf16 tensor map: rows x cols (cols contiguous), row pitch in elements,
// box = box_rows x box_cols, 128-byte swizzle (box_cols * 2 == 128).
e3_status make_tmap_2d(CUtensorMap *m, const void *base, uint64_t rows, uint64_t cols,
                       uint64_t row_pitch_elems, uint32_t box_rows, uint32_t box_cols);
// same with 64-byte swizzle (box_cols * 2 == 64): GEMM epilogue store / residual tiles
e3_status make_tmap_2d_sw64(CUtensorMap *m, const void *base, uint64_t rows, uint64_t cols,
                            uint64_t row_pitch_elems, uint32_t box_rows, uint32_t box_cols);
// 3-D bf16 tensor map [d2][d1][d0] (d0 contiguous) with pitches in elements.
e3_status make_tmap_3d(CUtensorMap *m, const void *base, uint64_t d0, uint64_t d1, uint64_t d2,
                       uint64_t pitch1, uint64_t pitch2, uint32_t b0, uint32_t b1, uint32_t b2);

int num_sms(int device);

// Programmatic dependent launch: every kernel of the split path is launched
// with cudaLaunchAttributeProgrammaticStreamSerialization so its prologue
// (barrier init, TMEM alloc, descriptor prefetch, weight loads) overlaps the
// tail of the previous kernel; each kernel calls pdl_wait() before it touches
// anything a previous kernel wrote (or reads).  E3_NO_PDL=1 disables it.
bool pdl_enabled();
template <typename... KArgs, typename... Args>
cudaError_t launch_k(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                     Args &&...args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

// ------------------------------------------------------------ device side --
#ifdef __CUDACC__

__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ float bf2f(__nv_bfloat16 v) { return __bfloat162float(v); }
__device__ __forceinline__ float bf_lo(uint32_t w) { return __uint_as_float(w << 16); }
__device__ __forceinline__ float bf_hi(uint32_t w) { return __uint_as_float(w & 0xFFFF0000u); }
__device__ __forceinline__ uint32_t pack_bf16(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);  // .x = a (low), .y = b (high)
  return *reinterpret_cast<uint32_t *>(&h);
}

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ---- mbarrier
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  uint32_t addr = smem_u32(bar);
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@!P1 bra WAIT_%=;\n\t}" ::"r"(addr),
      "r"(parity)
      : "memory");
}

// ---- TMA
__device__ __forceinline__ void tma_prefetch(const CUtensorMap *m) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(m)) : "memory");
}
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *m, uint64_t *bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(m)), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}
// TMA store smem -> global (bulk async-group of the issuing thread)
__device__ __forceinline__ void tma_store_2d(const CUtensorMap *m, const void *src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(m)),
               "r"(smem_u32(src)), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void tma_store_3d(const CUtensorMap *m, const void *src, int c0, int c1, int c2) {
  asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(m)),
               "r"(smem_u32(src)), "r"(c0), "r"(c1), "r"(c2)
               : "memory");
}
__device__ __forceinline__ float ex2_approx(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait() {
  asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void tma_load_3d(void *dst, const CUtensorMap *m, uint64_t *bar, int c0, int c1,
                                            int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], "
      "[%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(m)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}

// ---- tcgen05 / TMEM
__device__ __forceinline__ void tmem_alloc(uint32_t *dst_smem, uint32_t ncols) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(dst_smem)),
               "r"(ncols)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr, uint32_t ncols) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_commit(uint64_t *bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}
// D[tmem] (+)= A[smem] * B[smem], kind::f16 (bf16 in, fp32 accumulate)
__device__ __forceinline__ void tc_mma_f16(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                                           uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
// D (+)= A * B with A (M x 16, 16-bit elements, two per 32-bit column) in
// tensor memory at a_tmem and B from a shared-memory descriptor
__device__ __forceinline__ void tc_mma_f16_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                                              uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
      "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// 32 lanes x 32b, 16 consecutive columns <- 16 registers per thread
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15, %16};" ::"r"(taddr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]), "r"(v[9]),
      "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
      : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// 32 lanes x 32b, 32 consecutive columns -> 32 registers per thread.
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
        "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
        "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr)
      : "memory");
}

// UMMA shared-memory descriptor (sm_100 "version 1"), 128-byte swizzle.
//   bits  0-13 start >> 4 | 16-29 LBO >> 4 | 32-45 SBO >> 4 | 46-47 version=1
//   bits 49-51 base offset (0: atoms 1024-B aligned) | 61-63 layout (2 = SWIZZLE_128B)
__device__ __forceinline__ uint64_t smem_desc_sw128(uint32_t saddr, uint32_t lbo_bytes, uint32_t sbo_bytes) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo_bytes >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo_bytes >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}

// Instruction descriptor, kind::f16: bf16 A/B, fp32 D, dense.
//   bits 4-5 D fmt (1=f32) | 7-9 A fmt (1=bf16) | 10-12 B fmt (1=bf16)
//   bit 15 A major (0=K) | bit 16 B major (0=K, 1=MN) | 17-22 N>>3 | 24-28 M>>4
__host__ __device__ constexpr uint32_t idesc_bf16_f32(int M, int N, int b_mn_major) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)b_mn_major << 16) | ((uint32_t)(N >> 3) << 17) |
         ((uint32_t)(M >> 4) << 24);
}

// ---- clusters / CTA pairs (cta_group::2)
__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// shared::cta address -> shared::cluster address of the same offset in CTA `rank`
__device__ __forceinline__ uint32_t mapa_shared(uint32_t saddr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
// 2-SM TMA: data lands in this CTA's smem, completion bytes go to the mbarrier
// at `mbar_cluster` (the leader CTA's barrier)
__device__ __forceinline__ void tma_load_2d_2sm(void *dst, const CUtensorMap *m, uint32_t mbar_cluster, int c0,
                                                int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, "
      "%4}], [%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(m)), "r"(mbar_cluster), "r"(c0), "r"(c1)
      : "memory");
}
// 2-SM TMA multicast: the box lands at the same smem offset in every CTA of
// cta_mask; each destination's completion bytes go to the barrier at this
// offset in the LEADER of the destination's pair (peer bit of the address
// cleared, as the sm_100 2-SM multicast form requires)
__device__ __forceinline__ void tma_load_2d_2sm_mc(void *dst, const CUtensorMap *m, uint32_t mbar_local, int c0,
                                                   int c1, uint16_t cta_mask) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster"
      " [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(m)), "r"(mbar_local & 0xFEFFFFFFu), "r"(c0), "r"(c1), "h"(cta_mask)
      : "memory");
}
__device__ __forceinline__ void tmem_alloc2(uint32_t *dst_smem, uint32_t ncols) {
  asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(dst_smem)),
               "r"(ncols)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc2(uint32_t taddr, uint32_t ncols) {
  asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
__device__ __forceinline__ void tc_mma2_f16(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                                            uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// arrive once on the barrier at the same smem offset in every CTA of cta_mask
__device__ __forceinline__ void tc_commit2_mc(uint64_t *bar, uint16_t cta_mask) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"(cta_mask)
      : "memory");
}

__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ float gelu_erf(float x) { return 0.5f * x * (1.0f + erff(x * 0.70710678118654752f)); }

// Exact-erf GELU, x * Phi(x), at ~half the instruction cost of erff: Phi is
// taken from erfc(|x|/sqrt 2) with the Chebyshev-fitted erfc of Numerical
// Recipes (erfcc; fractional error < 1.2e-7 everywhere), so Phi keeps full
// RELATIVE accuracy in both tails (x*Phi(x) -> 0 for x << 0).  One MUFU.RCP,
// one MUFU.EX2, ~16 FMA-pipe ops; error << one bf16 ulp of the result.
__device__ __forceinline__ float gelu_fast(float x) {
  const float z = fabsf(x) * 0.70710678118654752f;
  float t;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t) : "f"(fmaf(0.5f, z, 1.0f)));
  float p = 0.17087277f;
  p = fmaf(p, t, -0.82215223f);
  p = fmaf(p, t, 1.48851587f);
  p = fmaf(p, t, -1.13520398f);
  p = fmaf(p, t, 0.27886807f);
  p = fmaf(p, t, -0.18628806f);
  p = fmaf(p, t, 0.09678418f);
  p = fmaf(p, t, 0.37409196f);
  p = fmaf(p, t, 1.00002368f);
  p = fmaf(p, t, -1.26551223f);
  float e;                                                       // exp(-z^2 + p)
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e) : "f"(fmaf(-z, z, p) * 1.4426950408889634f));
  const float half_erfc = 0.5f * t * e;                          // 0.5 erfc(z) = Phi(-|x|)
  const float phi = x >= 0.f ? 1.0f - half_erfc : half_erfc;
  return x * phi;
}

// gelu_fast on a pair of values with Blackwell's packed fp32x2 FMA/MUL
// (FFMA2): same arithmetic, same rounding per element, ~35 % fewer issued
// instructions -- the FFN1 epilogue is issue-bound.
#ifndef E3_GELU_NR
// GELU(x) = x Phi(x) on packed fp32x2 with Abramowitz-Stegun 7.1.26:
// erfc(z) = t (a1 + a2 t + ... + a5 t^4) e^{-z^2}, t = 1 / (1 + p z), |error|
// <= 1.5e-7 absolute (GELU relative error <= 5e-5 for |x| < 3; the output is
// rounded to bf16, 2^-9).  Half the polynomial of the Numerical Recipes erfc
// (E3_GELU_NR): the GELU epilogue of FFN1 is issue-bound next to the MMAs.
__device__ __forceinline__ float2 gelu_fast2(float2 x) {
  const float2 z = __fmul2_rn(make_float2(fabsf(x.x), fabsf(x.y)), make_float2(0.70710678118654752f, 0.70710678118654752f));
  const float2 d = __ffma2_rn(make_float2(0.3275911f, 0.3275911f), z, make_float2(1.0f, 1.0f));
  float2 t;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t.x) : "f"(d.x));
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t.y) : "f"(d.y));
  // 0.5 * a_i folded in: he = Phi(-|x|) = 0.5 erfc(|x| / sqrt 2)
  float2 p = make_float2(0.5307027145f, 0.5307027145f);
  p = __ffma2_rn(p, t, make_float2(-0.7265760135f, -0.7265760135f));
  p = __ffma2_rn(p, t, make_float2(0.7107068705f, 0.7107068705f));
  p = __ffma2_rn(p, t, make_float2(-0.142248368f, -0.142248368f));
  p = __ffma2_rn(p, t, make_float2(0.127414796f, 0.127414796f));
  const float2 arg = __fmul2_rn(x, __fmul2_rn(x, make_float2(-0.7213475204444817f, -0.7213475204444817f)));
  float2 e;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e.x) : "f"(arg.x));
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e.y) : "f"(arg.y));
  const float2 he = __fmul2_rn(__fmul2_rn(t, p), e);
  const float2 phi = make_float2(x.x >= 0.f ? 1.0f - he.x : he.x, x.y >= 0.f ? 1.0f - he.y : he.y);
  return __fmul2_rn(x, phi);
}
#else
__device__ __forceinline__ float2 gelu_fast2(float2 x) {
  const float2 z = __fmul2_rn(make_float2(fabsf(x.x), fabsf(x.y)), make_float2(0.70710678118654752f, 0.70710678118654752f));
  const float2 d = __ffma2_rn(make_float2(0.5f, 0.5f), z, make_float2(1.0f, 1.0f));
  float2 t;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t.x) : "f"(d.x));
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t.y) : "f"(d.y));
  float2 p = make_float2(0.17087277f, 0.17087277f);
  p = __ffma2_rn(p, t, make_float2(-0.82215223f, -0.82215223f));
  p = __ffma2_rn(p, t, make_float2(1.48851587f, 1.48851587f));
  p = __ffma2_rn(p, t, make_float2(-1.13520398f, -1.13520398f));
  p = __ffma2_rn(p, t, make_float2(0.27886807f, 0.27886807f));
  p = __ffma2_rn(p, t, make_float2(-0.18628806f, -0.18628806f));
  p = __ffma2_rn(p, t, make_float2(0.09678418f, 0.09678418f));
  p = __ffma2_rn(p, t, make_float2(0.37409196f, 0.37409196f));
  p = __ffma2_rn(p, t, make_float2(1.00002368f, 1.00002368f));
  p = __ffma2_rn(p, t, make_float2(-1.26551223f, -1.26551223f));
  const float2 nz = __fmul2_rn(z, make_float2(-1.0f, -1.0f));
  const float2 arg = __fmul2_rn(__ffma2_rn(nz, z, p), make_float2(1.4426950408889634f, 1.4426950408889634f));
  float2 e;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e.x) : "f"(arg.x));
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(e.y) : "f"(arg.y));
  const float2 he = __fmul2_rn(__fmul2_rn(t, e), make_float2(0.5f, 0.5f));   // Phi(-|x|)
  const float2 phi = make_float2(x.x >= 0.f ? 1.0f - he.x : he.x, x.y >= 0.f ? 1.0f - he.y : he.y);
  return __fmul2_rn(x, phi);
}
#endif

__device__ __forceinline__ int warp_id() { return threadIdx.x >> 5; }
__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }


// ---- diagnostics: kernel timeline (e3_debug_timeline).  When a device buffer
// is set (per translation unit: tl_set_<file>), thread 0 of every CTA of the
// instrumented kernels appends {kernel id | blockIdx.x << 16 | smid << 48, entry, released
// (after griddepcontrol.wait), end} globaltimer stamps; buf[0] is the count.
namespace {
__device__ unsigned long long *g_tl = nullptr;
}
constexpr int kTlCap = 1 << 15;
__device__ __forceinline__ unsigned long long tl_now() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
// b: g_tl read at kernel entry (a load at the CTA's last instruction would
// hold its exit for an L2 round trip)
__device__ __forceinline__ void tl_rec(unsigned long long *b, int kid, unsigned long long t0, unsigned long long t1) {
  if (!b) return;
  const unsigned long long t2 = tl_now();
  const unsigned long long i = atomicAdd(b, 1ull);
  if (i >= (unsigned long long)kTlCap) return;
  unsigned smid;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  b[1 + 4 * i] = (unsigned long long)kid | ((unsigned long long)blockIdx.x << 16) | ((unsigned long long)smid << 48);
  b[2 + 4 * i] = t0;
  b[3 + 4 * i] = t1;
  b[4 + 4 * i] = t2;
}
#define E3_TL_SETTER(name)                                             \
  e3_status name(void *buf) {                                         \
    unsigned long long *p = static_cast<unsigned long long *>(buf);   \
    E3_CUDA_TRY(cudaMemcpyToSymbol(g_tl, &p, sizeof(p)));             \
    return E3_OK;                                                     \
  }

#endif  // __CUDACC__

}  // namespace e3
