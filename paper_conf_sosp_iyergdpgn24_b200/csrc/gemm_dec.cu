// Decode-shaped GEMMs of the LLaMA split:
//     Y[T, N] = epi( X[T, K] . W[N, K]^T ),   T = tokens of the batch (32..128)
// bf16 operands, fp32 accumulation in TMEM.
//
// T is far below one MMA tile and the weights are read exactly once per
// launch, so the path is bound by streaming W from HBM (405 MB per Llama-7B
// layer).  Design (DESIGN.md §6 K7):
//   * SWAP AB: the weight tile is the MMA's M side (128 rows of W), the
//     tokens are its N side: D[128, T] = W_tile . X^T with both operands
//     K-major in 128-byte-swizzled smem, tcgen05.mma.cta_group::1 M=128 N=T.
//     No padding of T up to a 128-row tile, no wasted tensor work.
//   * persistent CTAs (one per SM) walk UNITS = (128-row tile, K slice);
//     split-K (ks slices) keeps >= 148 units in flight for the narrow
//     matrices (W_o, W_down: 32 tiles).  A slice's fp32 partial goes to a
//     workspace; the last CTA of a tile (atomic ticket) sums the ks partials
//     in slice order (deterministic) and runs the epilogue.
//   * warp 0 = TMA producer: the first stages' W boxes are issued BEFORE
//     griddepcontrol.wait (weights never depend on the previous kernel), so
//     the weight stream starts while the previous kernel drains; warp 1 = one
//     MMA thread; warps 2-5 = epilogue (TMEM lane quarter = warp % 4), through
//     an fp32 smem tile [128][T+1].
//   * epilogues: STORE, RESID (+ residual), SWIGLU (tile rows 0-63 = W_gate
//     rows, 64-127 = the matching W_up rows, two TMA boxes per stage; out =
//     SiLU(g) * u), QKV_ROPE (one head per tile since head_dim = 128: rotate
//     pairs (j, j+64) with a cos/sin table of exact angles, q -> Q buffer, k/v
//     -> the KV cache at (slot, pos) of each token), LOGITS (fp32 logits + per
//     tile softmax statistics (max, sum e, sum e*(z-max), argmax) per token).
#include <cmath>
#include <vector>

#include "common.cuh"
#include "kernels.h"
#include "prof.h"

namespace e3 {

namespace {

constexpr int DM = 128;            // weight rows per tile (MMA M)
constexpr int DK = 64;             // K per 128-byte swizzle atom / TMA box
constexpr int kDThreads = 192;     // warp 0 TMA, warp 1 MMA, warps 2-5 epilogue
constexpr int kSmemMax = 232448;

template <int T>
struct DCfg {
  static constexpr int kWBytes = DM * DK * 2;               // 16 KB
  static constexpr int kXBytes = T * DK * 2;
  static constexpr int kStageBytes = kWBytes + kXBytes;
  static constexpr int kEBytes = DM * (T + 1) * 4;          // fp32 epilogue tile
  static constexpr int kStages = (kSmemMax - kEBytes - 1024 - 2048) / kStageBytes;
  static constexpr int kTmemCols = (2 * T <= 32) ? 32 : (2 * T <= 64) ? 64 : (2 * T <= 128) ? 128 : 256;
  static constexpr int kSmem = kStages * kStageBytes + kEBytes + 1024 + 2048;   // + barriers, token tables
};

__device__ __forceinline__ void epi_bar() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

template <int T, int EPI>
__global__ void __launch_bounds__(kDThreads, 1)
    gemm_dec_kernel(const __grid_constant__ CUtensorMap tmW, const __grid_constant__ CUtensorMap tmW2,
                    const __grid_constant__ CUtensorMap tmX, DecArgs a) {
  using CF = DCfg<T>;
  constexpr int S = CF::kStages;
  constexpr int P = T + 1;
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *sW = smem;
  uint8_t *sX = smem + S * CF::kWBytes;
  float *sE = reinterpret_cast<float *>(smem + S * CF::kStageBytes);
  uint64_t *full = reinterpret_cast<uint64_t *>(reinterpret_cast<uint8_t *>(sE) + CF::kEBytes);
  uint64_t *empty = full + S;
  uint64_t *tfull = empty + S;     // [2]
  uint64_t *tempty = tfull + 2;    // [2]
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(tempty + 2);
  int *s_last = reinterpret_cast<int *>(tmem_slot + 1);
  int *sPos = s_last + 1;          // [T]
  int *sSlot = sPos + T;           // [T]

  const int warp = warp_id(), lane = lane_id();
  const int tiles = (EPI == E3_DEC_SWIGLU) ? a.N / 64 : (a.N + DM - 1) / DM;
  const int units = tiles * a.ks;
  const int nkb = a.K / DK / a.ks;

  if (warp == 0 && lane == 0) {
    tma_prefetch(&tmW);
    if (EPI == E3_DEC_SWIGLU) tma_prefetch(&tmW2);
    tma_prefetch(&tmX);
  }
  if (warp == 1 && lane == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&tfull[i], 1);
      mbar_init(&tempty[i], 4);    // 4 epilogue warps
    }
    fence_barrier_init();
  }
  if (warp == 2) tmem_alloc(tmem_slot, CF::kTmemCols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------- TMA producer
    if (lane == 0) {
      auto coords = [&](int it, int &n0, int &k0) {   // it-th (unit, kb) of this CTA
        const int u = blockIdx.x + (it / nkb) * gridDim.x;
        const int kb = it % nkb;
        const int tile = u / a.ks, ksl = u % a.ks;
        n0 = (EPI == E3_DEC_SWIGLU) ? tile * 64 : tile * DM;
        k0 = (ksl * nkb + kb) * DK;
        return u < units;
      };
      int my_units = 0;
      for (int u = blockIdx.x; u < units; u += gridDim.x) ++my_units;
      const int total = my_units * nkb;
      const int pre = total < S ? total : S;
      // weights first: they do not depend on the previous kernel
      for (int it = 0; it < pre; ++it) {
        int n0, k0;
        coords(it, n0, k0);
        mbar_expect_tx(&full[it], CF::kStageBytes);
        if (EPI == E3_DEC_SWIGLU) {
          tma_load_2d(sW + it * CF::kWBytes, &tmW, &full[it], k0, n0);
          tma_load_2d(sW + it * CF::kWBytes + CF::kWBytes / 2, &tmW2, &full[it], k0, n0);
        } else {
          tma_load_2d(sW + it * CF::kWBytes, &tmW, &full[it], k0, n0);
        }
      }
      pdl_wait();
      pdl_trigger();
      for (int it = 0; it < pre; ++it) {
        int n0, k0;
        coords(it, n0, k0);
        tma_load_2d(sX + it * CF::kXBytes, &tmX, &full[it], k0, 0);
      }
      int stage = pre % S;
      uint32_t phase = (pre == S) ? 1 : 0;
      for (int it = pre; it < total; ++it) {
        int n0, k0;
        coords(it, n0, k0);
        mbar_wait(&empty[stage], phase ^ 1);
        mbar_expect_tx(&full[stage], CF::kStageBytes);
        if (EPI == E3_DEC_SWIGLU) {
          tma_load_2d(sW + stage * CF::kWBytes, &tmW, &full[stage], k0, n0);
          tma_load_2d(sW + stage * CF::kWBytes + CF::kWBytes / 2, &tmW2, &full[stage], k0, n0);
        } else {
          tma_load_2d(sW + stage * CF::kWBytes, &tmW, &full[stage], k0, n0);
        }
        tma_load_2d(sX + stage * CF::kXBytes, &tmX, &full[stage], k0, 0);
        if (++stage == S) { stage = 0; phase ^= 1; }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------- MMA issuer
    pdl_wait();
    pdl_trigger();
    if (lane == 0) {
      constexpr uint32_t idesc = idesc_bf16_f32(DM, T, 0);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      for (int u = blockIdx.x; u < units; u += gridDim.x) {
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * T;
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint64_t da = smem_desc_sw128(smem_u32(sW + stage * CF::kWBytes), 16, 1024);
          const uint64_t db = smem_desc_sw128(smem_u32(sX + stage * CF::kXBytes), 16, 1024);
#pragma unroll
          for (int k = 0; k < DK / 16; ++k)
            tc_mma_f16(d_tmem, da + (uint64_t)(2 * k), db + (uint64_t)(2 * k), idesc, (kb | k) != 0);
          tc_commit(&empty[stage]);
          if (++stage == S) { stage = 0; phase ^= 1; }
        }
        tc_commit(&tfull[acc]);
        if (++acc == 2) { acc = 0; acc_phase ^= 1; }
      }
    }
  } else {
    // ------------------------------------------------------- epilogue (warps 2-5)
    pdl_wait();
    pdl_trigger();
    const int q = warp & 3;
    const int r = q * 32 + lane;       // weight row of the tile == TMEM lane
    const int et = threadIdx.x - 64;   // 0..127
    if (EPI == E3_DEC_QKV_ROPE) {
      const int nv = a.n_valid_dev ? *a.n_valid_dev : a.n_valid_host;
      for (int t = et; t < T; t += 128) {
        int pos = 0, slot = -1;
        const int64_t id = a.ids[t];
        if (t < nv && id >= 0 && id < a.id_cap) {
          slot = a.slot_of_id[id];
          pos = a.pos_of_slot[slot];
        }
        sPos[t] = pos;
        sSlot[t] = slot;
      }
      epi_bar();
    }
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int u = blockIdx.x; u < units; u += gridDim.x) {
      const int tile = u / a.ks;
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16) + acc * T;
#pragma unroll
      for (int c = 0; c < T / 32; ++c) {
        uint32_t v[32];
        tmem_ld32(taddr + c * 32, v);
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 32; ++j) sE[r * P + c * 32 + j] = __uint_as_float(v[j]);
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[acc]);
      if (++acc == 2) { acc = 0; acc_phase ^= 1; }
      epi_bar();

      if (a.ks > 1) {
        // split-K: publish this slice, the tile's last arrival reduces in slice order
        float *part = a.part + (size_t)u * T * DM;
        for (int t = 0; t < T; ++t) part[t * DM + r] = sE[r * P + t];
        __threadfence();
        epi_bar();
        if (et == 0) {
          const unsigned prev = atomicAdd(&a.tickets[tile], 1u);
          *s_last = (prev == (unsigned)(a.ks - 1));
          if (*s_last) a.tickets[tile] = 0;   // ready for the next launch
        }
        epi_bar();
        if (!*s_last) continue;
        __threadfence();
        const float *base = a.part + (size_t)tile * a.ks * T * DM;
        for (int t = 0; t < T; ++t) {
          float s = 0.f;
          for (int j = 0; j < a.ks; ++j) s += __ldcg(base + ((size_t)j * T + t) * DM + r);
          sE[r * P + t] = s;
        }
        epi_bar();
      }

      // ---------------------------------------------------- final epilogue
      if (EPI == E3_DEC_STORE || EPI == E3_DEC_RESID) {
        const int n = tile * DM + r;
        if (n < a.N) {
          for (int t = 0; t < T; ++t) {
            float v = sE[r * P + t];
            if (EPI == E3_DEC_RESID) v += bf2f(a.R[(size_t)t * a.ldo + n]);
            a.Y[(size_t)t * a.ldo + n] = __float2bfloat16_rn(v);
          }
        }
      } else if (EPI == E3_DEC_SWIGLU) {
        if (r < 64) {
          const int f = tile * 64 + r;
          for (int t = 0; t < T; ++t) {
            const float g = sE[r * P + t], up = sE[(r + 64) * P + t];
            a.Y[(size_t)t * a.ldo + f] = __float2bfloat16_rn(g / (1.0f + expf(-g)) * up);
          }
        }
      } else if (EPI == E3_DEC_QKV_ROPE) {
        // tile = one head (head_dim 128): q heads, then k heads, then v heads
        const int hq = tile;
        const bool is_q = hq < a.nh, is_k = !is_q && hq < a.nh + a.kvh;
        const int j = r & 63;
        for (int t = 0; t < T; ++t) {
          float v = sE[r * P + t];
          if (is_q || is_k) {
            const float pr = sE[(r ^ 64) * P + t];
            const float2 cs = a.rope[(size_t)sPos[t] * 64 + j];
            v = (r < 64) ? fmaf(v, cs.x, -pr * cs.y) : fmaf(v, cs.x, pr * cs.y);
          }
          const __nv_bfloat16 o = __float2bfloat16_rn(v);
          if (is_q) {
            a.Y[(size_t)t * a.ldo + hq * 128 + r] = o;
          } else if (sSlot[t] >= 0) {
            const int kh = is_k ? hq - a.nh : hq - a.nh - a.kvh;
            __nv_bfloat16 *cache = is_k ? a.kc : a.vc;
            cache[(((size_t)sSlot[t] * a.kvh + kh) * a.max_ctx + sPos[t]) * 128 + r] = o;
          }
        }
      } else if (EPI == E3_DEC_LOGITS) {
        const int n0 = tile * DM;
        const int rows = (a.N - n0) < DM ? (a.N - n0) : DM;
        if (r < rows)
          for (int t = 0; t < T; ++t) a.Z[(size_t)t * a.N + n0 + r] = sE[r * P + t];
        for (int t = et; t < T; t += 128) {
          float m = sE[t];
          int idx = 0;
          for (int i = 1; i < rows; ++i) {
            const float z = sE[i * P + t];
            if (z > m) { m = z; idx = i; }
          }
          float s = 0.f, uu = 0.f;
          for (int i = 0; i < rows; ++i) {
            const float d = sE[i * P + t] - m;
            const float e = expf(d);
            s += e;
            uu = fmaf(e, d, uu);
          }
          a.stats[(size_t)tile * T + t] = make_float4(m, s, uu, __int_as_float(n0 + idx));
        }
      }
      epi_bar();                        // sE is reused by the next unit
    }
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2) tmem_dealloc(tmem_base, CF::kTmemCols);
}

template <int T, int EPI>
e3_status dec_launch(const DecMaps &m, const DecArgs &a, int grid, cudaStream_t st) {
  auto kern = gemm_dec_kernel<T, EPI>;
  static bool attr_done = false;
  if (!attr_done) {
    E3_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, DCfg<T>::kSmem));
    attr_done = true;
  }
  E3_CUDA_TRY(launch_k(kern, dim3(grid), dim3(kDThreads), DCfg<T>::kSmem, st, m.w, m.w2, m.x, a));
  E3_CUDA_TRY(cudaGetLastError());
  count_launch();
  return E3_OK;
}

template <int T>
e3_status dec_launch_epi(const DecMaps &m, const DecArgs &a, int grid, cudaStream_t st) {
  switch (a.epi) {
    case E3_DEC_STORE: return dec_launch<T, E3_DEC_STORE>(m, a, grid, st);
    case E3_DEC_RESID: return dec_launch<T, E3_DEC_RESID>(m, a, grid, st);
    case E3_DEC_SWIGLU: return dec_launch<T, E3_DEC_SWIGLU>(m, a, grid, st);
    case E3_DEC_QKV_ROPE: return dec_launch<T, E3_DEC_QKV_ROPE>(m, a, grid, st);
    case E3_DEC_LOGITS: return dec_launch<T, E3_DEC_LOGITS>(m, a, grid, st);
  }
  set_error("bad decode epilogue");
  return E3_EINVAL;
}

}  // namespace

int dec_tiles(int N, int epi) { return epi == E3_DEC_SWIGLU ? N / 64 : (N + DM - 1) / DM; }

int dec_pick_ks(int N, int K, int epi, int sms) {
  // minimise (units per CTA) x (K per unit + split-K traffic in K columns);
  // a partial [T x 128] fp32 written and read back ~ 256 columns of W
  const int tiles = dec_tiles(N, epi);
  int best = 1;
  long best_cost = -1;
  for (int ks = 1; ks <= 16; ++ks) {
    if (K % (ks * DK)) continue;
    const long units = (long)tiles * ks;
    const long per = (units + sms - 1) / sms;
    const long cost = per * (K / ks + (ks > 1 ? 256 : 0));
    if (best_cost < 0 || cost < best_cost) { best = ks; best_cost = cost; }
  }
  return best;
}

e3_status dec_tmaps(DecMaps *m, const void *X, int T, int K, const void *W, const void *W2, int N, int epi) {
  const uint32_t wrows = (epi == E3_DEC_SWIGLU) ? 64 : DM;
  e3_status s = make_tmap_2d(&m->w, W, (uint64_t)N, (uint64_t)K, (uint64_t)K, wrows, DK);
  if (s == E3_OK) s = make_tmap_2d(&m->w2, W2 ? W2 : W, (uint64_t)N, (uint64_t)K, (uint64_t)K, wrows, DK);
  if (s == E3_OK) s = make_tmap_2d(&m->x, X, (uint64_t)T, (uint64_t)K, (uint64_t)K, (uint32_t)T, DK);
  return s;
}

e3_status dec_run(const DecMaps &m, const DecArgs &a, int sms, cudaStream_t st) {
  const int units = dec_tiles(a.N, a.epi) * a.ks;
  const int grid = units < sms ? units : sms;
  switch (a.T) {
    case 32: return dec_launch_epi<32>(m, a, grid, st);
    case 64: return dec_launch_epi<64>(m, a, grid, st);
    case 128: return dec_launch_epi<128>(m, a, grid, st);
  }
  set_error("decode GEMM: batch must be 32, 64 or 128 tokens");
  return E3_EUNSUPPORTED;
}

e3_status rope_table(int max_ctx, int head_dim, double theta, float2 **out) {
  const int half = head_dim / 2;
  std::vector<float2> h((size_t)max_ctx * half);
  for (int p = 0; p < max_ctx; ++p)
    for (int j = 0; j < half; ++j) {
      const double ang = (double)p * std::pow(theta, -2.0 * j / head_dim);
      h[(size_t)p * half + j] = make_float2((float)std::cos(ang), (float)std::sin(ang));
    }
  float2 *d = nullptr;
  E3_CUDA_TRY(cudaMalloc(&d, h.size() * sizeof(float2)));
  E3_CUDA_TRY(cudaMemcpy(d, h.data(), h.size() * sizeof(float2), cudaMemcpyHostToDevice));
  *out = d;
  return E3_OK;
}

}  // namespace e3
