// Mergeable softmax statistics of a slice of logits: (max m, argmax, s = sum
// e^(z-m), u = sum e^(z-m) (z-m)).  Two slices merge exactly (up to fp32
// rounding) into the statistics of their union; max-prob = 1 / s and
// entropy = log s - u / s of the whole row (used by the ViT ramp's cluster
// merge and the LM-head ramp's tile merge).
#pragma once

#include "common.cuh"

namespace e3 {

struct SoftStat {
  float m, s, u;
  int idx;   // -1: empty slice
};

// merge b into a; ties in the max keep the lower class index
__device__ __forceinline__ SoftStat soft_merge(SoftStat a, SoftStat b) {
  if (b.idx < 0) return a;
  if (a.idx < 0) return b;
  const float M = fmaxf(a.m, b.m);
  const float ea = expf(a.m - M), eb = expf(b.m - M);
  SoftStat r;
  r.m = M;
  r.s = a.s * ea + b.s * eb;
  r.u = ea * (a.u + a.s * (a.m - M)) + eb * (b.u + b.s * (b.m - M));
  r.idx = (b.m > a.m || (b.m == a.m && b.idx < a.idx)) ? b.idx : a.idx;
  return r;
}

__device__ __forceinline__ SoftStat soft_shfl_xor(const SoftStat &st, int o) {
  SoftStat r;
  r.m = __shfl_xor_sync(0xffffffffu, st.m, o);
  r.s = __shfl_xor_sync(0xffffffffu, st.s, o);
  r.u = __shfl_xor_sync(0xffffffffu, st.u, o);
  r.idx = __shfl_xor_sync(0xffffffffu, st.idx, o);
  return r;
}

}  // namespace e3
