// Counter-based (patience) exit rule of dependent-exit EE-DNNs (SURVEY §8(f)
// NEXT-4; "require off-ramps classifiers to continuously
// generate identical predictions for pre-defined times", PABEE in §5.6; DESIGN
// R26).  The state of an input -- its previous prediction and counter --
// lives in e3_exits.state[id] (packed (label + 1) << 16 | count; 0 = no ramp
// evaluated yet) and travels with the input from split to split, as §3.4 asks
// ("𝐸3 keeps track of this information").  Exactly one
// ramp thread updates an input's state at a time (rows are disjoint).
#pragma once

#include "common.cuh"

namespace e3 {

// counter update at an evaluated ramp; *metric <- the counter; pass iff
// counter >= patience (tau holds the patience t)
__device__ __forceinline__ bool patience_step(int32_t *state, int64_t id, int64_t cap, int label, float tau,
                                              float *metric) {
  int c = 0;
  if (state && id >= 0 && id < cap) {
    const int32_t s = state[id];
    const int prev = (s >> 16) - 1;
    c = (s != 0 && prev == label) ? (s & 0xffff) + 1 : 0;
    if (c > 0xffff) c = 0xffff;
    state[id] = ((label + 1) << 16) | c;
  }
  *metric = (float)c;
  return c >= (int)tau;
}

}  // namespace e3
