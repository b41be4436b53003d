// Launch counter and optional per-kernel CUDA-event profiling (bench.py's
// roofline numbers).  Disabled by default; when enabled every kernel of the
// split path is bracketed by two events on its own stream.
#pragma once

#include <cuda_runtime.h>

namespace e3 {

enum ProfKind {
  PK_GEMM_QKV = 0,
  PK_ATTN,
  PK_GEMM_O,
  PK_LN,
  PK_GEMM_FFN1,
  PK_GEMM_FFN2,
  PK_RAMP,
  PK_COMPACT,
  PK_COPY,
  PK_N
};

void count_launch();
// per-kernel profiling on (its events bracket each launch; the pipeline then
// runs a split's tail on the main stream, so no interval includes waiting for
// SMs held by an overlapping kernel)
bool prof_enabled();
// add algorithmic bytes to a kind after the fact (e.g. compaction: n_surv is
// only known once the run completed)
void prof_add_bytes(int kind, double bytes);

// RAII: event pair around one launch when profiling is on.  flops / bytes
// are the ALGORITHMIC work of the launch (valid rows only), accumulated per
// kind for achieved-rate reporting.
struct ProfScope {
  int kind;
  cudaStream_t st;
  double flops, bytes;
  int slot = -1;
  ProfScope(int kind, cudaStream_t st, double flops, double bytes);
  ~ProfScope();
};

}  // namespace e3
