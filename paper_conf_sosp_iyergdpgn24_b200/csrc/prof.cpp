// Launch counter + per-kernel event profiling (see prof.h, e3_ops.h).
#include "prof.h"

#include <atomic>
#include <cstring>
#include <mutex>
#include <vector>

#include "../../include/e3_ops.h"
#include "common.cuh"

namespace e3 {

namespace {

std::atomic<long long> g_launches{0};
std::atomic<int> g_enabled{0};

struct Pending {
  int kind;
  cudaEvent_t a, b;
  double flops, bytes;
};

struct Profiler {
  std::mutex mu;
  std::vector<cudaEvent_t> pool;
  std::vector<Pending> pending;
  double ms[PK_N] = {};
  double flops[PK_N] = {};
  double bytes[PK_N] = {};
  long long count[PK_N] = {};

  cudaEvent_t get() {
    if (!pool.empty()) {
      cudaEvent_t e = pool.back();
      pool.pop_back();
      return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
  }
  void drain() {
    for (auto &p : pending) {
      float t = 0.f;
      cudaEventSynchronize(p.b);
      cudaEventElapsedTime(&t, p.a, p.b);
      ms[p.kind] += t;
      flops[p.kind] += p.flops;
      bytes[p.kind] += p.bytes;
      count[p.kind] += 1;
      pool.push_back(p.a);
      pool.push_back(p.b);
    }
    pending.clear();
  }
};

Profiler &prof() {
  static Profiler *p = new Profiler();
  return *p;
}

const char *kNames[PK_N] = {"gemm_qkv", "attention", "gemm_o", "layernorm", "gemm_ffn1",
                            "gemm_ffn2", "ramp",      "compact", "queue_copy"};

}  // namespace

void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

void prof_add_bytes(int kind, double b) {
  if (!g_enabled.load(std::memory_order_relaxed)) return;
  Profiler &P = prof();
  std::lock_guard<std::mutex> g(P.mu);
  P.bytes[kind] += b;
}

ProfScope::ProfScope(int kind_, cudaStream_t st_, double flops_, double bytes_)
    : kind(kind_), st(st_), flops(flops_), bytes(bytes_) {
  if (!g_enabled.load(std::memory_order_relaxed)) return;
  Profiler &P = prof();
  std::lock_guard<std::mutex> g(P.mu);
  Pending p{kind, P.get(), P.get(), flops, bytes};
  cudaEventRecord(p.a, st);
  P.pending.push_back(p);
  slot = (int)P.pending.size() - 1;
}

ProfScope::~ProfScope() {
  if (slot < 0) return;
  Profiler &P = prof();
  std::lock_guard<std::mutex> g(P.mu);
  cudaEventRecord(P.pending[slot].b, st);
}

bool prof_enabled() { return g_enabled.load() != 0; }

}  // namespace e3

extern "C" {

long long e3_kernel_launches(void) { return e3::g_launches.load(); }

e3_status e3_profile_enable(int32_t on) {
  e3::Profiler &P = e3::prof();
  std::lock_guard<std::mutex> g(P.mu);
  P.drain();
  e3::g_enabled.store(on ? 1 : 0);
  return E3_OK;
}

e3_status e3_profile_read(int32_t kind, double *ms, double *flops, double *bytes, long long *launches,
                          const char **name) {
  if (kind < 0 || kind >= e3::PK_N) {
    e3::set_error("profile kind out of range");
    return E3_EINVAL;
  }
  e3::Profiler &P = e3::prof();
  std::lock_guard<std::mutex> g(P.mu);
  P.drain();
  if (ms) *ms = P.ms[kind];
  if (flops) *flops = P.flops[kind];
  if (bytes) *bytes = P.bytes[kind];
  if (launches) *launches = P.count[kind];
  if (name) *name = e3::kNames[kind];
  return E3_OK;
}

e3_status e3_profile_reset(void) {
  e3::Profiler &P = e3::prof();
  std::lock_guard<std::mutex> g(P.mu);
  P.drain();
  std::memset(P.ms, 0, sizeof P.ms);
  std::memset(P.flops, 0, sizeof P.flops);
  std::memset(P.bytes, 0, sizeof P.bytes);
  std::memset(P.count, 0, sizeof P.count);
  return E3_OK;
}

}  // extern "C"
