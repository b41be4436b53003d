// Split executor internals (shared by split.cu and pipeline.cu).
#pragma once

#include <memory>
#include <vector>

#include "kernels.h"

namespace e3 {

// compaction ticket, one ramp ticket per group of kRampRowsPerCta rows (B <=
// 4096), the fused ramp + compaction's counters (kernels.h)
constexpr int kCtrWords = kCtrWordsAll;

// Activation workspace for one batch of B rows.  Splits that run serially on
// one stream may share a workspace (the pipeline does).
struct Workspace {
  int device = 0;
  int B = 0, S = 0, H = 0, F = 0;
  int elem = 2;                   // bytes per activation element: 2 (BF16) or 4 (FP32)
  void *qkv = nullptr, *ctx = nullptr, *y = nullptr, *x1 = nullptr, *h = nullptr, *xa = nullptr, *xb = nullptr;
  // the split's last layer output and alive flags of runs with parity 1 (the
  // last ramp + compaction of run j overlaps run j+1 on a second stream:
  // split_run_to's tail_st)
  void *yt = nullptr;
  void *yt0 = nullptr;            // the same for runs with parity 0 (never a non-last layer's output)
  uint8_t *alive_t = nullptr;
  float *pool = nullptr;
  uint8_t *alive = nullptr;
  unsigned *ctr = nullptr;        // [kCtrWords]: compaction ticket, ramp row-group tickets, attention items
  int attn_parity = 0;            // which attention counter pair the next launch uses (attn_run)
  int *err = nullptr;             // device error flag: a kernel saw an argument outside its range
  // LLAMA decode (allocated by ensure_llama): LM-head tile statistics,
  // stream-K partials and tickets of the decode GEMMs, RoPE cos/sin table
  float4 *lm_stats = nullptr;
  float *dec_part = nullptr;
  unsigned *dec_tickets = nullptr;
  float2 *rope = nullptr;
  size_t lm_stats_elems = 0, part_elems = 0, ticket_elems = 0;
  int rope_ctx = 0, rope_hd = 0;
  double rope_theta = 0;
  e3_status ensure_llama(int V, size_t part_elems, size_t tickets, int max_ctx, int head_dim, double theta);
  ~Workspace();
  static e3_status create(int device, int B, int S, int H, int F, int elem, std::shared_ptr<Workspace> *out);
};

}  // namespace e3

struct e3_split {
  e3_split_desc d;
  int device = 0;
  int sms = 148;
  bool poisoned = false;
  std::vector<e3_layer_weights> L;      // layers [begin, end)
  std::vector<e3_ramp_weights> R;       // ramps listed in d.ramp_layer
  std::shared_ptr<e3::Workspace> ws;
  struct LayerMaps {
    e3::GemmMaps qkv, o, f1, f2;
    e3::GemmMaps f2t;     // last layer: FFN2 writing Workspace::yt (runs with parity 1)
    e3::GemmMaps f2t0;    // last layer: FFN2 writing Workspace::yt0 (runs with parity 0)
    e3::LnGemmMaps oln;   // fused O projection + residual + LayerNorm (when use_oln)
  };
  bool use_oln = false;
  std::vector<LayerMaps> maps;
  // LLAMA decode: per layer the four decode GEMMs, per ramp the LM head
  struct DecLayer {
    e3::DecMaps qkv, o, gu, down;
  };
  std::vector<DecLayer> dmaps;
  std::vector<e3::DecMaps> lm_maps;
  int mc_qkv = 1, mc_o = 1, mc_gu = 1, mc_down = 1, mc_lm = 1;   // stream-K partial slots per tile
  e3_kv_cache kv{};
  std::vector<void *> kv_k, kv_v;       // this split's layers' cache pointers
  e3::AttnMaps attn;
  int bn_qkv = 0, bn_o = 0, bn_f1 = 0, bn_f2 = 0;
};

namespace e3 {

e3_status split_validate(const e3_split_desc *d, const e3_weights *w);
e3_status split_create_shared(const e3_split_desc *d, const e3_weights *w, int device,
                              std::shared_ptr<Workspace> ws, e3_split **out);
// Runs the split; survivors go to `dst` (contiguous or a queue ring).
// tail_st (optional): the stream the run ENDS on.  Where the split allows it
// (bf16 encoder, one active ramp: split_tail_overlap) the last ramp and the
// compaction run there, forked from `st` by `fork` after the last layer, and
// read the parity-`par` copies of the last layer output and alive flags, so
// they overlap the next run's layers on `st`; otherwise `tail_st` just waits
// for `st`.  The caller orders run j's start on `st` after run j-2's tail
// (the parity buffers are reused) and reads dst / id_in until the tail ends.
e3_status split_run_to(e3_split *s, cudaStream_t st, const void *x_in, const int64_t *id_in,
                       const int32_t *n_valid_dev, int n_valid_host, const RingDst &dst, int32_t *n_surv_dev,
                       const e3_exits *ex, cudaStream_t tail_st = nullptr, int par = 0, cudaEvent_t fork = nullptr);
bool split_tail_overlap(const e3_split *s);
// multi-step decode: K/V of layer l (in this split) for the chunk's tokens exited before l
e3_status llama_fill_layer(e3_split *s, int l, cudaStream_t st, const int64_t *ids_in, int nv, const e3_exits &ex,
                           int64_t *ids_buf);

}  // namespace e3
