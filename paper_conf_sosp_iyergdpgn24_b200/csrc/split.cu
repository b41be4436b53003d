// Split executor: one split of the early-exit encoder
// on one constant-size batch, stream-ordered, no host synchronisation.
//
// For each layer l of the split (BERT post-LN, R11):
//   qkv = gemm(x, W_qkv) + b                    [tcgen05 GEMM, bias epilogue]
//   ctx = attention(qkv)                        [tcgen05 attention]
//   y   = gemm(ctx, W_o) + b_o + x              [residual epilogue]
//   x1  = LN1(y)                                [row LayerNorm]
//   h   = GELU(gemm(x1, W_1) + b_1)             [GELU epilogue]
//   y   = gemm(h, W_2) + b_2 + x1               [residual epilogue]
//   x2  = LN2(y)
//   if a ramp follows l (and is evaluated): fused ramp + threshold test
// then the stable compaction of the rows still alive.  Rows that exit at an
// inner ramp (inner = EXACT) are recorded there and carried masked to the end
// of the split ("mark and carry"; R7), which yields plan-independent
// results.  Activations ping-pong between two workspace buffers so the caller's
// x_in is never written.
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>

#include "common.cuh"
#include "prof.h"
#include "split.h"
#include "fp32_path.h"

namespace e3 {

namespace {
// Diagnostics only: E3_SKIP=<bitmask of profile kinds> leaves those kernels of
// the BERT split path out (results are then meaningless; used to measure each
// kernel's incremental cost inside the PDL-chained sequence,
// scripts/layer_time.py).
bool skip(int kind) {
  static const int mask = [] {
    const char *e = getenv("E3_SKIP");
    return e ? atoi(e) : 0;
  }();
  return (mask >> kind) & 1;
}
}  // namespace

Workspace::~Workspace() {
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(device);
  void *bufs[] = {qkv, ctx, y, x1, h, xa, xb, yt, yt0, alive_t, pool, alive, ctr, err, lm_stats, dec_part, dec_tickets, rope};
  for (void *p : bufs)
    if (p) cudaFree(p);
  cudaSetDevice(prev);
}

e3_status Workspace::ensure_llama(int V, size_t part, size_t tickets, int max_ctx, int head_dim, double theta) {
  const size_t st = (size_t)((V + 127) / 128) * B;
  if (st > lm_stats_elems) {
    if (lm_stats) cudaFree(lm_stats);
    lm_stats = nullptr;
    E3_CUDA_TRY(cudaMalloc(&lm_stats, st * sizeof(float4)));
    lm_stats_elems = st;
  }
  if (part > part_elems) {
    if (dec_part) cudaFree(dec_part);
    dec_part = nullptr;
    E3_CUDA_TRY(cudaMalloc(&dec_part, part * sizeof(float)));
    part_elems = part;
  }
  if (tickets > ticket_elems) {
    if (dec_tickets) cudaFree(dec_tickets);
    dec_tickets = nullptr;
    E3_CUDA_TRY(cudaMalloc(&dec_tickets, tickets * sizeof(unsigned)));
    E3_CUDA_TRY(cudaMemset(dec_tickets, 0, tickets * sizeof(unsigned)));
    ticket_elems = tickets;
  }
  if (!rope || rope_ctx != max_ctx || rope_hd != head_dim || rope_theta != theta) {
    if (rope) cudaFree(rope);
    rope = nullptr;
    e3_status r = rope_table(max_ctx, head_dim, theta, &rope);
    if (r != E3_OK) return r;
    rope_ctx = max_ctx;
    rope_hd = head_dim;
    rope_theta = theta;
  }
  return E3_OK;
}

e3_status Workspace::create(int device, int B, int S, int H, int F, int elem, std::shared_ptr<Workspace> *out) {
  auto ws = std::make_shared<Workspace>();
  ws->device = device;
  ws->B = B;
  ws->S = S;
  ws->H = H;
  ws->F = F;
  ws->elem = elem;
  const size_t M = (size_t)B * S, e = (size_t)elem;
  // qkv [M, 3H]; also the FP32 LLaMA decode's SwiGLU gate [M, F] (Llama-3: F = 3.5 H)
  E3_CUDA_TRY(cudaMalloc(&ws->qkv, M * (size_t)(3 * H > F ? 3 * H : F) * e));
  E3_CUDA_TRY(cudaMalloc(&ws->ctx, M * H * e));
  E3_CUDA_TRY(cudaMalloc(&ws->y, M * H * e));
  E3_CUDA_TRY(cudaMalloc(&ws->x1, M * H * e));
  E3_CUDA_TRY(cudaMalloc(&ws->h, M * F * e));
  E3_CUDA_TRY(cudaMalloc(&ws->xa, M * H * e));
  E3_CUDA_TRY(cudaMalloc(&ws->xb, M * H * e));
  E3_CUDA_TRY(cudaMalloc(&ws->pool, (size_t)B * H * 4));
  E3_CUDA_TRY(cudaMalloc(&ws->alive, (size_t)B));
  if (elem == 2) {   // tail buffers (bf16 encoder runs only)
    E3_CUDA_TRY(cudaMalloc(&ws->yt, M * H * e));
    E3_CUDA_TRY(cudaMalloc(&ws->yt0, M * H * e));
    E3_CUDA_TRY(cudaMalloc(&ws->alive_t, (size_t)B));
    E3_CUDA_TRY(cudaMemset(ws->alive_t, 0, (size_t)B));
  }
  E3_CUDA_TRY(cudaMalloc(&ws->ctr, kCtrWords * sizeof(unsigned)));
  E3_CUDA_TRY(cudaMemset(ws->ctr, 0, kCtrWords * sizeof(unsigned)));
  E3_CUDA_TRY(cudaMemset(ws->alive, 0, (size_t)B));
  E3_CUDA_TRY(cudaMalloc(&ws->err, sizeof(int)));
  E3_CUDA_TRY(cudaMemset(ws->err, 0, sizeof(int)));
  *out = ws;
  return E3_OK;
}

static bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

// LLAMA decode: head_dim 128, one token per row (S = 1),
// B in {32, 64, 128}, the caller's KV cache covering the split's layers.
static e3_status llama_validate(const e3_split_desc *d, const e3_weights *w) {
  if (d->dtype != E3_DTYPE_BF16 && d->dtype != E3_DTYPE_FP32) {
    set_error("e3_split_create (LLAMA): dtype must be BF16 or FP32");
    return E3_EUNSUPPORTED;
  }
  const int kvh = d->kv_heads > 0 ? d->kv_heads : d->heads;
  if (d->heads <= 0 || d->hidden != d->heads * 128 || d->heads % kvh || d->seq_len != 1 || d->ffn % 128 ||
      d->ffn <= 0 || (d->batch != 32 && d->batch != 64 && d->batch != 128) || d->num_labels < 1 ||
      d->hidden > 8192) {
    set_error("e3_split_create (LLAMA): need head_dim 128 (H = 128 * heads), heads % kv_heads == 0, S == 1, "
              "F % 128 == 0, B in {32, 64, 128}, H <= 8192");
    return E3_EUNSUPPORTED;
  }
  E3_CHECK_ARG(d->layer_begin >= 0 && d->layer_end > d->layer_begin && d->layer_end <= w->n_layers,
               "layer range outside the model");
  E3_CHECK_ARG(d->n_ramps >= 1 && d->n_ramps <= E3_MAX_RAMPS, "a split needs 1..64 ramps");
  for (int r = 0; r < d->n_ramps; ++r) {
    E3_CHECK_ARG(d->ramp_layer[r] >= d->layer_begin && d->ramp_layer[r] < d->layer_end, "ramp outside split");
    E3_CHECK_ARG(r == 0 || d->ramp_layer[r] > d->ramp_layer[r - 1], "ramp layers not ascending");
    E3_CHECK_ARG(d->ramp_index[r] >= 0 && d->ramp_index[r] < w->n_ramps, "ramp index outside the model");
    const e3_ramp_weights &R = w->ramp[d->ramp_index[r]];
    E3_CHECK_ARG(R.ln_g && R.w_c && aligned16(R.w_c), "LLAMA ramp needs ln_g (final norm) and w_c (LM head)");
  }
  E3_CHECK_ARG(d->ramp_layer[d->n_ramps - 1] == d->layer_end - 1, "a split must end in a ramp");
  E3_CHECK_ARG(d->test == E3_TEST_MAXPROB || d->test == E3_TEST_ENTROPY || d->test == E3_TEST_PATIENCE, "bad test");
  E3_CHECK_ARG(d->inner == E3_INNER_EXACT || d->inner == E3_INNER_DISABLED, "bad inner mode");
  for (int l = d->layer_begin; l < d->layer_end; ++l) {
    const e3_layer_weights &L = w->layer[l];
    const void *ps[] = {L.w_qkv, L.w_o, L.ln1_g, L.w_1, L.w_2, L.w_3, L.ln2_g};
    for (const void *p : ps) E3_CHECK_ARG(p && aligned16(p), "LLAMA layer weight pointer null or misaligned");
  }
  const e3_kv_cache *kv = w->kv;
  E3_CHECK_ARG(kv && kv->k && kv->v && kv->slot_of_id && kv->pos_of_slot, "LLAMA needs e3_weights.kv");
  E3_CHECK_ARG(kv->n_layers >= d->layer_end && kv->n_slots > 0 && kv->max_ctx > 0 && kv->id_capacity > 0,
               "KV cache does not cover the split");
  if (kv->max_ctx > 16384) {
    set_error("e3_split_create (LLAMA): max_ctx > 16384");
    return E3_EUNSUPPORTED;
  }
  for (int l = d->layer_begin; l < d->layer_end; ++l)
    E3_CHECK_ARG(kv->k[l] && kv->v[l] && aligned16(kv->k[l]) && aligned16(kv->v[l]), "KV layer pointer");
  return E3_OK;
}

e3_status split_validate(const e3_split_desc *d, const e3_weights *w) {
  E3_CHECK_ARG(d && w, "null descriptor or weights");
  if (d->arch != E3_ARCH_BERT && d->arch != E3_ARCH_VIT && d->arch != E3_ARCH_LLAMA_DECODE) {
    set_error("e3_split_create: unknown arch");
    return E3_EUNSUPPORTED;
  }
  if (d->arch == E3_ARCH_LLAMA_DECODE) return llama_validate(d, w);
  const bool vit = d->arch == E3_ARCH_VIT;
  if (d->dtype != E3_DTYPE_BF16 && d->dtype != E3_DTYPE_FP32) {
    set_error("e3_split_create: dtype must be BF16 or FP32");
    return E3_EUNSUPPORTED;
  }
  if (d->dtype == E3_DTYPE_FP32 && d->hidden > 2048) {
    set_error("e3_split_create: FP32 mode needs H <= 2048");
    return E3_EUNSUPPORTED;
  }
  E3_CHECK_ARG(d->hidden > 0 && d->heads > 0 && d->ffn > 0 && d->seq_len > 0 && d->batch > 0, "non-positive dims");
  if (d->hidden % 128 || d->hidden / d->heads != 64 || d->hidden % d->heads || d->ffn % 128 || d->seq_len > 256 ||
      d->batch > 4096 || d->num_labels < 1 || d->num_labels > (vit ? 2048 : 16) || d->hidden > 4096) {
    set_error("e3_split_create: unsupported shape (need H % 128 == 0, head_dim 64, F % 128 == 0, S <= 256, "
              "B <= 4096, 1 <= C <= 16 (BERT) or 2048 (VIT), H <= 4096)");
    return E3_EUNSUPPORTED;
  }
  E3_CHECK_ARG(d->layer_begin >= 0 && d->layer_end > d->layer_begin && d->layer_end <= w->n_layers,
               "layer range outside the model");
  E3_CHECK_ARG(d->n_ramps >= 1 && d->n_ramps <= E3_MAX_RAMPS, "a split needs 1..64 ramps");
  for (int r = 0; r < d->n_ramps; ++r) {
    E3_CHECK_ARG(d->ramp_layer[r] >= d->layer_begin && d->ramp_layer[r] < d->layer_end, "ramp outside split");
    E3_CHECK_ARG(r == 0 || d->ramp_layer[r] > d->ramp_layer[r - 1], "ramp layers not ascending");
    E3_CHECK_ARG(d->ramp_index[r] >= 0 && d->ramp_index[r] < w->n_ramps, "ramp index outside the model");
  }
  E3_CHECK_ARG(d->ramp_layer[d->n_ramps - 1] == d->layer_end - 1, "a split must end in a ramp");
  E3_CHECK_ARG(d->test == E3_TEST_MAXPROB || d->test == E3_TEST_ENTROPY || d->test == E3_TEST_PATIENCE, "bad test");
  E3_CHECK_ARG(d->inner == E3_INNER_EXACT || d->inner == E3_INNER_DISABLED, "bad inner mode");
  for (int l = d->layer_begin; l < d->layer_end; ++l) {
    const e3_layer_weights &L = w->layer[l];
    const void *ps[] = {L.w_qkv, L.b_qkv, L.w_o, L.b_o, L.ln1_g, L.ln1_b, L.w_1, L.b_1, L.w_2, L.b_2, L.ln2_g, L.ln2_b};
    for (const void *p : ps) E3_CHECK_ARG(p && aligned16(p), "layer weight pointer null or not 16-byte aligned");
  }
  for (int r = 0; r < d->n_ramps; ++r) {
    const e3_ramp_weights &R = w->ramp[d->ramp_index[r]];
    if (vit)
      E3_CHECK_ARG(R.ln_g && R.ln_b && R.w_c && R.b_c && aligned16(R.w_c), "ViT ramp weight pointer null / misaligned");
    else
      E3_CHECK_ARG(R.w_p && R.b_p && R.w_c && R.b_c && aligned16(R.w_p), "ramp weight pointer null / misaligned");
  }
  return E3_OK;
}

static e3_status check_device(int device) {
  cudaDeviceProp p;
  E3_CUDA_TRY(cudaGetDeviceProperties(&p, device));
  if (p.major != 10 || p.minor != 0) {
    set_error("E3 kernels are built for sm_100a (B200); device is sm_" + std::to_string(p.major * 10 + p.minor));
    return E3_EUNSUPPORTED;
  }
  return E3_OK;
}

// LLAMA: tensor maps of the decode GEMMs (activations in the workspace, so
// the maps are fixed for the handle's life), split-K choices, shared buffers
static e3_status llama_create(e3_split *s, const e3_weights *w) {
  const e3_split_desc &d = s->d;
  Workspace &ws = *s->ws;
  const int B = d.batch, H = d.hidden, F = d.ffn, V = d.num_labels;
  const int kvh = d.kv_heads > 0 ? d.kv_heads : d.heads;
  const int nqkv = (d.heads + 2 * kvh) * 128;
  s->kv = *w->kv;
  for (int l = 0; l < w->kv->n_layers; ++l) {
    s->kv_k.push_back(w->kv->k[l]);
    s->kv_v.push_back(w->kv->v[l]);
  }
  if (d.dtype == E3_DTYPE_FP32)   // SIMT fp32 kernels: the RoPE table, and a [B][V] logits scratch for the ramp
    return ws.ensure_llama(V, (size_t)B * V, 0, w->kv->max_ctx, 128, d.rope_theta > 0.f ? d.rope_theta : 10000.0);
  s->mc_qkv = dec_max_contrib(nqkv, H, E3_DEC_QKV_ROPE, s->sms);
  s->mc_o = dec_max_contrib(H, H, E3_DEC_RESID, s->sms);
  s->mc_gu = dec_max_contrib(F, H, E3_DEC_SWIGLU, s->sms);
  s->mc_down = dec_max_contrib(H, F, E3_DEC_RESID, s->sms);
  s->mc_lm = dec_max_contrib(V, H, E3_DEC_LOGITS, s->sms);
  size_t part = 0, tickets = 0;
  auto need = [&](int N, int mc, int epi) {
    const size_t t = (size_t)dec_tiles(N, epi);
    if (t * mc * B * 128 > part) part = t * mc * B * 128;
    if (t > tickets) tickets = t;
  };
  need(nqkv, s->mc_qkv, E3_DEC_QKV_ROPE);
  need(H, s->mc_o, E3_DEC_RESID);
  need(F, s->mc_gu, E3_DEC_SWIGLU);
  need(H, s->mc_down, E3_DEC_RESID);
  need(V, s->mc_lm, E3_DEC_LOGITS);
  if ((size_t)4 * B * H > part) part = (size_t)4 * B * H;   // split-K-by-4 partials (E3_DEC_PARTIAL), reused
  e3_status st = ws.ensure_llama(V, part, tickets, w->kv->max_ctx, 128, d.rope_theta > 0.f ? d.rope_theta : 10000.0);
  if (st != E3_OK) return st;
  const int nl = d.layer_end - d.layer_begin;
  s->dmaps.resize(nl);
  for (int i = 0; i < nl && st == E3_OK; ++i) {
    const e3_layer_weights &L = s->L[i];
    auto &m = s->dmaps[i];
    st = dec_tmaps(&m.qkv, ws.x1, B, H, L.w_qkv, nullptr, nqkv, E3_DEC_QKV_ROPE);
    if (st == E3_OK) st = dec_tmaps(&m.o, ws.ctx, B, H, L.w_o, nullptr, H, E3_DEC_RESID);
    if (st == E3_OK) st = dec_tmaps(&m.gu, ws.x1, B, H, L.w_1, L.w_3, F, E3_DEC_SWIGLU);
    if (st == E3_OK) st = dec_tmaps(&m.down, ws.h, B, F, L.w_2, nullptr, H, E3_DEC_RESID);
  }
  s->lm_maps.resize(d.n_ramps);
  for (int r = 0; r < d.n_ramps && st == E3_OK; ++r)
    st = dec_tmaps(&s->lm_maps[r], ws.x1, B, H, s->R[r].w_c, nullptr, V, E3_DEC_LOGITS);
  return st;
}

e3_status split_create_shared(const e3_split_desc *d, const e3_weights *w, int device, std::shared_ptr<Workspace> ws,
                              e3_split **out) {
  E3_CHECK_ARG(out, "null out");
  e3_status st = split_validate(d, w);
  if (st != E3_OK) return st;
  st = check_device(device);
  if (st != E3_OK) return st;
  E3_CUDA_TRY(cudaSetDevice(device));
  e3_split *s = new (std::nothrow) e3_split();
  if (!s) {
    set_error("out of host memory");
    return E3_ECUDA;
  }
  s->d = *d;
  s->device = device;
  s->sms = num_sms(device);
  const int B = d->batch, S = d->seq_len, H = d->hidden, F = d->ffn;
  for (int l = d->layer_begin; l < d->layer_end; ++l) s->L.push_back(w->layer[l]);
  for (int r = 0; r < d->n_ramps; ++r) s->R.push_back(w->ramp[d->ramp_index[r]]);
  const int elem = d->dtype == E3_DTYPE_FP32 ? 4 : 2;
  if (!ws) {
    st = Workspace::create(device, B, S, H, F, elem, &ws);
    if (st != E3_OK) {
      delete s;
      return st;
    }
  } else if (ws->B != B || ws->S != S || ws->H != H || ws->F != F || ws->elem != elem) {
    delete s;
    set_error("shared workspace shape mismatch");
    return E3_EINVAL;
  }
  s->ws = ws;
  if (d->arch == E3_ARCH_LLAMA_DECODE) {
    st = llama_create(s, w);
    if (st != E3_OK) {
      delete s;
      return st;
    }
    *out = s;
    return E3_OK;
  }
  if (d->dtype == E3_DTYPE_FP32) {   // SIMT fp32 kernels: no tensor maps
    *out = s;
    return E3_OK;
  }
  const int M = B * S;
  s->bn_qkv = gemm_pick_bn(M, 3 * H, H, s->sms, E3_EPI_BIAS);
  s->bn_o = gemm_pick_bn(M, H, H, s->sms, E3_EPI_BIAS_RESID);
  s->bn_f1 = gemm_pick_bn(M, F, H, s->sms, E3_EPI_BIAS_GELU);
  s->bn_f2 = gemm_pick_bn(M, H, F, s->sms, E3_EPI_BIAS_RESID);
  const int nl = d->layer_end - d->layer_begin;
  s->maps.resize(nl);
  const bool vit = d->arch == E3_ARCH_VIT;
  // Fused O projection + LayerNorm (K1b, gemm_ln.cu) unless E3_NO_FUSED_LN
  // is set: r01 timeline (scripts/timeline.py) 155.1 -> 149.8 us per BB
  // layer; E3_FUSED_LN forces it.  Only where its one-CTA-per-(128 rows, H/2 columns) grid is a
  // single wave: VT (788 CTAs) ran it at ~450 TF/s, 131 us vs ~85 us split
  s->use_oln = ln_gemm_supported(H, H) && getenv("E3_NO_FUSED_LN") == nullptr &&
               (getenv("E3_FUSED_LN") != nullptr || 2 * ((d->batch * d->seq_len + 127) / 128) <= s->sms);
  for (int i = 0; i < nl && st == E3_OK; ++i) {
    auto &m = s->maps[i];
    const void *prev = (i % 2 == 1) ? ws->xa : ws->xb;   // output of layer i-1
    void *out = (i % 2 == 0) ? ws->xa : ws->xb;          // output of layer i
    if (vit) {
      // pre-LN: QKV and FFN1 read the LayerNorm output in x1; FFN2 writes the
      // layer output (x1 + MLP) to the ping-pong buffer
      st = gemm_tmaps(&m.qkv, ws->x1, H, s->L[i].w_qkv, ws->qkv, M, 3 * H, H, s->bn_qkv);
    } else if (i > 0) {
      st = gemm_tmaps(&m.qkv, prev, H, s->L[i].w_qkv, ws->qkv, M, 3 * H, H, s->bn_qkv);
    }
    if (st == E3_OK) st = gemm_tmaps(&m.o, ws->ctx, H, s->L[i].w_o, ws->y, M, H, H, s->bn_o);
    if (st == E3_OK && s->use_oln)   // BERT: x1 = LN1(y1); ViT: y1 kept (residual), n2 = LN2(y1)
      st = ln_gemm_tmaps(&m.oln, ws->ctx, s->L[i].w_o, prev /* layer 0: the run's input, re-encoded per run */,
                         vit ? ws->y : nullptr, ws->x1, M, H, H);
    if (st == E3_OK) st = gemm_tmaps(&m.f1, ws->x1, H, s->L[i].w_1, ws->h, M, F, H, s->bn_f1);
    if (st == E3_OK) st = gemm_tmaps(&m.f2, ws->h, F, s->L[i].w_2, vit ? out : ws->y, M, H, F, s->bn_f2);
    if (st == E3_OK && i == nl - 1) st = gemm_tmaps(&m.f2t, ws->h, F, s->L[i].w_2, ws->yt, M, H, F, s->bn_f2);
    if (st == E3_OK && i == nl - 1) st = gemm_tmaps(&m.f2t0, ws->h, F, s->L[i].w_2, ws->yt0, M, H, F, s->bn_f2);
  }
  if (st == E3_OK) st = attn_tmaps(&s->attn, ws->qkv, ws->ctx, B, S, H);
  if (st != E3_OK) {
    delete s;
    return st;
  }
  *out = s;
  return E3_OK;
}

// LLAMA decode split (R22-R24): per layer
//   n1 = RMSNorm1(x)                          rmsnorm_kernel
//   q | cache[k, v] = RoPE(n1 W_qkv^T)         decode GEMM, QKV_ROPE epilogue
//   ctx = attention(q, cache[0..pos])          attn_dec_kernel
//   h = x + ctx W_o^T                          decode GEMM (split-K), RESID
//   n2 = RMSNorm2(h)
//   a = SiLU(n2 W_gate^T) * (n2 W_up^T)        decode GEMM, SWIGLU
//   x' = h + a W_down^T                        decode GEMM (split-K), RESID
// ramp after layer l: nf = RMSNorm_f(x'), z = nf W_lm^T (LOGITS epilogue with
// per-tile softmax statistics), lm_decide; then the survivors are compacted.
static e3_status llama_run(e3_split *s, cudaStream_t st, const void *x_in, const int64_t *id_in,
                           const int32_t *n_valid_dev, int n_valid_host, const RingDst &dst, int32_t *n_surv_dev,
                           const e3_exits *ex) {
  const e3_split_desc &d = s->d;
  Workspace &ws = *s->ws;
  const int B = d.batch, H = d.hidden, F = d.ffn, V = d.num_labels;
  const int kvh = d.kv_heads > 0 ? d.kv_heads : d.heads;
  const int nqkv = (d.heads + 2 * kvh) * 128;
  const int nl = d.layer_end - d.layer_begin;
  e3_exits exits{};
  if (ex) exits = *ex;
  const void *cur = x_in;
  bool first_ramp = true;
  int ri = 0;
  e3_status r = E3_OK;
#define E3_RUN(expr)              \
  do {                            \
    r = (expr);                   \
    if (r != E3_OK) return r;     \
  } while (0)
  // algorithmic bytes (the path is HBM-bound): weights once per launch, the
  // valid tokens' activations, the KV positions 0..ctx of every valid token
  const double nv = n_valid_host, b2 = 2.0;
  const double kv_bytes = nv * d.heads * (double)(d.ctx_len + 1) * 128 * 2 * b2 / (d.heads / kvh);
  DecArgs base{};
  base.T = B;
  base.part = ws.dec_part;
  base.tickets = ws.dec_tickets;
  // O and down as split-K-by-4 partials reduced by the RMSNorm that follows
  // (reduce_rmsnorm_run), where the cluster split-K would run and the
  // following norm is the one-CTA-per-row kernel (bitwise the same results)
  const bool cta_norm = H >= 2048 && B <= 256;
  const bool fuse_o = cta_norm && dec_partial_ok(H, H, s->sms);
  const bool fuse_down = cta_norm && dec_partial_ok(H, F, s->sms);
  bool n1_ready = false;     // ws.x1 already holds this layer's RMSNorm1 (fused into the previous down)
  bool rnorm_ready = false;  // ws.x1 already holds the ramp's final norm of this layer's output
  for (int i = 0; i < nl; ++i) {
    const int l = d.layer_begin + i;
    const e3_layer_weights &L = s->L[i];
    auto &m = s->dmaps[i];
    void *out = (i % 2 == 0) ? ws.xa : ws.xb;
    if (!n1_ready) {
      ProfScope ps(PK_LN, st, 0, nv * H * 2 * b2);
      E3_RUN(rmsnorm_run(cur, L.ln1_g, ws.x1, B, H, d.norm_eps, st));
    }
    n1_ready = false;
    {
      DecArgs a = base;
      a.N = nqkv;
      a.K = H;
      a.max_contrib = s->mc_qkv;
      a.epi = E3_DEC_QKV_ROPE;
      a.Y = reinterpret_cast<__nv_bfloat16 *>(ws.qkv);
      a.ldo = d.heads * 128;
      a.nh = d.heads;
      a.kvh = kvh;
      a.max_ctx = s->kv.max_ctx;
      a.kc = reinterpret_cast<__nv_bfloat16 *>(s->kv_k[l]);
      a.vc = reinterpret_cast<__nv_bfloat16 *>(s->kv_v[l]);
      a.rope = ws.rope;
      a.ids = id_in;
      a.n_valid_dev = n_valid_dev;
      a.n_valid_host = n_valid_host;
      a.slot_of_id = s->kv.slot_of_id;
      a.id_cap = s->kv.id_capacity;
      a.pos_of_slot = s->kv.pos_of_slot;
      a.n_slots = s->kv.n_slots;
      a.err = ws.err;
      a.alive = first_ramp ? nullptr : ws.alive;   // after the split's first ramp: live rows only
      a.init_alive = first_ramp;
      ProfScope ps(PK_GEMM_QKV, st, 0, (double)nqkv * H * b2 + nv * (H + nqkv) * b2);
      E3_RUN(dec_run(m.qkv, a, s->sms, st));
    }
    {
      ProfScope ps(PK_ATTN, st, 0, kv_bytes);
      E3_RUN(attn_dec_run(ws.qkv, ws.ctx, s->kv_k[l], s->kv_v[l], id_in, n_valid_dev, n_valid_host,
                          s->kv.slot_of_id, s->kv.id_capacity, s->kv.pos_of_slot, s->kv.n_slots, B, d.heads, kvh,
                          s->kv.max_ctx,
                          st));
    }
    {
      DecArgs a = base;
      a.N = H;
      a.K = H;
      a.max_contrib = s->mc_o;
      a.epi = fuse_o ? E3_DEC_PARTIAL : E3_DEC_RESID;
      a.part_out = ws.dec_part;
      a.R = reinterpret_cast<const __nv_bfloat16 *>(cur);
      a.Y = reinterpret_cast<__nv_bfloat16 *>(ws.y);
      a.ldo = H;
      ProfScope ps(PK_GEMM_O, st, 0, (double)H * H * b2 + nv * 3 * H * b2);
      E3_RUN(dec_run(m.o, a, s->sms, st));
    }
    {
      ProfScope ps(PK_LN, st, 0, nv * H * 2 * b2);
      if (fuse_o) E3_RUN(reduce_rmsnorm_run(ws.dec_part, cur, ws.y, L.ln2_g, ws.x1, B, H, d.norm_eps, st));
      else E3_RUN(rmsnorm_run(ws.y, L.ln2_g, ws.x1, B, H, d.norm_eps, st));
    }
    {
      DecArgs a = base;
      a.N = F;
      a.K = H;
      a.max_contrib = s->mc_gu;
      a.epi = E3_DEC_SWIGLU;
      a.Y = reinterpret_cast<__nv_bfloat16 *>(ws.h);
      a.ldo = F;
      ProfScope ps(PK_GEMM_FFN1, st, 0, 2.0 * F * H * b2 + nv * (H + F) * b2);
      E3_RUN(dec_run(m.gu, a, s->sms, st));
    }
    {
      DecArgs a = base;
      a.N = H;
      a.K = F;
      a.max_contrib = s->mc_down;
      a.epi = fuse_down ? E3_DEC_PARTIAL : E3_DEC_RESID;
      a.part_out = ws.dec_part;
      a.R = reinterpret_cast<const __nv_bfloat16 *>(ws.y);
      a.Y = reinterpret_cast<__nv_bfloat16 *>(out);
      a.ldo = H;
      ProfScope ps(PK_GEMM_FFN2, st, 0, (double)F * H * b2 + nv * (F + 2 * H) * b2);
      E3_RUN(dec_run(m.down, a, s->sms, st));
    }
    if (fuse_down) {
      // the first norm that reads this layer's output: the ramp's final norm
      // (an evaluated ramp after layer l), else the next layer's RMSNorm1
      const void *g = nullptr;
      for (int rj = ri; rj < d.n_ramps && d.ramp_layer[rj] == l; ++rj)
        if (rj == d.n_ramps - 1 || d.inner == E3_INNER_EXACT) {
          g = s->R[rj].ln_g;
          rnorm_ready = true;
          break;
        }
      if (!g && i + 1 < nl) {
        g = s->L[i + 1].ln1_g;
        n1_ready = true;
      }
      ProfScope ps(PK_LN, st, 0, nv * H * 2 * b2);
      E3_RUN(reduce_rmsnorm_run(ws.dec_part, ws.y, out, g, ws.x1, B, H, d.norm_eps, st));
    }
    cur = out;
    while (ri < d.n_ramps && d.ramp_layer[ri] == l) {
      const bool last = (ri == d.n_ramps - 1);
      if (last || d.inner == E3_INNER_EXACT) {
        ProfScope ps(PK_RAMP, st, 0, (double)V * H * b2 + nv * (H * b2 + V * 4.0));
        if (!rnorm_ready) E3_RUN(rmsnorm_run(cur, s->R[ri].ln_g, ws.x1, B, H, d.norm_eps, st));
        rnorm_ready = false;
        DecArgs a = base;
        a.N = V;
        a.K = H;
        a.max_contrib = s->mc_lm;
        a.epi = E3_DEC_LOGITS;
        a.Z = exits.logits;
        a.ids = id_in;
        a.n_valid_dev = n_valid_dev;
        a.n_valid_host = n_valid_host;
        a.id_cap = exits.capacity;
        a.alive = ws.alive;
        a.init_alive = first_ramp;
        a.stats = ws.lm_stats;
        E3_RUN(dec_run(s->lm_maps[ri], a, s->sms, st));
        RampArgs ra{};
        ra.arch = d.arch;
        ra.id = id_in;
        ra.B = B;
        ra.S = 1;
        ra.H = H;
        ra.C = V;
        ra.test = d.test;
        ra.tau = d.tau[ri];
        ra.final_ramp = last && d.final_ramp;
        ra.layer = l;
        ra.ramp_index = d.ramp_index[ri];
        ra.alive = ws.alive;
        ra.init_alive = first_ramp;
        ra.n_valid_dev = n_valid_dev;
        ra.n_valid_host = n_valid_host;
        ra.ex = exits;
        ra.lm_stats = ws.lm_stats;
        ra.lm_tiles = dec_tiles(V, E3_DEC_LOGITS);
        ra.x = cur;   // the exiting rows -> ex.hidden (multi-step decode)
        E3_RUN(lm_decide_run(ra, st));
        first_ramp = false;
      }
      ++ri;
    }
  }
  {
    ProfScope ps(PK_COMPACT, st, 0, 0);
    E3_RUN(ln_compact_run(cur, id_in, ws.alive, B, 1, H, nullptr, nullptr, d.norm_eps, dst, n_surv_dev, s->sms,
                          st));
  }
#undef E3_RUN
  return E3_OK;
}

// FP32 mode (fp32_path.cu): the layer recipes of DESIGN.md R11 with fp32
// activations, LN2 materialised for every layer, the ramp on the post-LN
// rows, survivors copied (4-byte elements as pairs of 2-byte ones).
static e3_status f32_run(e3_split *s, cudaStream_t st, const void *x_in, const int64_t *id_in,
                         const int32_t *n_valid_dev, int n_valid_host, const RingDst &dst, int32_t *n_surv_dev,
                         const e3_exits *ex) {
  const e3_split_desc &d = s->d;
  Workspace &ws = *s->ws;
  const int B = d.batch, S = d.seq_len, H = d.hidden, F = d.ffn, M = B * S;
  const int nl = d.layer_end - d.layer_begin;
  const bool vit = d.arch == E3_ARCH_VIT;
  e3_exits exits{};
  if (ex) exits = *ex;
  auto *qkv = static_cast<float *>(ws.qkv), *ctx = static_cast<float *>(ws.ctx), *y = static_cast<float *>(ws.y);
  auto *x1 = static_cast<float *>(ws.x1), *hb = static_cast<float *>(ws.h);
  const float *cur = static_cast<const float *>(x_in);
  bool first_ramp = true;
  int ri = 0;
  e3_status r = E3_OK;
#define E3_RUN(expr)              \
  do {                            \
    r = (expr);                   \
    if (r != E3_OK) return r;     \
  } while (0)
  const bool llama = d.arch == E3_ARCH_LLAMA_DECODE;
  DecArgs da{};   // LLAMA: tokens, slots, positions (as the bf16 path's DecArgs)
  if (llama) {
    da.T = B;
    da.nh = d.heads;
    da.kvh = d.kv_heads > 0 ? d.kv_heads : d.heads;
    da.max_ctx = s->kv.max_ctx;
    da.ids = id_in;
    da.n_valid_dev = n_valid_dev;
    da.n_valid_host = n_valid_host;
    da.slot_of_id = s->kv.slot_of_id;
    da.id_cap = s->kv.id_capacity;
    da.pos_of_slot = s->kv.pos_of_slot;
    da.n_slots = s->kv.n_slots;
    da.err = ws.err;
  }
  const int nqkv = llama ? (da.nh + 2 * da.kvh) * 128 : 3 * H;
  for (int i = 0; i < nl; ++i) {
    const int l = d.layer_begin + i;
    const e3_layer_weights &L = s->L[i];
    float *out = static_cast<float *>((i % 2 == 0) ? ws.xa : ws.xb);
    if (llama) {   // R22: n1 = RMSNorm1(x); q, k = RoPE; h = x + attn W_o; x' = h + SwiGLU(RMSNorm2(h)) W_down
      DecArgs a = da;
      a.alive = first_ramp ? nullptr : ws.alive;   // exited rows append no K/V (R15)
      a.init_alive = first_ramp;
      E3_RUN(f32_rms_run(cur, L.ln1_g, x1, B, H, d.norm_eps, st));
      E3_RUN(f32_gemm_run(x1, H, L.w_qkv, nullptr, nullptr, qkv, B, nqkv, H, E3_EPI_BIAS, st));
      float *kc = static_cast<float *>(s->kv_k[l]), *vc = static_cast<float *>(s->kv_v[l]);
      E3_RUN(f32_rope_kv_run(qkv, ws.pool, kc, vc, ws.rope, a, st));
      E3_RUN(f32_attn_dec_run(ws.pool, ctx, kc, vc, a, st));
      E3_RUN(f32_gemm_run(ctx, H, L.w_o, nullptr, cur, y, B, H, H, E3_EPI_BIAS_RESID, st));
      E3_RUN(f32_rms_run(y, L.ln2_g, x1, B, H, d.norm_eps, st));
      E3_RUN(f32_gemm_run(x1, H, L.w_1, nullptr, nullptr, qkv, B, F, H, E3_EPI_BIAS, st));   // gate
      E3_RUN(f32_gemm_run(x1, H, L.w_3, nullptr, nullptr, hb, B, F, H, E3_EPI_BIAS, st));    // up
      E3_RUN(f32_swiglu_run(qkv, hb, hb, (size_t)B * F, st));
      E3_RUN(f32_gemm_run(hb, F, L.w_2, nullptr, y, out, B, H, F, E3_EPI_BIAS_RESID, st));
    } else if (vit) {   // n1 = LN1(x); y1 = x + attn(n1) W_o; n2 = LN2(y1); x2 = y1 + MLP(n2)
      E3_RUN(f32_ln_run(cur, L.ln1_g, L.ln1_b, x1, M, H, d.norm_eps, st));
      E3_RUN(f32_gemm_run(x1, H, L.w_qkv, L.b_qkv, nullptr, qkv, M, 3 * H, H, E3_EPI_BIAS, st));
      E3_RUN(f32_attn_run(qkv, ctx, B, S, H, st));
      E3_RUN(f32_gemm_run(ctx, H, L.w_o, L.b_o, cur, y, M, H, H, E3_EPI_BIAS_RESID, st));
      E3_RUN(f32_ln_run(y, L.ln2_g, L.ln2_b, x1, M, H, d.norm_eps, st));
      E3_RUN(f32_gemm_run(x1, H, L.w_1, L.b_1, nullptr, hb, M, F, H, E3_EPI_BIAS_GELU, st));
      E3_RUN(f32_gemm_run(hb, F, L.w_2, L.b_2, y, out, M, H, F, E3_EPI_BIAS_RESID, st));
    } else {     // x1 = LN1(x + attn(x) W_o); x2 = LN2(x1 + MLP(x1))
      E3_RUN(f32_gemm_run(cur, H, L.w_qkv, L.b_qkv, nullptr, qkv, M, 3 * H, H, E3_EPI_BIAS, st));
      E3_RUN(f32_attn_run(qkv, ctx, B, S, H, st));
      E3_RUN(f32_gemm_run(ctx, H, L.w_o, L.b_o, cur, y, M, H, H, E3_EPI_BIAS_RESID, st));
      E3_RUN(f32_ln_run(y, L.ln1_g, L.ln1_b, x1, M, H, d.norm_eps, st));
      E3_RUN(f32_gemm_run(x1, H, L.w_1, L.b_1, nullptr, hb, M, F, H, E3_EPI_BIAS_GELU, st));
      E3_RUN(f32_gemm_run(hb, F, L.w_2, L.b_2, x1, y, M, H, F, E3_EPI_BIAS_RESID, st));
      E3_RUN(f32_ln_run(y, L.ln2_g, L.ln2_b, out, M, H, d.norm_eps, st));
    }
    cur = out;
    while (ri < d.n_ramps && d.ramp_layer[ri] == l) {
      const bool last = (ri == d.n_ramps - 1);
      if (last || d.inner == E3_INNER_EXACT) {
        RampArgs a{};
        a.arch = d.arch;
        a.x = cur;
        a.id = id_in;
        a.B = B;
        a.S = S;
        a.H = H;
        a.C = d.num_labels;
        a.w = s->R[ri];
        a.test = d.test;
        a.tau = d.tau[ri];
        a.final_ramp = last && d.final_ramp;
        a.layer = l;
        a.ramp_index = d.ramp_index[ri];
        a.eps = d.norm_eps;
        a.alive = ws.alive;
        a.init_alive = first_ramp;
        a.n_valid_dev = n_valid_dev;
        a.n_valid_host = n_valid_host;
        a.ex = exits;
        // logits that do not fit shared memory next to two H rows: the
        // decode GEMMs' partial scratch, sized [B][C] for FP32 (llama_create)
        if ((2 * (size_t)H + a.C) * 4 > 200 * 1024) {
          if (!ws.dec_part || ws.part_elems < (size_t)B * a.C) {
            set_error("FP32 ramp: no logits scratch for C classes");
            return E3_EUNSUPPORTED;
          }
          a.pool_ws = ws.dec_part;
        }
        E3_RUN(f32_ramp_run(a, st));
        first_ramp = false;
      }
      ++ri;
    }
  }
  // survivors: fp32 rows copied byte for byte (stable order)
  E3_RUN(compact_run(cur, id_in, ws.alive, B, (int64_t)S * H * 4, dst, n_surv_dev, ws.ctr, s->sms, st));
#undef E3_RUN
  return E3_OK;
}

// Multi-step decode (e3_decode_run; R27): layer l of this split's
// K/V entries for the tokens of one chunk (<= B, ids_in [nv]) whose exit
// layer lies before l, computed from their exit hidden rows (ex->hidden):
// RMSNorm1_l -> the layer's QKV projection with the RoPE + KV-append epilogue
// (rows outside the mask write nothing; q goes to scratch).
e3_status llama_fill_layer(e3_split *s, int l, cudaStream_t st, const int64_t *ids_in, int nv, const e3_exits &ex,
                           int64_t *ids_buf) {
  const e3_split_desc &d = s->d;
  Workspace &ws = *s->ws;
  const int B = d.batch, H = d.hidden;
  const int i = l - d.layer_begin;
  const int kvh = d.kv_heads > 0 ? d.kv_heads : d.heads;
  const int nqkv = (d.heads + 2 * kvh) * 128;
  const int elem = d.dtype == E3_DTYPE_FP32 ? 4 : 2;
  const e3_layer_weights &L = s->L[i];
  e3_status r = fill_prep_run(ids_in, nv, B, ex.hidden, ex.capacity, ex.exit_layer, l, (int64_t)H * elem, ws.xa,
                              ids_buf, ws.alive, st);
  if (r != E3_OK) return r;
  DecArgs a{};
  a.T = B;
  a.nh = d.heads;
  a.kvh = kvh;
  a.max_ctx = s->kv.max_ctx;
  a.ids = ids_buf;
  a.n_valid_host = B;
  a.slot_of_id = s->kv.slot_of_id;
  a.id_cap = s->kv.id_capacity;
  a.pos_of_slot = s->kv.pos_of_slot;
  a.n_slots = s->kv.n_slots;
  a.err = ws.err;
  a.alive = ws.alive;
  a.init_alive = 0;
  if (d.dtype == E3_DTYPE_FP32) {
    auto *x1 = static_cast<float *>(ws.x1), *qkv = static_cast<float *>(ws.qkv);
    r = f32_rms_run(static_cast<const float *>(ws.xa), L.ln1_g, x1, B, H, d.norm_eps, st);
    if (r == E3_OK) r = f32_gemm_run(x1, H, L.w_qkv, nullptr, nullptr, qkv, B, nqkv, H, E3_EPI_BIAS, st);
    if (r == E3_OK)
      r = f32_rope_kv_run(qkv, ws.pool, static_cast<float *>(s->kv_k[l]), static_cast<float *>(s->kv_v[l]), ws.rope,
                          a, st);
    return r;
  }
  r = rmsnorm_run(ws.xa, L.ln1_g, ws.x1, B, H, d.norm_eps, st);
  if (r != E3_OK) return r;
  a.N = nqkv;
  a.K = H;
  a.max_contrib = s->mc_qkv;
  a.epi = E3_DEC_QKV_ROPE;
  a.Y = reinterpret_cast<__nv_bfloat16 *>(ws.qkv);
  a.ldo = d.heads * 128;
  a.kc = reinterpret_cast<__nv_bfloat16 *>(s->kv_k[l]);
  a.vc = reinterpret_cast<__nv_bfloat16 *>(s->kv_v[l]);
  a.rope = ws.rope;
  a.part = ws.dec_part;
  a.tickets = ws.dec_tickets;
  return dec_run(s->dmaps[i].qkv, a, s->sms, st);
}

static LnGemmArgs oln_args(const void *bias, const void *R, const void *g, const void *b, float eps, int M, int H,
                           int store_pre) {
  LnGemmArgs a{};
  a.bias = reinterpret_cast<const __nv_bfloat16 *>(bias);
  a.R = reinterpret_cast<const __nv_bfloat16 *>(R);
  a.g = reinterpret_cast<const __nv_bfloat16 *>(g);
  a.b = reinterpret_cast<const __nv_bfloat16 *>(b);
  a.eps = eps;
  a.M = M;
  a.N = H;
  a.K = H;
  a.store_pre = store_pre;
  return a;
}

bool split_tail_overlap(const e3_split *s) {
  static const bool off = getenv("E3_NO_TAIL_OVERLAP") != nullptr;
  const e3_split_desc &d = s->d;
  return !off && d.dtype == E3_DTYPE_BF16 && d.arch != E3_ARCH_LLAMA_DECODE && d.n_ramps >= 1 &&
         (d.n_ramps == 1 || d.inner == E3_INNER_DISABLED) && d.ramp_layer[d.n_ramps - 1] == d.layer_end - 1;
}

static e3_status split_run_body(e3_split *s, cudaStream_t st, const void *x_in, const int64_t *id_in,
                                const int32_t *n_valid_dev, int n_valid_host, const RingDst &dst,
                                int32_t *n_surv_dev, const e3_exits *ex, cudaStream_t tail_st, int par,
                                cudaEvent_t fork);

e3_status split_run_to(e3_split *s, cudaStream_t st, const void *x_in, const int64_t *id_in,
                       const int32_t *n_valid_dev, int n_valid_host, const RingDst &dst, int32_t *n_surv_dev,
                       const e3_exits *ex, cudaStream_t tail_st, int par, cudaEvent_t fork) {
  const bool ovl = tail_st && tail_st != st && fork && split_tail_overlap(s);
  e3_status r;
  if (s->d.dtype == E3_DTYPE_FP32)
    r = f32_run(s, st, x_in, id_in, n_valid_dev, n_valid_host, dst, n_surv_dev, ex);
  else if (s->d.arch == E3_ARCH_LLAMA_DECODE)
    r = llama_run(s, st, x_in, id_in, n_valid_dev, n_valid_host, dst, n_surv_dev, ex);
  else
    r = split_run_body(s, st, x_in, id_in, n_valid_dev, n_valid_host, dst, n_surv_dev, ex, ovl ? tail_st : st,
                       ovl ? (par & 1) : 0, fork);
  if (r == E3_OK && !ovl && tail_st && tail_st != st) {   // the run ends on tail_st all the same
    E3_CHECK_ARG(fork, "split_run_to: tail stream without a fork event");
    E3_CUDA_TRY(cudaEventRecord(fork, st));
    E3_CUDA_TRY(cudaStreamWaitEvent(tail_st, fork, 0));
  }
  return r;
}

static e3_status split_run_body(e3_split *s, cudaStream_t st, const void *x_in, const int64_t *id_in,
                                const int32_t *n_valid_dev, int n_valid_host, const RingDst &dst,
                                int32_t *n_surv_dev, const e3_exits *ex, cudaStream_t tst, int par,
                                cudaEvent_t fork) {
  const e3_split_desc &d = s->d;
  Workspace &ws = *s->ws;
  const int B = d.batch, S = d.seq_len, H = d.hidden, F = d.ffn, M = B * S;
  const int nl = d.layer_end - d.layer_begin;
  e3_exits exits{};
  if (ex) exits = *ex;
  const void *cur = x_in;
  bool first_ramp = true;
  int ri = 0;
  e3_status r = E3_OK;
#define E3_RUN(expr)              \
  do {                            \
    r = (expr);                   \
    if (r != E3_OK) return r;     \
  } while (0)
  // algorithmic work of this run counts valid rows only (padding is overhead)
  const double nvS = (double)n_valid_host * S;
  const double f_qkv = 2.0 * nvS * 3 * H * H, f_o = 2.0 * nvS * H * H, f_1 = 2.0 * nvS * F * H;
  const double f_att = 4.0 * n_valid_host * (double)S * S * H, b_ln = 2.0 * nvS * H * 2;
  const bool vit = d.arch == E3_ARCH_VIT;
  bool compacted = false;   // the last ramp's fused kernel also compacted the survivors
  // tst != st: the last ramp and the compaction run on tst (split_run_to)
  const bool ovl = tst != st;
  // The split's last layer writes a buffer of its own per run parity: the
  // run's tail (last ramp + compaction, on tst) still reads it while the next
  // run's layers execute, and a multi-layer split's earlier layers write
  // ws.y / xa / xb (BERT: every FFN2 writes ws.y -- a parity-0 tail reading
  // ws.y raced the next run's first FFN2: EE-BERT-large, 4-layer splits)
  void *const y_last = par ? ws.yt : ws.yt0;      // BERT: the last layer's pre-LN2 output
  uint8_t *const alive = par ? ws.alive_t : ws.alive;
  for (int i = 0; i < nl; ++i) {
    const int l = d.layer_begin + i;
    const e3_layer_weights &L = s->L[i];
    auto &m = s->maps[i];
    void *out = (i % 2 == 0) ? ws.xa : ws.xb;
    const bool last_layer = (i == nl - 1);
    if (vit) {
      // ViT pre-LN (R11): n1 = LN1(x); x1 = x + attn(n1 W_qkv) W_o;
      // n2 = LN2(x1); x2 = x1 + GELU(n2 W_1) W_2
      {
        ProfScope ps(PK_LN, st, 0, b_ln);
        E3_RUN(layernorm_run(cur, L.ln1_g, L.ln1_b, ws.x1, M, H, d.norm_eps, st));
      }
      {
        ProfScope ps(PK_GEMM_QKV, st, f_qkv, 0);
        E3_RUN(gemm_run(m.qkv, L.b_qkv, nullptr, M, 3 * H, H, E3_EPI_BIAS, s->sms, st));
      }
      {
        ProfScope ps(PK_ATTN, st, f_att, 0);
        E3_RUN(attn_run(s->attn, B, S, H, d.heads, ws.ctr + kAttnCtr, &ws.attn_parity, st));
      }
      if (s->use_oln) {
        LnGemmMaps lm = m.oln;
        if (i == 0) E3_RUN(make_tmap_2d(&lm.r, cur, (uint64_t)M, (uint64_t)H, (uint64_t)H, 128, 64));
        ProfScope ps(PK_GEMM_O, st, f_o, 0);
        E3_RUN(ln_gemm_run(lm, oln_args(L.b_o, cur, L.ln2_g, L.ln2_b, d.norm_eps, M, H, 1), st));
      } else {
        {
          ProfScope ps(PK_GEMM_O, st, f_o, 0);
          E3_RUN(gemm_run(m.o, L.b_o, cur, M, H, H, E3_EPI_BIAS_RESID, s->sms, st));
        }
        ProfScope ps(PK_LN, st, 0, b_ln);
        E3_RUN(layernorm_run(ws.y, L.ln2_g, L.ln2_b, ws.x1, M, H, d.norm_eps, st));
      }
      {
        ProfScope ps(PK_GEMM_FFN1, st, f_1, 0);
        E3_RUN(gemm_run(m.f1, L.b_1, nullptr, M, F, H, E3_EPI_BIAS_GELU, s->sms, st));
      }
      {
        ProfScope ps(PK_GEMM_FFN2, st, f_1, 0);
        E3_RUN(gemm_run(last_layer ? (par ? m.f2t : m.f2t0) : m.f2, L.b_2, ws.y, M, H, F, E3_EPI_BIAS_RESID, s->sms,
                        st));
      }
      cur = last_layer ? y_last : out;
    } else {
    {
      ProfScope ps(PK_GEMM_QKV, st, f_qkv, 0);
      if (i == 0) {
        GemmMaps g0;
        E3_RUN(gemm_tmaps(&g0, cur, H, L.w_qkv, ws.qkv, M, 3 * H, H, s->bn_qkv));
        if (!skip(PK_GEMM_QKV)) E3_RUN(gemm_run(g0, L.b_qkv, nullptr, M, 3 * H, H, E3_EPI_BIAS, s->sms, st));
      } else {
        if (!skip(PK_GEMM_QKV)) E3_RUN(gemm_run(m.qkv, L.b_qkv, nullptr, M, 3 * H, H, E3_EPI_BIAS, s->sms, st));
      }
    }
    {
      ProfScope ps(PK_ATTN, st, f_att, 0);
      if (!skip(PK_ATTN)) E3_RUN(attn_run(s->attn, B, S, H, d.heads, ws.ctr + kAttnCtr, &ws.attn_parity, st));
    }
    if (s->use_oln) {
      LnGemmMaps lm = m.oln;
      if (i == 0) E3_RUN(make_tmap_2d(&lm.r, cur, (uint64_t)M, (uint64_t)H, (uint64_t)H, 128, 64));
      ProfScope ps(PK_GEMM_O, st, f_o, 0);
      if (!skip(PK_GEMM_O)) E3_RUN(ln_gemm_run(lm, oln_args(L.b_o, cur, L.ln1_g, L.ln1_b, d.norm_eps, M, H, 0), st));
    } else {
      {
        ProfScope ps(PK_GEMM_O, st, f_o, 0);
        if (!skip(PK_GEMM_O)) E3_RUN(gemm_run(m.o, L.b_o, cur, M, H, H, E3_EPI_BIAS_RESID, s->sms, st));
      }
      ProfScope ps(PK_LN, st, 0, b_ln);
      if (!skip(PK_LN)) E3_RUN(layernorm_run(ws.y, L.ln1_g, L.ln1_b, ws.x1, M, H, d.norm_eps, st));
    }
    {
      ProfScope ps(PK_GEMM_FFN1, st, f_1, 0);
      if (!skip(PK_GEMM_FFN1)) E3_RUN(gemm_run(m.f1, L.b_1, nullptr, M, F, H, E3_EPI_BIAS_GELU, s->sms, st));
    }
    {
      ProfScope ps(PK_GEMM_FFN2, st, f_1, 0);
      if (!skip(PK_GEMM_FFN2))
        E3_RUN(gemm_run(last_layer ? (par ? m.f2t : m.f2t0) : m.f2, L.b_2, ws.x1, M, H, F, E3_EPI_BIAS_RESID, s->sms,
                        st));
    }
    // The split's last layer never materialises LN2: its ramp normalises the
    // CLS rows itself and the fused LN2 + compaction normalises only the
    // survivors, writing them straight to the destination.
    if (!last_layer) {
      ProfScope ps(PK_LN, st, 0, b_ln);
      if (!skip(PK_LN)) E3_RUN(layernorm_run(ws.y, L.ln2_g, L.ln2_b, out, M, H, d.norm_eps, st));
      cur = out;
    }
    }
    if (ovl && last_layer) {   // fork: the tail waits for the last layer only
      E3_CUDA_TRY(cudaEventRecord(fork, st));
      E3_CUDA_TRY(cudaStreamWaitEvent(tst, fork, 0));
    }
    while (ri < d.n_ramps && d.ramp_layer[ri] == l) {
      const bool last = (ri == d.n_ramps - 1);
      cudaStream_t rst = last ? tst : st;
      if (last || d.inner == E3_INNER_EXACT) {
        RampArgs a{};
        a.arch = d.arch;
        const bool pre_ln_rows = last_layer && !vit;   // BERT: the ramp applies LN2 itself
        a.x = pre_ln_rows ? y_last : cur;
        a.ln_g = pre_ln_rows ? L.ln2_g : nullptr;
        a.ln_b = pre_ln_rows ? L.ln2_b : nullptr;
        a.id = id_in;
        a.B = B;
        a.S = S;
        a.H = H;
        a.C = d.num_labels;
        a.w = s->R[ri];
        a.test = d.test;
        a.tau = d.tau[ri];
        a.final_ramp = last && d.final_ramp;
        a.layer = l;
        a.ramp_index = d.ramp_index[ri];
        a.eps = d.norm_eps;
        a.alive = alive;
        a.init_alive = first_ramp;
        a.n_valid_dev = n_valid_dev;
        a.n_valid_host = n_valid_host;
        a.ex = exits;
        a.pool_ws = ws.pool;
        a.done_ctr = ws.ctr;       // workspace counters (tickets, fused ramp + compaction)
        {
          // pooler weights + CLS rows + classifier weights (bytes); 2H^2 + 2HC per row (flops)
          const double hh = vit ? 0.0 : 2.0 * H * H;
          ProfScope ps(PK_RAMP, rst, (double)n_valid_host * (hh + 2.0 * H * d.num_labels),
                       hh + 2.0 * n_valid_host * H + 2.0 * d.num_labels * H);
          if (last && pre_ln_rows && !skip(PK_RAMP)) {
            // the split's last ramp and the LN2 + compaction of its survivors in one launch
            bool fused = false;
            E3_RUN(ramp_compact_run(a, ws.ctr, dst, n_surv_dev, s->sms, rst, &fused));
            compacted = fused;
          }
          if (!compacted && !skip(PK_RAMP)) E3_RUN(ramp_run(a, rst));
        }
        first_ramp = false;
      }
      ++ri;
    }
  }
  if (!compacted) {
    // survivors: LN2 of the last layer fused with the stable compaction
    // (bytes added once n_surv is known, in the pipeline)
    const e3_layer_weights &L = s->L[nl - 1];
    ProfScope ps(PK_COMPACT, tst, 0, 0);
    if (skip(PK_COMPACT)) return E3_OK;
    if (vit)   // pre-LN: the layer output is final, survivors are copied
      E3_RUN(ln_compact_run(cur, id_in, alive, B, S, H, nullptr, nullptr, d.norm_eps, dst, n_surv_dev, s->sms,
                            tst));
    else
      E3_RUN(ln_compact_run(y_last, id_in, alive, B, S, H, L.ln2_g, L.ln2_b, d.norm_eps, dst, n_surv_dev, s->sms,
                            tst));
  }
#undef E3_RUN
  return E3_OK;
}

}  // namespace e3

using namespace e3;

extern "C" {

e3_status e3_split_create(const e3_split_desc *d, const e3_weights *w, int device, e3_split **out) {
  return split_create_shared(d, w, device, nullptr, out);
}

e3_status e3_split_destroy(e3_split *s) {
  delete s;
  return E3_OK;
}

e3_status e3_split_run(e3_split *s, void *stream, const void *x_in, const int64_t *id_in, const int32_t *n_valid_dev,
                       void *x_out, int64_t *id_out, int32_t *n_surv_dev, const e3_exits *ex) {
  E3_CHECK_ARG(s, "null split");
  if (s->poisoned) {
    set_error("split handle poisoned by an earlier CUDA failure");
    return E3_ESTATE;
  }
  E3_CHECK_ARG(x_in && id_in && x_out && id_out && n_surv_dev, "null buffer");
  E3_CHECK_ARG(x_in != x_out, "x_in must not alias x_out");
  E3_CHECK_ARG(aligned16(x_in) && aligned16(x_out), "activations must be 16-byte aligned");
  const int B = s->d.batch;
  RingDst dst{};
  dst.rows = reinterpret_cast<uint8_t *>(x_out);
  dst.ids = id_out;
  dst.cap = B;
  int dev = 0;
  E3_CUDA_TRY(cudaGetDevice(&dev));
  if (dev != s->device) E3_CUDA_TRY(cudaSetDevice(s->device));
  e3_status r = split_run_to(s, reinterpret_cast<cudaStream_t>(stream), x_in, id_in, n_valid_dev, B, dst, n_surv_dev,
                             ex);
  if (r == E3_ECUDA) s->poisoned = true;
  if (dev != s->device) cudaSetDevice(dev);
  return r;
}

// ------------------------------------------------------------- e3_ops.h --

e3_status e3_op_gemm(void *stream, const void *A, int64_t lda, const void *W, const void *bias, const void *resid,
                     void *C, int32_t M, int32_t N, int32_t K, int32_t epilogue) {
  E3_CHECK_ARG(A && W && bias && C, "null buffer");
  E3_CHECK_ARG(epilogue >= 0 && epilogue <= 2, "bad epilogue");
  E3_CHECK_ARG(epilogue != E3_EPI_BIAS_RESID || resid, "residual epilogue needs resid");
  E3_CHECK_ARG(M > 0 && N > 0 && K > 0 && lda >= K, "bad dims");
  if (K % 128 || N % 64 || lda % 8 || !aligned16(A) || !aligned16(W) || !aligned16(C) || !aligned16(bias)) {
    set_error("e3_op_gemm: need K % 128 == 0, N % 64 == 0, lda % 8 == 0, 16-byte aligned pointers");
    return E3_EUNSUPPORTED;
  }
  int dev = 0;
  E3_CUDA_TRY(cudaGetDevice(&dev));
  const int sms = num_sms(dev);
  GemmMaps g;
  e3_status r = gemm_tmaps(&g, A, lda, W, C, M, N, K, gemm_pick_bn(M, N, K, sms, epilogue));
  if (r != E3_OK) return r;
  return gemm_run(g, bias, resid, M, N, K, epilogue, sms, reinterpret_cast<cudaStream_t>(stream));
}

e3_status e3_debug_timeline(void *dev_buf) {
  e3_status r = tl_set_gemm(dev_buf);
  if (r == E3_OK) r = tl_set_attn(dev_buf);
  if (r == E3_OK) r = tl_set_ln(dev_buf);
  if (r == E3_OK) r = tl_set_ramp(dev_buf);
  if (r == E3_OK) r = tl_set_compact(dev_buf);
  if (r == E3_OK) r = tl_set_gemm_ln(dev_buf);
  if (r == E3_OK) r = tl_set_dec(dev_buf);
  if (r == E3_OK) r = tl_set_llama(dev_buf);
  if (r == E3_OK) r = tl_set_rampc(dev_buf);
  return r;
}

e3_status e3_debug_gemm_trace(void *dev_buf) {
  const e3_status r = gemm_set_trace(dev_buf);
  return r != E3_OK ? r : attn_set_trace(dev_buf ? static_cast<uint64_t *>(dev_buf) + 148 * 16 * 6 : nullptr);
}

e3_status e3_op_dec_gemm(void *stream, const void *X, int32_t T, const void *W, const void *W2, int32_t N, int32_t K,
                         int32_t epilogue, const void *R, void *Y) {
  E3_CHECK_ARG(X && W && Y && N > 0 && K > 0, "bad arguments");
  E3_CHECK_ARG(epilogue >= 0 && epilogue <= 2, "bad epilogue");
  E3_CHECK_ARG(epilogue != 1 || R, "residual epilogue needs R");
  E3_CHECK_ARG(epilogue != 2 || W2, "SwiGLU epilogue needs W2");
  if ((T != 32 && T != 64 && T != 128) || K % 128 || (epilogue == 2 && N % 64) || !aligned16(X) || !aligned16(W) ||
      (W2 && !aligned16(W2))) {
    set_error("e3_op_dec_gemm: need T in {32,64,128}, K % 128 == 0, SwiGLU N % 64 == 0, aligned operands");
    return E3_EUNSUPPORTED;
  }
  int dev = 0;
  E3_CUDA_TRY(cudaGetDevice(&dev));
  const int sms = num_sms(dev);
  const int epi = epilogue == 0 ? E3_DEC_STORE : epilogue == 1 ? E3_DEC_RESID : E3_DEC_SWIGLU;
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  DecMaps m;
  e3_status r = dec_tmaps(&m, X, T, K, W, W2, N, epi);
  if (r != E3_OK) return r;
  const int tiles = dec_tiles(N, epi), mc = dec_max_contrib(N, K, epi, sms);
  // stream-K scratch kept per device across calls (the tickets reset
  // themselves at the end of every launch), so back-to-back calls are
  // kernel-to-kernel like the split path's: an allocation + memset + free
  // per call put ~6-10 us of graph nodes between the kernels.  Calls on one
  // device must not run concurrently on different streams.
  struct Scratch {
    float *part = nullptr;
    unsigned *tick = nullptr;
    size_t part_elems = 0, tick_elems = 0;
  };
  static std::mutex mu;
  static Scratch scr[64];
  E3_CHECK_ARG(dev >= 0 && dev < 64, "device index");
  std::lock_guard<std::mutex> lock(mu);
  Scratch &sc = scr[dev];
  const size_t pe = (size_t)tiles * mc * T * 128, te = (size_t)tiles;
  if (pe > sc.part_elems) {
    E3_CUDA_TRY(cudaStreamSynchronize(st));
    if (sc.part) cudaFree(sc.part);
    sc.part = nullptr;
    sc.part_elems = 0;
    E3_CUDA_TRY(cudaMalloc(reinterpret_cast<void **>(&sc.part), pe * 4));
    sc.part_elems = pe;
  }
  if (te > sc.tick_elems) {
    E3_CUDA_TRY(cudaStreamSynchronize(st));
    if (sc.tick) cudaFree(sc.tick);
    sc.tick = nullptr;
    sc.tick_elems = 0;
    E3_CUDA_TRY(cudaMalloc(reinterpret_cast<void **>(&sc.tick), te * 4));
    E3_CUDA_TRY(cudaMemset(sc.tick, 0, te * 4));
    sc.tick_elems = te;
  }
  float *part = sc.part;
  unsigned *tick = sc.tick;
  DecArgs a{};
  a.T = T;
  a.N = N;
  a.K = K;
  a.epi = epi;
  a.max_contrib = mc;
  a.R = reinterpret_cast<const __nv_bfloat16 *>(R);
  a.Y = reinterpret_cast<__nv_bfloat16 *>(Y);
  a.ldo = N;
  a.part = part;
  a.tickets = tick;
  return dec_run(m, a, sms, st);
}

e3_status e3_op_gemm_ln(void *stream, const void *A, const void *W, const void *bias, const void *R, const void *g,
                        const void *b, float eps, void *pre, void *out, int32_t M, int32_t N, int32_t K) {
  E3_CHECK_ARG(A && W && bias && R && g && b && out && M > 0, "bad arguments");
  if (!ln_gemm_supported(N, K) || !aligned16(A) || !aligned16(W) || !aligned16(R) || !aligned16(out) ||
      (pre && !aligned16(pre))) {
    set_error("e3_op_gemm_ln: need N in {128,256,384,512,640,768,1024}, K % 64 == 0, aligned buffers");
    return E3_EUNSUPPORTED;
  }
  LnGemmMaps m;
  e3_status r = ln_gemm_tmaps(&m, A, W, R, pre, out, M, N, K);
  if (r != E3_OK) return r;
  LnGemmArgs a = oln_args(bias, R, g, b, eps, M, N, pre != nullptr);
  a.K = K;
  return ln_gemm_run(m, a, reinterpret_cast<cudaStream_t>(stream));
}

e3_status e3_op_attention(void *stream, const void *qkv, void *ctx, int32_t B, int32_t S, int32_t H, int32_t heads) {
  E3_CHECK_ARG(qkv && ctx && B > 0 && S > 0 && H > 0 && heads > 0, "bad arguments");
  if (H / heads != 64 || H % heads || S > 256 || !aligned16(qkv) || !aligned16(ctx)) {
    set_error("e3_op_attention: need head_dim 64, S <= 256, aligned buffers");
    return E3_EUNSUPPORTED;
  }
  AttnMaps m;
  e3_status r = attn_tmaps(&m, qkv, ctx, B, S, H);
  if (r != E3_OK) return r;
  // the item counter: one per device, zeroed once (every launch leaves it
  // zero), so launches of this op on one device must be stream-ordered
  int dev = 0;
  E3_CUDA_TRY(cudaGetDevice(&dev));
  static unsigned *ctr_of[64] = {};
  static int par_of[64] = {};
  if (dev < 0 || dev >= 64) return E3_EINVAL;
  if (!ctr_of[dev]) {
    E3_CUDA_TRY(cudaMalloc(reinterpret_cast<void **>(&ctr_of[dev]), 4 * sizeof(unsigned)));
    E3_CUDA_TRY(cudaMemset(ctr_of[dev], 0, 4 * sizeof(unsigned)));
  }
  return attn_run(m, B, S, H, heads, ctr_of[dev], &par_of[dev], reinterpret_cast<cudaStream_t>(stream));
}

e3_status e3_op_layernorm(void *stream, const void *x, const void *g, const void *b, void *y, int32_t rows, int32_t H,
                          float eps) {
  E3_CHECK_ARG(x && g && b && y && rows > 0 && H > 0, "bad arguments");
  if (H % 8 || H > 4096 || !aligned16(x) || !aligned16(y) || !aligned16(g) || !aligned16(b)) {
    set_error("e3_op_layernorm: need H % 8 == 0, H <= 4096, aligned buffers");
    return E3_EUNSUPPORTED;
  }
  return layernorm_run(x, g, b, y, rows, H, eps, reinterpret_cast<cudaStream_t>(stream));
}

e3_status e3_op_ramp(void *stream, int32_t arch, const void *x, const int64_t *id, int32_t B, int32_t S, int32_t H,
                     int32_t C, const e3_ramp_weights *rw, int32_t test, float tau, int32_t final, int32_t layer,
                     int32_t ramp_index, float norm_eps, uint8_t *alive, int32_t init_alive,
                     const int32_t *n_valid_dev, const e3_exits *ex) {
  E3_CHECK_ARG(x && id && rw && alive && B > 0 && S > 0 && H > 0 && C > 0, "bad arguments");
  E3_CHECK_ARG(B <= 4096, "B > 4096");
  E3_CHECK_ARG(aligned16(x) && aligned16(arch == E3_ARCH_VIT ? rw->w_c : rw->w_p), "misaligned");
  int dev = 0;
  E3_CUDA_TRY(cudaGetDevice(&dev));
  // per-call scratch: pooled activations + ticket (freed asynchronously)
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  float *pool = nullptr;
  unsigned *ctr = nullptr;
  E3_CUDA_TRY(cudaMallocAsync(reinterpret_cast<void **>(&pool), (size_t)B * H * 4, st));
  const size_t nctr = (size_t)kCtrWords * sizeof(unsigned);
  E3_CUDA_TRY(cudaMallocAsync(reinterpret_cast<void **>(&ctr), nctr, st));
  E3_CUDA_TRY(cudaMemsetAsync(ctr, 0, nctr, st));
  RampArgs a{};
  a.arch = arch;
  a.x = x;
  a.id = id;
  a.B = B;
  a.S = S;
  a.H = H;
  a.C = C;
  a.w = *rw;
  a.test = test;
  a.tau = tau;
  a.final_ramp = final;
  a.layer = layer;
  a.ramp_index = ramp_index;
  a.eps = norm_eps;
  a.alive = alive;
  a.init_alive = init_alive;
  a.n_valid_dev = n_valid_dev;
  a.n_valid_host = B;
  if (ex) a.ex = *ex;
  a.pool_ws = pool;
  a.done_ctr = ctr;
  e3_status r = ramp_run(a, st);
  cudaFreeAsync(pool, st);
  cudaFreeAsync(ctr, st);
  return r;
}

e3_status e3_op_compact(void *stream, const void *x, const int64_t *id, const uint8_t *alive, int32_t B,
                        int64_t row_bytes, void *x_out, int64_t *id_out, int32_t *n_surv_dev) {
  E3_CHECK_ARG(x && id && alive && x_out && id_out && n_surv_dev && B > 0 && row_bytes > 0, "bad arguments");
  E3_CHECK_ARG(x != x_out, "x must not alias x_out");
  if (row_bytes % 16 || B > 4096 || !aligned16(x) || !aligned16(x_out)) {
    set_error("e3_op_compact: need row_bytes % 16 == 0, B <= 4096, aligned buffers");
    return E3_EUNSUPPORTED;
  }
  int dev = 0;
  E3_CUDA_TRY(cudaGetDevice(&dev));
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  unsigned *ctr = nullptr;
  E3_CUDA_TRY(cudaMallocAsync(reinterpret_cast<void **>(&ctr), sizeof(unsigned), st));
  E3_CUDA_TRY(cudaMemsetAsync(ctr, 0, sizeof(unsigned), st));
  RingDst dst{};
  dst.rows = reinterpret_cast<uint8_t *>(x_out);
  dst.ids = id_out;
  dst.cap = B;
  e3_status r = compact_run(x, id, alive, B, row_bytes, dst, n_surv_dev, ctr, num_sms(dev), st);
  cudaFreeAsync(ctr, st);
  return r;
}

}  // extern "C"
