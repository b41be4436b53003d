/*
 * e3.h — C ABI of the B200-native E3 early-exit split executor.
 *
 * E3 (Iyer et al., SOSP '24) keeps the batch size of an early-exit (EE) DNN
 * constant by cutting the model into splits at exit ramps, running each split
 * on full batches and re-batching the survivors of several upstream runs into
 * one full batch for the next split (§3.2 PAPER.md:755-768,
 * §3.3).  This library executes that data path on sm_100a:
 *
 *   e3_split_run   one split on one constant-size batch: encoder layers
 *                  (tcgen05 GEMMs + attention), fused exit ramp + threshold
 *                  test, stable compaction of the surviving rows;
 *   e3_rebatch     pop exactly B rows FIFO from a survivor queue (top-up);
 *   e3_pipeline_run  the whole split chain over n inputs with per-split
 *                  queues, on one GPU or one rank of a multi-GPU plan.
 *
 * Conventions (all calls):
 *   - Every call returns an e3_status and never throws or aborts.  On failure
 *     e3_last_error() returns a thread-local message.
 *   - Validation failures return E3_EINVAL / E3_EUNSUPPORTED before any
 *     launch (no side effects).  A CUDA/NCCL failure poisons the handle; later
 *     calls on it return E3_ESTATE.
 *   - "stream" arguments are cudaStream_t passed as void* (NULL = legacy
 *     default stream).  Calls marked ASYNC enqueue work and do not
 *     synchronise the host.
 *   - Activations are bf16, row-major [B, S, H] (token matrix [B*S, H]).
 *     Weights are bf16 in nn.Linear layout [out_features, in_features];
 *     biases / norm parameters are bf16 vectors.  Weight pointers are
 *     BORROWED device pointers that must outlive the handle.
 *   - Layer / ramp indices are 0-based ("ramp after layer 2" == layer 1).
 *   - Numerics: bf16 storage with fp32 accumulation at the points listed in
 *     DESIGN.md "Rounding contract"; ramp math in fp32.
 */
#ifndef E3_H_
#define E3_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define E3_MAX_RAMPS 64
#define E3_MAX_SPLITS 64
#define E3_COMM_ID_BYTES 128

typedef enum {
  E3_OK = 0,
  E3_EINVAL = 1,        /* bad argument (checked before any launch)            */
  E3_EUNSUPPORTED = 2,  /* not sm_100, or dims outside the kernels' tiling     */
  E3_ECUDA = 3,         /* CUDA runtime / launch failure (handle poisoned)     */
  E3_ENCCL = 4,         /* NCCL failure or NCCL unavailable                    */
  E3_ECAPACITY = 5,     /* a queue push would overflow the ring                */
  E3_ESTATE = 6         /* handle poisoned by an earlier failure               */
} e3_status;

typedef enum { E3_ARCH_BERT = 0, E3_ARCH_VIT = 1, E3_ARCH_LLAMA_DECODE = 2 } e3_arch;
typedef enum { E3_DTYPE_BF16 = 0, E3_DTYPE_FP32 = 1 } e3_dtype;
/* Exit criteria: confidence ("certainty level is higher
 * than a pre-defined threshold") -> exit iff max softmax > tau; entropy
 * ("entropy ... smaller than pre-defined threshold") -> exit iff H < tau
 * (natural log).  Comparisons are strict. */
typedef enum { E3_TEST_MAXPROB = 0, E3_TEST_ENTROPY = 1, E3_TEST_PATIENCE = 2 } e3_test;
/* E3_TEST_PATIENCE -- dependent exits, the counter-based criterion ("require
 * off-ramps classifiers to continuously generate identical predictions for
 * pre-defined times"; PABEE, §5.6; R26): at
 * every evaluated ramp the counter of an input becomes prev + 1 if its argmax
 * equals the previous ramp's, else 0; exit iff counter >= tau (the patience).
 * The per-input state lives in e3_exits.state (caller-zeroed per job) and
 * travels with the input across splits; single-rank plans only. */
/* Ramps inside a split (§3.4 exit-wrapper; §5.8.6):
 * EXACT evaluates every ramp (plan-independent results; rows that exit at an
 * inner ramp are recorded there and carried, masked, to the split end);
 * DISABLED evaluates only the split's last ramp. */
typedef enum { E3_INNER_EXACT = 0, E3_INNER_DISABLED = 1 } e3_inner;

const char *e3_last_error(void);
const char *e3_version(void);

/* ------------------------------------------------------------- split --- */

/* One split: layers [layer_begin, layer_end) of the EE model ending in a ramp
 * ("a contiguous block of encoder layers ending in an exit ramp").
 * ramp_layer[] lists the model ramps whose layer lies in the split, ascending;
 * the last must equal layer_end-1.  ramp_index[] are their model-wide ramp
 * numbers (used for stats).  final_ramp = 1 iff the split's last ramp is the
 * model's last ramp: "Remaining samples exit" there (Fig. 1). */
typedef struct e3_split_desc {
  int32_t arch;        /* e3_arch                                               */
  int32_t dtype;       /* e3_dtype (only BF16 is implemented)                   */
  int32_t hidden;      /* H   (multiple of 64)                                  */
  int32_t heads;       /* nh  (H / nh == 64)                                    */
  int32_t kv_heads;    /* LLAMA only                                            */
  int32_t ffn;         /* F   (multiple of 64)                                  */
  int32_t seq_len;     /* S   (<= 256)                                          */
  int32_t num_labels;  /* C   (ramp classes)                                    */
  int32_t ctx_len;     /* LLAMA only                                            */
  float norm_eps;
  int32_t layer_begin, layer_end;
  int32_t n_ramps;
  int32_t ramp_layer[E3_MAX_RAMPS];
  int32_t ramp_index[E3_MAX_RAMPS];
  float tau[E3_MAX_RAMPS];
  int32_t test;        /* e3_test                                               */
  int32_t final_ramp;
  int32_t inner;       /* e3_inner                                              */
  int32_t batch;       /* constant batch B (rows per run)                       */
  float rope_theta;    /* LLAMA: RoPE base (Llama-2 10000, Llama-3 500000);
                          <= 0 means 10000                                      */
} e3_split_desc;

typedef struct e3_layer_weights {
  const void *w_qkv, *b_qkv;   /* [3H,H], [3H]  rows: q | k | v, head-major   */
  const void *w_o, *b_o;       /* [H,H], [H]                                  */
  const void *ln1_g, *ln1_b;   /* [H]  (LLAMA: RMSNorm gain, ln1_b NULL)      */
  const void *w_1, *b_1;       /* [F,H], [F]   (LLAMA: W_gate, no bias)       */
  const void *w_2, *b_2;       /* [H,F], [H]   (LLAMA: W_down, no bias)       */
  const void *ln2_g, *ln2_b;   /* [H]                                         */
  const void *w_3;             /* LLAMA: W_up [F,H] (NULL otherwise)          */
} e3_layer_weights;

typedef struct e3_ramp_weights {
  const void *w_p, *b_p;       /* BERT pooler [H,H], [H]   */
  const void *w_c, *b_c;       /* classifier [C,H], [C] (LLAMA: LM head [V,H], */
                               /* b_c NULL)               */
  const void *ln_g, *ln_b;     /* VIT ramp LayerNorm [H] / LLAMA final RMSNorm */
                               /* gain [H] (ln_b NULL); NULL for BERT          */
} e3_ramp_weights;

/* LLAMA decode: the caller-owned KV cache (R22-R24).
 * Per layer l, k[l] and v[l] point to [n_slots][kv_heads][max_ctx][head_dim]
 * bf16 device arrays.  Token id i belongs to the sequence in slot
 * slot_of_id[i] (device int32, indexed by id < id_capacity) whose cached
 * length is pos_of_slot[slot] (device int32): the decode step writes the
 * token's k, v at that position of every layer it runs and attends over
 * positions 0..pos.  Nothing is written for layers a token skips (R24).
 * e3_pipeline_run never advances pos_of_slot (the caller does, between
 * steps); e3_decode_run advances it by one per step. */
typedef struct e3_kv_cache {
  int32_t n_layers;
  void *const *k;              /* host array of n_layers device pointers       */
  void *const *v;
  int32_t n_slots, max_ctx;
  const int32_t *slot_of_id;
  int64_t id_capacity;
  const int32_t *pos_of_slot;
} e3_kv_cache;

/* Model weights indexed by model-wide layer / ramp number. */
typedef struct e3_weights {
  int32_t n_layers;
  const e3_layer_weights *layer;
  int32_t n_ramps;
  const e3_ramp_weights *ramp;
  const e3_kv_cache *kv;       /* LLAMA only (NULL otherwise); borrowed        */
} e3_weights;

/* Exit records, written by the ramp kernel for every exiting valid row into
 * arrays INDEXED BY INPUT ID (ids must lie in [0, capacity)).  All device
 * memory, caller-owned; any pointer may be NULL to skip that field.
 * logits is [capacity, C] fp32.  n_exit and ramp_count (indexed by model
 * ramp number) are device counters that are incremented, never reset. */
typedef struct e3_exits {
  int32_t *exit_layer;
  int32_t *label;      /* argmax, lowest index on ties                        */
  float *conf;         /* the exit metric (max-prob or entropy)               */
  float *logits;
  int64_t capacity;
  int32_t *n_exit;
  int32_t *ramp_count;
  int32_t *state;      /* E3_TEST_PATIENCE: [capacity] per-input (label + 1) << 16 | counter,
                          zero before an input's first ramp; NULL otherwise            */
  void *hidden;        /* LLAMA: [capacity, H] (activation dtype) -- the hidden row each
                          token exited with (e3_decode_run fills the skipped layers'
                          K/V from it); NULL: not recorded                             */
  float *ramp_metric;  /* [capacity, ramp_metric_stride]: the exit metric of EVERY ramp a
                          row is evaluated at (model ramp index), exiting or not -- the
                          profile the exit-wrapper's ramp choice needs (planner); NULL: off */
  int32_t ramp_metric_stride;
} e3_exits;

typedef struct e3_split e3_split;

/* Validates the descriptor, checks the device is sm_100, borrows the weights
 * (layers [layer_begin, layer_end), the listed ramps) and allocates the
 * handle-owned workspace for batch B.  E3_EUNSUPPORTED for shapes outside the
 * kernels' tiling (H % 128, F % 128, head_dim != 64, S > 256, C > 16, B > 4096). */
e3_status e3_split_create(const e3_split_desc *d, const e3_weights *w, int device, e3_split **out);
e3_status e3_split_destroy(e3_split *s);

/* ASYNC.  Runs the split on one batch.
 *   x_in     [B,S,H] bf16 device, read-only; must not alias x_out
 *   id_in    [B] int64 device; rows >= n_valid are padding (never exit, never emitted)
 *   n_valid_dev  device int32 (NULL: all B rows valid)
 *   x_out    [B,S,H] bf16 device: survivors in stable (input) order
 *   id_out   [B] int64 device: survivor ids, same order
 *   n_surv_dev   device int32: number of survivors
 *   ex       exit records (may be NULL)
 * Conservation: exits recorded + n_surv == n_valid. */
e3_status e3_split_run(e3_split *s, void *stream, const void *x_in, const int64_t *id_in,
                       const int32_t *n_valid_dev, void *x_out, int64_t *id_out, int32_t *n_surv_dev,
                       const e3_exits *ex);

/* ------------------------------------------------------ queue / rebatch --- */

/* Device FIFO ring of survivor rows ("a queue that holds the partial
 * results") of row_bytes each (+ an int64 id per row),
 * cap_rows rows.  Owned by the handle. */
typedef struct e3_queue e3_queue;
e3_status e3_queue_create(int device, int64_t row_bytes, int32_t cap_rows, e3_queue **q);
e3_status e3_queue_destroy(e3_queue *q);
/* ASYNC.  Appends *n_dev rows (device count, <= max_rows) of rows[]/ids[] in
 * order.  If the ring would overflow nothing is written and the queue is
 * flagged: the next e3_queue_count / e3_rebatch returns E3_ECAPACITY. */
e3_status e3_queue_push(e3_queue *q, void *stream, const void *rows, const int64_t *ids, const int32_t *n_dev,
                        int32_t max_rows);
/* Synchronises `stream`-ordered work already enqueued on the queue's device
 * and returns the exact row count. */
e3_status e3_queue_count(e3_queue *q, int32_t *host_count);
/* Re-batching top-up ("combine the two outputs to obtain a
 * batch size of 16"; "multiple batches are fused"):
 * synchronises the stream, then if count >= B pops exactly B rows FIFO into
 * x_out/id_out, or if flush && count > 0 pops the remainder padded to B
 * (padding rows zero, id -1).  Never emits more than B rows.
 * *n_valid_dev (device) receives the valid count; *emitted (host) 1 or 0. */
e3_status e3_rebatch(e3_queue *q, void *stream, int32_t B, int32_t flush, void *x_out, int64_t *id_out,
                     int32_t *n_valid_dev, int32_t *emitted);

/* --------------------------------------------------------------- comm --- */

/* Inter-split transfer: "Tx is the communication
 * time for sending data from the end of a split to the next" (§3.2.1,
 * PAPER.md:887-903); split outputs "are then directed to the machines hosting
 * the next split" into "a queue that holds the partial results" (§3.3,
 * PAPER.md:962-972).  One process per GPU; the communicator is owned by the
 * library.
 *   NCCL      ncclSend / ncclRecv over NVLink, one 2-rank communicator per
 *             (sender, receiver) link split off the world communicator at
 *             e3_pipeline_create (NCCL is resolved at run time from the
 *             process's libnccl.so.2; E3_ENCCL if absent).
 *   LOOPBACK  every rank of the plan lives in THIS process on one device
 *             (tests and single-GPU runs of a multi-rank plan): a message is a
 *             device-to-device copy matched by a host-side hub, with the same
 *             ordering / EOS protocol as NCCL.
 *   P2P       reserved (fused compaction -> peer-ring stores); E3_EUNSUPPORTED. */
typedef enum { E3_TRANSPORT_NCCL = 0, E3_TRANSPORT_P2P = 1, E3_TRANSPORT_LOOPBACK = 2 } e3_transport;

typedef struct e3_comm e3_comm;
/* NCCL unique id, created on one rank and broadcast by the caller (e.g. over
 * a torch process group) to every rank before e3_comm_init. */
e3_status e3_comm_unique_id(uint8_t id[E3_COMM_ID_BYTES]);
/* Collective over `world` ranks: the NCCL world communicator of this rank on
 * `device`.  E3_ENCCL on any NCCL failure. */
e3_status e3_comm_init(const uint8_t id[E3_COMM_ID_BYTES], int rank, int world, int device, e3_comm **out);
/* LOOPBACK: `world` rank handles out[0..world-1] sharing one in-process hub on
 * `device`.  Each handle is used by one thread at a time. */
e3_status e3_comm_init_loopback(int world, int device, e3_comm **out);
e3_status e3_comm_rank(const e3_comm *c, int32_t *rank, int32_t *world);
/* Destroy every pipeline using the handle first. */
e3_status e3_comm_destroy(e3_comm *c);

/* ----------------------------------------------------------- pipeline --- */

#define E3_MAX_REPLICA_SLOTS 256

/* Split plan ("the apt number of splits ..., the number of resources to place
 * them, and the batch sizes to run the splits with"). */
typedef struct e3_plan {
  int32_t n_splits;
  e3_split_desc split[E3_MAX_SPLITS];  /* contiguous: split[s+1].layer_begin == split[s].layer_end;
                                          same model dims, batch and dtype in every split */
  int32_t lag;                         /* host look-behind: 0 serial, 1 (default)   */
  int32_t queue_cap_batches;           /* ring capacity per split in batches (>= 4) */
  int32_t trace;                       /* record dispatch order (e3_pipeline_trace) */
  /* Placement (multi-GPU; all zero = every split on the calling rank):
   * replicas[s] copies of split s; replica j of split s runs on comm rank
   * device_of[off(s) + j], off(s) = sum_{t<s} replicas[t].  The splits a rank
   * hosts must be contiguous and share one replica set (a STAGE); adjacent
   * stages use disjoint ranks.  Stage g's replica i sends its k-th output
   * batch to replica (i + k) mod r of stage g+1. */
  int32_t replicas[E3_MAX_SPLITS];
  int32_t device_of[E3_MAX_REPLICA_SLOTS];
  int32_t transport;                   /* e3_transport (ignored on one rank)        */
  int32_t deterministic;               /* 1: a receiver appends its senders' batches in
                                          round-robin sender order (exact batch
                                          composition); 0: in arrival order        */
} e3_plan;

typedef struct e3_stats {
  int64_t runs;
  int64_t batches[E3_MAX_SPLITS];
  int64_t valid_rows[E3_MAX_SPLITS];
  int64_t padded_rows[E3_MAX_SPLITS];
  int64_t rows_out[E3_MAX_SPLITS];
  int64_t host_waits;                  /* times the host blocked on a run          */
  double host_launch_ms;               /* host time spent issuing runs (launches)  */
  double host_sync_ms;                 /* host time spent waiting on run events    */
  int64_t msgs_sent, msgs_recv;        /* inter-stage data messages of this rank   */
  int64_t flushes[E3_MAX_SPLITS];      /* padded (flush) batches per split          */
} e3_stats;

typedef struct e3_pipeline e3_pipeline;
/* SPMD: every rank of the plan calls it with the same plan (c == NULL: one
 * rank, every split on `device` -- the paper's base formulation, "each GPU
 * executes the splits sequentially").  With a communicator
 * the rank creates only the splits it hosts (weights of other layers may be
 * NULL) and, for NCCL, one link communicator per (sender, receiver) pair of
 * adjacent stages (collective: all ranks must call).  `device` must equal the
 * communicator's device. */
e3_status e3_pipeline_create(const e3_plan *p, const e3_weights *w, int device, e3_comm *c, e3_pipeline **out);
e3_status e3_pipeline_destroy(e3_pipeline *pl);
/* Runs every input through the split chain until it exits.
 *   x    [n,S,H] activations (bf16, or fp32 for an FP32 plan), ids [n] int64
 *        (ids in [0, ex->capacity)).  Both may be DEVICE or HOST memory; host
 *        inputs are staged batch by batch on a copy stream (H2D copies
 *        overlap compute).  Multi-rank: ranks hosting split 0 pass their own
 *        share of the inputs, the others n = 0.
 *   ex   exit records (device arrays) of the inputs exiting on THIS rank.
 * Blocks until all of this rank's work is done (returns with the stream idle).
 * Split 0 takes inputs in order, B at a time; every split runs exactly B rows
 * per batch; the deepest split holding >= B queued rows runs first; a queue
 * is flushed (padded to B) only when nothing upstream of it can still
 * deliver rows -- for the first split of a stage, after every sender's
 * end-of-stream message.  Survivors of a stage's
 * last split travel to the next stage as fixed-size messages [n, flag | B ids
 * | B rows] (a rank's link buffers are reused only after the transfer
 * completed); the host loop never blocks on a transfer while it has a run to
 * issue. */
e3_status e3_pipeline_run(e3_pipeline *pl, void *stream, const void *x, const int64_t *ids, int64_t n,
                          const e3_exits *ex, e3_stats *st);
/* A plan truncated before the model's final ramp (single rank): like
 * e3_pipeline_run, the survivors of the plan's last split are appended in
 * dispatch order (stable within each run) to x_out / id_out (device,
 * capacity out_cap rows; E3_ECAPACITY beyond it) and *n_out (host) receives
 * their number. */
e3_status e3_pipeline_run_out(e3_pipeline *pl, void *stream, const void *x, const int64_t *ids, int64_t n,
                              const e3_exits *ex, e3_stats *st, void *x_out, int64_t *id_out, int64_t out_cap,
                              int64_t *n_out);
/* Multi-step greedy early-exit decode (LLAMA_DECODE plans, every split on
 * this rank; R27).  PAPER.md leaves the KV of
 * exited tokens open; here, CALM-style state propagation: for
 * step = 0 .. steps-1
 *   1. the n tokens run through the plan as in e3_pipeline_run (x [n, H],
 *      ids [n] device; each token its own sequence: slot_of_id[id] distinct);
 *   2. for every layer l after a token's exit layer, its K/V at its position
 *      are filled from the hidden row it exited with (ex->hidden, required):
 *      k = RoPE(RMSNorm1_l(h) W_k^l), v = RMSNorm1_l(h) W_v^l (the decode
 *      layer's own K/V arithmetic and storage points);
 *   3. tokens_out[step * n + i] = its label (argmax); x[i] <- embed[label]
 *      (embed [V, H] device, activation dtype); pos_of_slot[slot] += 1.
 * Blocks until done.  E3_EINVAL if a position would pass the cache
 * (max_ctx); st (optional) accumulates over the steps. */
e3_status e3_decode_run(e3_pipeline *pl, void *stream, void *x, const int64_t *ids, int64_t n, int32_t steps,
                        const void *embed, int32_t *tokens_out, const e3_exits *ex, e3_stats *st);

/* Dispatch order of the last run (plan.trace = 1): per run its split, valid
 * count and the B ids (padding = -1) into ids_out[run * B ...]. */
e3_status e3_pipeline_trace(e3_pipeline *pl, int32_t *split, int32_t *n_valid, int64_t *ids_out,
                            int64_t max_runs, int64_t *n_runs);

#ifdef __cplusplus
}
#endif
#endif /* E3_H_ */
