/*
 * abacus.h -- C ABI of the B200-native Abacus candidate-search library
 * (libabacus.so, built from paper_conf_sc_cui0czlzsmylg21_b200/csrc).
 *
 * What it computes: the data-parallel hot path of Abacus's headroom-based
 * query controller (Cui et al., "Enable Simultaneous DNN Services Based on
 * Deterministic Operator Overlap and Precise Latency Prediction", SC'21).
 * Citations are P:<line> into the paper text plus the section /
 * equation / figure; "reading cN" refers to DESIGN.md "Readings of the paper".
 *
 *   a1 headroom + order      Eq. 2, Eq. 3, sort
 *   a2 candidate enumeration operator groups
 *   a3 feature encoding      Fig. 8
 *   a4 predictor forward     MLP, 3 hidden layers of 32
 *   a5 mask + selection      largest group under the tightest headroom
 *   a6 cross-GPU combine     one NCCL collective (no counterpart in the paper)
 *   a7 decision assembly     drop mechanism
 *
 * Conventions (all entry points)
 *   - Return value: ABACUS_OK (0) or a negative ABACUS_E_* code.  On error no
 *     output is written and abacus_last_error(ctx) returns a message.  The
 *     decision OUTCOME is the separate field abacus_decision_t.status.
 *   - Ownership: the caller owns every buffer it passes.  Host structs are
 *     read during the call and never retained.  Device pointers must be
 *     allocations on the ctx's device.  The ctx owns its weight copies and a
 *     fixed scratch area allocated in abacus_create / abacus_load_predictor;
 *     no entry point allocates device memory on the hot path.
 *   - Streams: encode / predict / select are asynchronous on the given CUDA
 *     stream (NULL = the ctx's own stream).  abacus_search and
 *     abacus_search_grid block until the decision is in host memory.
 *   - Thread safety: none; use one ctx per host thread.
 *   - There is no CPU fallback: abacus_create fails with ABACUS_E_DEVICE on
 *     anything but an sm_100 device.
 *
 * Notation: N models (ids 1..N, Table 1 order, reading c6), L_m ops of model m
 * (1-based, inclusive ranges, reading c7), k co-located queries, K_MAX = 4,
 * D = N + 4*K_MAX feature width.
 */
#ifndef ABACUS_H
#define ABACUS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ABACUS_K_MAX 4
#define ABACUS_HIDDEN 32
#define ABACUS_ABI_VERSION 3
#define ABACUS_BATCH_MAX (1 << 20) /* decisions per abacus_search_batch call */
#define ABACUS_WHATIF_MAX (1 << 16) /* variants per abacus_search_whatif call */
#define ABACUS_TRAIN_MAX_BATCH 65536 /* samples per training step */

/* status codes */
enum {
    ABACUS_OK = 0,
    ABACUS_E_INVALID = -1,    /* bad argument (ranges, sizes, null pointers)        */
    ABACUS_E_DUP_MODEL = -2,  /* two queries/slots of one model (reading c9)        */
    ABACUS_E_NOT_LOADED = -3, /* no predictor loaded for the requested precision    */
    ABACUS_E_CUDA = -4,       /* CUDA runtime error                                 */
    ABACUS_E_NCCL = -5,       /* NCCL error                                         */
    ABACUS_E_DEVICE = -6      /* device is not sm_100 (no fallback exists)          */
};

/* predictor arithmetic (reading c16) */
enum {
    ABACUS_FP32 = 0, /* SIMT FFMA, fp32 weights and activations                     */
    ABACUS_BF16 = 1, /* tcgen05 kind::f16, fp32 accumulation in TMEM; bf16 operands */
                     /* for layers 2, 3 and the output (W3 split hi + lo, layer-2   */
                     /* and output weights hi only, hidden biases as hi + lo rows  */
                     /* of a bias K chunk, b4 in fp32); layer 1 of the fused search */
                     /* and of the D = 24 predictor enters through the fp16 operand */
                     /* of exact features / digits (1024 + v).  Error vs the fp64  */
                     /* oracle on config 5: max 8.1e-3 relative (DESIGN.md r2)      */
    ABACUS_FP16 = 2  /* tcgen05 kind::f16, fp16 operands with exact power-of-two    */
                     /* layer scaling; accumulation in TMEM is fp32 for the output  */
                     /* layer but F16 for hidden layers 2 and 3 (their biases are   */
                     /* added in f16 in the epilogue) and, in the search calls, for */
                     /* layer 1 (fp32 in abacus_predict_batch); the output bias is  */
                     /* added in fp32.  Error vs the fp64 oracle: predict_batch on  */
                     /* config 5 max 1.5e-3 relative, y(t*) of config-1 searches    */
                     /* max 6.5e-4 (reading r2)                           */
};

/* candidate space of abacus_search (reading c13) */
enum {
    ABACUS_SPACE_GRID = 0,  /* every end-op combination (exhaustive)                */
    ABACUS_SPACE_CHAIN = 1, /* the paper's chain: prefix of full queries, then one  */
                            /* partial query                          */
    ABACUS_SPACE_AUTO = 2   /* GRID if |GRID| <= grid_budget, else CHAIN            */
};

/* decision outcome */
enum {
    ABACUS_DECIDE_OK = 0,   /* end_op[] holds the group                             */
    ABACUS_DECIDE_DROP = 1, /* the critical query alone exceeds H: drop it          */
                            /* (reading c14)                           */
    ABACUS_DECIDE_NONE = 2  /* sweep only: no candidate fits under H                */
};

typedef struct abacus_ctx abacus_ctx; /* opaque; one per device per host thread */

/* One service of a candidate grid.  Digit d of the slot: allow_absent ?
 * (d == 0 -> absent, else ope = end_lo + d - 1) : ope = end_lo + d; radix
 * rho = allow_absent + end_hi - end_lo + 1.  seqlen is 0 for non-Bert models
 * (reading c8). */
typedef struct {
    int32_t model_id;     /* 1..N                                          */
    int32_t start_op;     /* ops: first op of the range, 1-based           */
    int32_t batch;        /* bs >= 1                                       */
    int32_t seqlen;       /* >= 0                                          */
    int32_t end_lo, end_hi; /* candidate ope range, start_op <= lo <= hi <= L */
    int32_t allow_absent; /* 0 or 1                                        */
} abacus_slot_t;

/* A candidate grid: slots in priority (headroom) order.  Candidate index
 * t in [0, T), T = prod rho_j < 2^40, mixed radix with the LAST slot fastest. */
typedef struct {
    int32_t k;
    abacus_slot_t slot[ABACUS_K_MAX];
} abacus_grid_t;

/* An explicit operator group (one row of config-5 instance samples). */
typedef struct {
    int32_t k;                       /* present models, 0..K_MAX            */
    struct {
        int32_t model_id, ops, ope, batch, seqlen;
    } slot[ABACUS_K_MAX];            /* any order; encoded by model id       */
} abacus_group_t;

/* One what-if variant of a grid (abacus_search_whatif): the batch size and
 * sequence length of every grid slot (slot j uses batch[j], seqlen[j]; the
 * grid's own values are replaced). */
typedef struct {
    int32_t batch[ABACUS_K_MAX];  /* >= 1 */
    int32_t seqlen[ABACUS_K_MAX]; /* >= 0 (0 for non-Bert models, reading c8) */
} abacus_variant_t;

/* One active query (Fig. 4, Eq. 2). */
typedef struct {
    int32_t model_id; /* 1..N                                  */
    int32_t next_op;  /* s: first op not yet run, 1..L         */
    int32_t batch;
    int32_t seqlen;
    double qos_ms;     /* T_QoS                                 */
    double t_start_ms; /* T_start                               */
} abacus_query_t;

typedef struct {
    int32_t status;     /* ABACUS_DECIDE_*                                         */
    int32_t critical;   /* index into the caller's query array (sweeps: 0)         */
    int32_t order[4];   /* headroom order as caller indices (sweeps: identity)     */
    int32_t end_op[4];  /* per caller query / grid slot: ope, 0 = not in the group */
    uint64_t key;       /* ((sum_n + 1) << 40) | index, 0 = nothing fits           */
    uint64_t index;     /* t* (GRID / sweep) or u* (CHAIN)                         */
    uint64_t evaluated; /* candidates evaluated (sweep: over all ranks)            */
    int32_t total_ops;  /* sum over the group of (ope - ops + 1)                   */
    float headroom_ms;  /* H, the fp32 threshold compared against                  */
    float pred_ms;      /* predicted latency of the chosen group (feeds Eq. 3)     */
    float pred_critical_only_ms; /* y of the critical query alone (drop test)     */
} abacus_decision_t;

/* ------------------------------------------------------------------------ */
/* Context                                                                   */
/* ------------------------------------------------------------------------ */

/* Create a ctx on CUDA device `device` for a registry of n_models models with
 * ops_per_model[m-1] = L_m (host array, copied).  k_max must be 4.
 * Errors: E_INVALID (n_models < 1 or > 64, L_m < 1 or > 32767, k_max != 4),
 * E_DEVICE (not sm_100), E_CUDA.  *out is written only on success. */
int abacus_create(int device, int32_t n_models, const int32_t* ops_per_model, int32_t k_max,
                  abacus_ctx** out);

/* Free the ctx and everything it owns (NULL is a no-op). */
void abacus_destroy(abacus_ctx* ctx);

/* Last error message of this ctx ("" if none); valid until the next call. */
const char* abacus_last_error(const abacus_ctx* ctx);

/* Load predictor weights (host, fp32, little endian), row-major [out][in]:
 *   W1[32][D] b1[32] W2[32][32] b2[32] W3[32][32] b3[32] w4[32] b4
 * n_params must be 32*D + 2*32*32 + 4*32 + 1 (2945 for D = 24).
 * `precision` selects the arithmetic later calls use (ABACUS_FP32/BF16/FP16);
 * the fp32 copy is always kept.  The ctx converts once at load time (RNE) and
 * owns the device copies.  Errors: E_INVALID (size / precision / non-finite). */
int abacus_load_predictor(abacus_ctx* ctx, const float* params, size_t n_params, int precision);

/* ------------------------------------------------------------------------ */
/* Building blocks (asynchronous on `stream`)                                */
/* ------------------------------------------------------------------------ */

/* a2 + a3: encode candidates t in [first, first+count) of `grid` (host struct)
 * into d_features (device, int16, count x D row-major, 16-byte aligned) per
 * Fig. 8: x[m-1] = 1 per present model; present models in
 * ascending id fill x[N+4p .. N+4p+3] = (ops, ope, bs, seqlen); zeros
 * elsewhere.  Errors: E_INVALID (grid validation as in abacus_search_grid,
 * first + count > T), E_DUP_MODEL. */
int abacus_encode_candidates(abacus_ctx* ctx, const abacus_grid_t* grid, uint64_t first, uint64_t count,
                             int16_t* d_features, void* stream);

/* a3 for explicit groups: d_groups (device, count records) -> d_features
 * (device, count x D).  A group with an invalid or duplicate model id is
 * encoded as all zeros and counted in *d_bad (device uint32, accumulated;
 * may be NULL). */
int abacus_encode_groups(abacus_ctx* ctx, const abacus_group_t* d_groups, uint64_t count,
                         int16_t* d_features, uint32_t* d_bad, void* stream);

/* a4: y = MLP(x) for count feature rows (device int16, count x D) into
 * d_latency_ms (device fp32, count), with the loaded precision.
 * Errors: E_NOT_LOADED, E_INVALID. */
int abacus_predict_batch(abacus_ctx* ctx, const int16_t* d_features, uint64_t count, float* d_latency_ms,
                         void* stream);

/* a5: fold candidates t in [first, first+count) of `grid` with predicted
 * latencies d_latency_ms[t - first] into the running max key *d_best_key
 * (device, in/out, initialise to 0): key(t) = ((sum_n + 1) << 40) | t over
 * y(t) <= headroom_ms (inclusive, readings c11/c12). */
int abacus_select_group(abacus_ctx* ctx, const abacus_grid_t* grid, uint64_t first, uint64_t count,
                        const float* d_latency_ms, float headroom_ms, unsigned long long* d_best_key,
                        void* stream);

/* ------------------------------------------------------------------------ */
/* Training the predictor                          */
/* ------------------------------------------------------------------------ */
/* The paper trains the MLP on instance-based samples (Fig. 9)
 * and measures MAPE (Eq. 1) but states no training procedure.
 * Readings (DESIGN.md t1-t3): loss = mean over the minibatch of
 * (y_pred / y_true - 1)^2; Adam with bias correction; the learning rate is
 * given per call.  All arithmetic is fp32 on the device. */
typedef struct {
    float beta1, beta2, eps; /* e.g. 0.9, 0.999, 1e-8 */
} abacus_adam_t;

/* Start (or restart) training from `params` (host, fp32, the
 * abacus_load_predictor layout): copies them to the ctx's training state and
 * zeroes the Adam moments and step counter.  Blocking.  Errors: E_INVALID
 * (size, non-finite values, hyper-parameters), E_CUDA. */
int abacus_train_begin(abacus_ctx* ctx, const float* params, size_t n_params, const abacus_adam_t* opt);

/* One Adam step on a minibatch: d_features (device int16, count x D, Fig. 8
 * rows as for abacus_predict_batch), d_latency_ms (device fp32, count, > 0).
 * 1 <= count <= ABACUS_TRAIN_MAX_BATCH.  d_grad (device fp32, n_params, may
 * be NULL) receives the minibatch gradient.  Async on `stream`.
 * Errors: E_NOT_LOADED (no abacus_train_begin), E_INVALID, E_CUDA. */
int abacus_train_step(abacus_ctx* ctx, const int16_t* d_features, const float* d_latency_ms, uint64_t count,
                      float lr, float* d_grad, void* stream);

/* Consecutive minibatches of `batch` rows (the last may be shorter), one
 * Adam step each, learning rate lr.  d_losses (device fp32, one per step,
 * may be NULL) receives each step's loss.  Async on `stream`. */
int abacus_train_epoch(abacus_ctx* ctx, const int16_t* d_features, const float* d_latency_ms, uint64_t count,
                       uint32_t batch, float lr, float* d_losses, void* stream);

/* Blocking: copy the current parameters to params_out (host, n_params) and,
 * if last_loss != NULL, the last step's loss.  Pass them to
 * abacus_load_predictor to search with the trained predictor. */
int abacus_train_params(abacus_ctx* ctx, float* params_out, float* last_loss);

/* ------------------------------------------------------------------------ */
/* Fused search (blocking)                                                   */
/* ------------------------------------------------------------------------ */

/* a1..a7 for one scheduling round (P:630-753 steps 1-2, §6.2-6.3):
 * h_i = qos_i - (now_ms - t_start_i) - inflight_pred_ms (Eq. 2 + Eq. 3, c15);
 * order ascending by (h, model id) (c10); H = (float)h_critical; critical
 * query fully included; other queries contribute ope in
 * [next_op, L] or are absent; candidate space per `space` / grid_budget;
 * result = largest feasible group (max sum_n, ties to lower-headroom queries,
 * c12); DROP iff y(critical alone) > H (c14).  q: host array of k queries
 * (1 <= k <= 4).  out: host.  Errors: E_INVALID, E_DUP_MODEL, E_NOT_LOADED,
 * E_CUDA. */
int abacus_search(abacus_ctx* ctx, const abacus_query_t* q, int32_t k, double now_ms, double inflight_pred_ms,
                  int32_t space, uint64_t grid_budget, abacus_decision_t* out);

/* Many independent scheduling rounds in one call (
 * the paper runs one round at a time): decision i is
 * abacus_search(q + 4 i, k[i], now_ms[i], inflight_pred_ms[i], space,
 * grid_budget) -- bit for bit when every round of the batch takes the same
 * layer-1 layout (every end-op range of <= 1,025 options, always true for
 * the paper's registry, L <= 471); a batch mixing wider rounds runs the split
 * layout for all of them, and the narrow rounds are then within the oracle's
 * acceptance window (reading c18) rather than bit-identical.  q: host array of 4 n query records (decision i uses
 * q[4i .. 4i + k[i] - 1]; the rest are ignored); k, now_ms,
 * inflight_pred_ms: host arrays of n; out: host array of n decisions.
 * 1 <= n <= ABACUS_BATCH_MAX.  fp16 / bf16: one batched tensor-core launch
 * (plus a decode kernel) for all n; fp32: one fused launch per decision.
 * The ctx grows its batch buffers on the first call with a larger n.
 * Errors: as abacus_search (the message names the failing decision; no
 * output is written on error). */
int abacus_search_batch(abacus_ctx* ctx, const abacus_query_t* q, const int32_t* k, const double* now_ms,
                        const double* inflight_pred_ms, int32_t n, int32_t space, uint64_t grid_budget,
                        abacus_decision_t* out);

/* The paper's multi-way search (§7.7)
 * for one scheduling round: same a1 step as abacus_search; candidates are the
 * CHAIN.  Round 1 is one batched prediction of u = 0 (drop test) and of every
 * block end (queries fully added, "between queries"); each later round
 * predicts `ways` evenly spaced points of the open interval (last fit, first
 * miss) inside the next query's operators (reading c17).  The result is the
 * last fitting chain position; it equals the exhaustive CHAIN result whenever
 * the prediction is monotone along the chain.  Predictions use the fp32
 * arithmetic.  out->evaluated = candidates predicted; *rounds_out (may be
 * NULL) = batched rounds.  1 <= ways <= 128.  Errors as abacus_search. */
int abacus_search_mway(abacus_ctx* ctx, const abacus_query_t* q, int32_t k, double now_ms, double inflight_pred_ms,
                       int32_t ways, abacus_decision_t* out, int32_t* rounds_out);

/* a2..a6 over a sweep grid: candidates t in [first, first+count) of `grid`
 * (host) under `headroom_ms`; this rank's shard.  With nccl_comm != NULL
 * (an ncclComm_t on this device, e.g. from abacus_nccl_comm_init, or a peer
 * communicator from abacus_peer_comm_init: the combine then runs inside the
 * search kernel) the per-rank results are combined so every rank returns
 * the same global decision (status OK or NONE, end_op per slot, pred_ms of
 * t*, evaluated summed over ranks, pred_critical_only_ms = y(index 0) from
 * the rank whose shard holds index 0; see abacus_combine_decisions).
 * Without a communicator pred_critical_only_ms = y(index 0) if
 * first == 0 < count, else NaN.  Validation: 1 <= k <= 4, model ids in
 * [1, N] and distinct, 1 <= start_op <= end_lo <= end_hi <= L, batch >= 1,
 * seqlen >= 0, T < 2^40, max sum_n + 1 < 2^24.  Errors: E_INVALID,
 * E_DUP_MODEL, E_NOT_LOADED, E_CUDA, E_NCCL. */
int abacus_search_grid(abacus_ctx* ctx, const abacus_grid_t* grid, float headroom_ms, uint64_t first,
                       uint64_t count, void* nccl_comm, abacus_decision_t* out);

/* What-if sweep (batch size and sequence length as
 * swept grid dimensions; the paper: "the batch size of query processing is
 * determined by the upper-level load balancer at runtime" and inputs vary in
 * length).  The candidates are every (variant v, end-op candidate
 * t) with v in [0, n_var), t in [0, T) of `grid` (host) whose slots take
 * variant v's batch sizes and sequence lengths (Fig.-8 features);
 * their index is v * T + t (the variant is the most significant digit, so
 * among groups of equal size the later variant wins, reading c12).
 * per_variant (host, n_var, may be NULL): variant v's own sweep decision,
 * exactly abacus_search_grid(variant grid v, headroom_ms, 0, T, NULL).
 * best (host, may be NULL): the largest feasible group over all variants --
 * key ((sum_n + 1) << 40) | (v T + t), index v T + t, end_op / pred_ms /
 * total_ops of that candidate, evaluated n_var T, pred_critical_only_ms =
 * y(index 0) of variant 0; status OK or NONE.  *best_variant (may be NULL)
 * = its v, -1 if nothing fits.  1 <= n_var <= ABACUS_WHATIF_MAX and
 * n_var T < 2^40.  Tensor precisions with T < 2^24: one batched launch for
 * all variants (each variant a plan of the NEXT-4 batch kernel); fp32, or
 * T >= 2^24: one fused search launch per variant.  Blocking.  Errors: as abacus_search_grid, plus E_INVALID for
 * a variant's batch outside [1, 32767] or seqlen outside [0, 32767]. */
int abacus_search_whatif(abacus_ctx* ctx, const abacus_grid_t* grid, const abacus_variant_t* variants,
                         int32_t n_var, float headroom_ms, abacus_decision_t* per_variant,
                         abacus_decision_t* best, int32_t* best_variant);

/* Per-decision sharded search (the paper's search is
 * single-node): the decision of abacus_search(q, k, now_ms,
 * inflight_pred_ms, space, grid_budget), computed by all ranks of `nccl_comm`
 * together.  Every rank must pass the same arguments.  Each rank runs a1
 * itself (deterministic: same order and H everywhere); a GRID decision's
 * index space [0, T) is split into contiguous shards
 * [floor(rT/G), floor((r+1)T/G)) over the G ranks, each rank searches its
 * shard with the fused kernel, and one ncclAllGather of the per-rank records
 * plus a 1-thread combine kernel (max key; y(0) for the drop test from the
 * rank whose shard holds index 0) gives every rank the same decision.
 * CHAIN decisions (incl. AUTO over the budget) are searched whole on every
 * rank with no collective.  nccl_comm == NULL: exactly abacus_search.
 * out->evaluated counts the candidates of all ranks.  Blocking.
 * Errors: as abacus_search, plus E_NCCL. */
int abacus_search_sharded(abacus_ctx* ctx, const abacus_query_t* q, int32_t k, double now_ms,
                          double inflight_pred_ms, int32_t space, uint64_t grid_budget, void* nccl_comm,
                          abacus_decision_t* out);

/* The cross-GPU combine step (a6) on the host, no ctx and no device needed:
 * per_rank[r] (host, nranks records, rank order) is rank r's
 * abacus_search_grid result without a communicator over shard r of a
 * contiguous partition of one grid under one headroom (status OK or NONE;
 * pred_critical_only_ms is NaN unless the shard holds index 0).  *out =
 * the global decision: the max key with its index, end_op, total_ops and
 * pred_ms; evaluated summed; pred_critical_only_ms from the first record
 * that holds index 0; status OK / NONE.  drop_test != 0 additionally applies
 * the decision drop rule of abacus_search (reading c14): status
 * DROP iff !(pred_critical_only_ms <= headroom_ms), then pred_ms = that
 * value, end_op and total_ops zero.  The device combine of
 * abacus_search_grid / abacus_search_sharded runs the same function.
 * Errors: E_INVALID (NULL, nranks outside [1, 64], headroom_ms differing
 * between records, status other than OK/NONE, key inconsistent with status). */
int abacus_combine_decisions(const abacus_decision_t* per_rank, int32_t nranks, int32_t drop_test,
                             abacus_decision_t* out);

/* ------------------------------------------------------------------------ */
/* NCCL bootstrap helpers (multi-GPU sweeps; one process per GPU)            */
/* ------------------------------------------------------------------------ */

/* 128-byte ncclUniqueId into `id128` (host).  Call on one rank, broadcast the
 * bytes (e.g. with torch.distributed), then abacus_nccl_comm_init on all. */
int abacus_nccl_unique_id(uint8_t* id128);
/* Create an ncclComm_t for (nranks, rank) on the ctx's device; *comm_out
 * receives it (owned by the caller; free with abacus_nccl_comm_destroy). */
int abacus_nccl_comm_init(abacus_ctx* ctx, int32_t nranks, int32_t rank, const uint8_t* id128,
                          void** comm_out);
void abacus_nccl_comm_destroy(void* comm);

/* ------------------------------------------------------------------------ */
/* a6 over peer memory: the combine inside the search kernel                 */
/* ------------------------------------------------------------------------ */
/* Instead of an ncclComm_t, abacus_search_grid and abacus_search_sharded
 * accept a peer communicator from abacus_peer_comm_init.  Each rank owns a
 * device mailbox of 2 x ABACUS_PEER_MAX tagged 64-byte records (two banks by
 * launch parity).  The last CTA of
 * a rank's fused search writes its 56-byte result into slot `rank` of every
 * rank's mailbox (peer stores: NVLink between GPUs, plain stores between
 * ctxs of one device), then waits in its own mailbox for every rank's record
 * of the same launch and combines them exactly as the NCCL path does (max
 * key, evaluated summed, y(0) from the lowest rank that holds index 0) -- no
 * collective launch, no finalize kernel.  Every rank must make the same
 * sequence of peer-combined calls (the launches are matched by a counter).
 * A rank whose record does not arrive within ABACUS_PEER_TIMEOUT_MS
 * milliseconds (environment, default 10000) fails the call with E_NCCL.
 * Ranks in one process may share a device (tests); ranks in different
 * processes exchange CUDA IPC handles. */
#define ABACUS_PEER_MAX 32   /* ranks per peer communicator */
#define ABACUS_PEER_BLOB 128 /* bytes of an exported mailbox description */

/* Allocate this ctx's mailbox (first call) and describe it in `blob`
 * (host, ABACUS_PEER_BLOB bytes: CUDA IPC handle, process id, device
 * address, device ordinal).  Errors: E_INVALID, E_CUDA. */
int abacus_peer_export(abacus_ctx* ctx, uint8_t* blob);
/* Build a peer communicator for (nranks, rank) from every rank's blob
 * (host, nranks x ABACUS_PEER_BLOB, rank order, e.g. all-gathered with
 * torch.distributed); opens the other processes' mailboxes with CUDA IPC.
 * *comm_out is owned by the caller (abacus_peer_comm_destroy).
 * Errors: E_INVALID (1 <= nranks <= ABACUS_PEER_MAX, blob of this rank not
 * from this ctx, no abacus_peer_export), E_CUDA. */
int abacus_peer_comm_init(abacus_ctx* ctx, int32_t nranks, int32_t rank, const uint8_t* blobs, void** comm_out);
/* Close the IPC mappings and free the communicator (NULL or an unknown
 * pointer is a no-op). */
void abacus_peer_comm_destroy(void* comm);

/* ------------------------------------------------------------------------ */
/* Introspection                                                             */
/* ------------------------------------------------------------------------ */

/* Number of device kernels the library launched on this ctx since creation
 * (used by bench.py for "gpu_launches"). */
uint64_t abacus_kernel_launches(const abacus_ctx* ctx);
/* Device time (ms, CUDA events on the launching stream) of the last fused
 * search kernel launch of this ctx; -1 if none. */
float abacus_last_kernel_ms(const abacus_ctx* ctx);
/* Use `stream` (a cudaStream_t on the ctx's device; NULL = the ctx's own
 * stream) for the blocking calls and as the default of the async ones. */
int abacus_set_stream(abacus_ctx* ctx, void* stream);
/* Enable (on != 0) CUDA-event timing of the fused search kernel on the ctx
 * stream, read back with abacus_last_kernel_ms. */
int abacus_set_timing(abacus_ctx* ctx, int on);
/* ABI version (ABACUS_ABI_VERSION). */
int abacus_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ABACUS_H */
