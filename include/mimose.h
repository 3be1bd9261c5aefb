/*
 * mimose.h — C ABI of the B200-native Mimose training-step library (libmimose.so).
 *
 * What it implements (PAPER.md = /root/reference/PAPER.md, "P:n" = line n):
 *   Mimose, an input-aware activation-checkpointing planner (§IV, Fig. 6):
 *     - shuttling online collector (§IV-B, Fig. 7)    -> mimose_collect
 *     - lightning memory estimator  (§IV-C, §VI-E)     -> fitted inside the ctx
 *     - responsive greedy scheduler (§IV-D, Algorithm 1) -> mimose_plan
 *     - applying the plan on the fly (§V)             -> mimose_forward / _backward
 *   around the checkpointed training step of a post-LN transformer encoder
 *   (P:51 forward -> loss -> backward -> update; P:160 attention structure),
 *   under a hard device-memory budget M (Algorithm 1 input).
 *   Readings of silent / garbled passages: DESIGN.md "Readings" (A1..A28, R-*).
 *
 * Conventions
 *   - Every call returns mimose_status; nothing throws across the ABI.
 *   - Pointers are plain host or device pointers as documented per field; no
 *     torch types.  The caller owns every struct it passes in.
 *   - All device work is enqueued on cfg.stream (a cudaStream_t); calls return
 *     before the device finishes unless an output pointer needs a host value
 *     (loss_out), in which case only that scalar is synchronised.
 *   - One ctx per device per host thread; no global mutable state.
 *   - MIMOSE_E_CUDA / MIMOSE_E_NCCL are sticky: the ctx refuses further work.
 *   - mimose_last_error() returns a human-readable message for the last failure.
 */
#ifndef MIMOSE_H_
#define MIMOSE_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MIMOSE_ABI_VERSION 1

typedef struct mimose_ctx mimose_ctx; /* opaque, owned by the library */

typedef enum {
  MIMOSE_OK = 0,
  MIMOSE_E_INVALID = 1,    /* bad argument / config / size                          */
  MIMOSE_E_STATE = 2,      /* call out of order (see "Call order")                 */
  MIMOSE_E_NOT_READY = 3,  /* mimose_plan before the estimator is fitted           */
  MIMOSE_E_INFEASIBLE = 4, /* even the deepest plan predicts peak > M - reserve    */
  MIMOSE_E_BUDGET = 5,     /* an arena request would make live bytes > M: the step
                              is abandoned before any launch, counted as a violation,
                              and the arena is rolled back                           */
  MIMOSE_E_CUDA = 6,       /* sticky */
  MIMOSE_E_NCCL = 7,       /* sticky */
  MIMOSE_E_NODEVICE = 8    /* device call on a host-only ctx (arena_base == NULL)   */
} mimose_status;

enum { MIMOSE_ARCH_POST_LN = 0, MIMOSE_ARCH_PRE_LN = 1, MIMOSE_ARCH_ENCDEC = 2 };
enum { MIMOSE_HEAD_SEQCLS = 0, MIMOSE_HEAD_MC = 1, MIMOSE_HEAD_QA = 2, MIMOSE_HEAD_LM = 3 };
enum { MIMOSE_FP32 = 0, MIMOSE_BF16 = 1 };
enum { MIMOSE_PHASE_SHELTERED = 0, MIMOSE_PHASE_RESPONSIVE = 1 };

typedef struct {
  /* ---- model (post-LN BERT/RoBERTa encoder, P:227 models; reading A24) ---- */
  int32_t arch;         /* MIMOSE_ARCH_POST_LN (BERT/RoBERTa) or MIMOSE_ARCH_PRE_LN (GPT-2:
                           causal, fp32 residual stream, tied wte, final LN)             */
  int32_t head;         /* MIMOSE_HEAD_*: seq-cls, multiple-choice, QA span (Table II);
                           MIMOSE_HEAD_LM (pre-LN only): chunked next-token CE          */
  int32_t dtype;        /* MIMOSE_FP32 (toy) or MIMOSE_BF16 (bf16 storage, fp32 accum,
                           fp32 master weights)                                          */
  int32_t n_layers;     /* L <= 64                                                      */
  int32_t hidden;       /* H, multiple of 64 (head dim d = H/heads must be 32 or 64)    */
  int32_t heads;
  int32_t ffn;          /* F, multiple of 64                                            */
  int32_t vocab, max_pos, type_vocab, pos_offset;
  int32_t n_choices;    /* MC: sequences per question                                   */
  int32_t n_labels;     /* seq-cls: classes                                             */
  float p_drop;         /* dropout probability on every site (reading A24)              */
  float ln_eps;
  uint64_t seed;        /* Philox4x32-10 key (reading R-B)                              */
  /* ---- Mimose ---- */
  int64_t budget_bytes;  /* M of Algorithm 1: hard cap on arena live bytes,
                            persistent state included                                   */
  int64_t reserve_bytes; /* paper's fragmentation reserve; default 0 (A22)       */
  int32_t enforce_budget;/* 1: an allocation beyond M -> MIMOSE_E_BUDGET;
                            0: record only (no-checkpoint baseline)                     */
  int32_t collect_iters; /* sheltered-phase length, default 10 (A17)            */
  int32_t bucket_num, bucket_den; /* Alg. 1 line 8 ratio, default 9/10 (A6)           */
  int32_t degree;        /* regression degree, default 2                        */
  int32_t max_seqs, max_seq_len; /* sizing limits of a batch                            */
  /* ---- device plumbing (supplied by the caller, e.g. PyTorch) ---- */
  void* arena_base;      /* device slab, >= arena_bytes, 256-B aligned, outlives ctx.
                            NULL -> host-only ctx: collector / estimator / planner /
                            dry-run accounting run, no kernel is launched            */
  int64_t arena_bytes;   /* slab size; must be >= budget_bytes when enforce_budget   */
  void* stream;          /* cudaStream_t for all compute                             */
  int32_t rank, world;   /* data parallel (weak scaling: each rank its own batch)    */
  const void* nccl_id;   /* 128-byte ncclUniqueId from rank 0 (broadcast by caller);
                            NULL when world == 1                                     */
  int32_t use_tc;        /* 1: tcgen05 GEMMs in bf16 mode (default); 0: SIMT GEMMs  */
  int32_t pad_id;        /* padding token id: its embedding row gets no gradient (HF
                            padding_idx semantics, reading A24); -1 = none           */
  int32_t granularity;   /* checkpoint unit: 0 = encoder layer (default, A14); 1 = sub-layer:
                            unit 2l = attention block of layer l (post-LN internals QKV, O,
                            LSE, z1, st1, output h1; pre-LN a, st1, QKV, O, LSE, output r1),
                            unit 2l+1 = its FFN block (post-LN u, g, z2, st2; pre-LN st2, m,
                            u, g; output y), so 2L <= 64 units (SURVEY f1, P:125/P:140
                            "attention block"; reading A30).  Samples, series and drop
                            masks are then indexed by unit.                              */
  int32_t comm_force;    /* 1: create the NCCL communicator (and run the per-bucket
                            ncclAllReduce, the loss all-reduce and the plan check) even
                            at world == 1 (a 1-rank communicator; test / single-GPU
                            evidence of the a10 path).  0: only when world > 1        */
  int32_t nccl_max_ctas; /* NCCL CTA cap (ncclConfig_t.maxCTAs): 0 = 16 (default),
                            < 0 = NCCL's own default                                   */
  int32_t check_plans;   /* 1: every mimose_forward all-gathers a 64-bit hash of
                            (x, drop mask, predicted peak) over the communicator and
                            fails with MIMOSE_E_STATE if any rank differs (
                            debug: one small device->host sync per step)               */
  int32_t zero1;         /* 1: ZeRO-1: the AdamW state (fp32 master, m, v) is
                            sharded over the ranks.  Each gradient bucket is padded to
                            64 x world elements, reduce-scattered (instead of all-reduced),
                            this rank's shard updated, and the bf16 working weights
                            all-gathered -- all overlapped with the backward when the
                            optimizer is fused.  Persistent bytes fall from 18 to
                            6 + 12 / world B/param.  Needs a communicator (world > 1 or
                            comm_force); mimose_get_master is then refused for world > 1. */
  int32_t n_dec_layers;  /* MIMOSE_ARCH_ENCDEC: decoder layers; n_layers is then
                            the encoder's.  Checkpoint units: encoder layers 0..n_layers-1,
                            decoder layers n_layers..n_layers+n_dec_layers-1            */
  const int32_t* ffn_layers; /* heterogeneous stages: FFN width of each of the
                            n_layers layers (multiples of 64, <= ffn; ffn is then the max
                            and sizes the shared workspaces); NULL = every layer uses ffn.
                            Read during mimose_init only.                             */
} mimose_config;

/* Fill defaults (collect_iters 10, ratio 9/10, degree 2, p 0.1, eps 1e-12,
   enforce 1, world 1, use_tc 1) into *cfg; the caller then sets the model fields. */
void mimose_default_config(mimose_config* cfg);

/* One mini-batch.  All arrays are int32, row-major, caller-owned and only read
   during the call.  on_host = 1: host pointers (pinned recommended) copied H2D
   inside the call; 0: device pointers.
     input_ids  [n_seqs, seq_len]   right-padded with the pad id
     token_type [n_seqs, seq_len]
     lengths    [n_seqs]            valid tokens per sequence, 1..seq_len
     labels     seq-cls: [n_seqs] class; MC: [n_seqs / n_choices] choice;
                QA: [2*n_seqs] (start, end) per sequence; LM: unused (targets are
                input_ids shifted by one inside each sequence, s < len - 1)
   The input size key of P:73/P:221 is x = n_seqs * seq_len. */
typedef struct {
  const int32_t* input_ids;
  const int32_t* token_type;
  const int32_t* lengths;
  const int32_t* labels;
  int32_t n_seqs, seq_len;
  int32_t on_host;
  /* encoder-decoder only (MIMOSE_ARCH_ENCDEC): the decoder's input ids
     [n_seqs, dec_len] (right-padded; the LM targets are these shifted by one
     inside each sequence) and valid lengths [n_seqs].  input_ids / lengths are
     then the encoder's source; token_type and labels are unused.  The input
     size key is 2-D: (n_seqs * seq_len, n_seqs * dec_len). */
  const int32_t* dec_ids;
  const int32_t* dec_lengths;
  int32_t dec_len;
  int32_t pad_;
} mimose_batch;

/* Algorithm 1 output L' as a bitmask over layers (bit l = layer l,
   0-based, is dropped and recomputed in backward). */
typedef struct {
  uint64_t drop_mask;
  int32_t n_dropped;
  int32_t from_cache;      /* 1 if served by the plan cache                  */
  int64_t input_size;      /* x                                                      */
  int64_t predicted_peak;  /* position-aware predicted peak of L' (reading A13)     */
  int64_t budget;          /* M - reserve                                            */
  int32_t status;          /* MIMOSE_OK or MIMOSE_E_INFEASIBLE                       */
  int32_t pad_;
} mimose_plan_t;

/* Collected sample of one sheltered iteration (shuttling collector):
   arena live-byte deltas; see DESIGN.md "Memory model". */
typedef struct {
  int64_t x;
  int64_t C;             /* persistent bytes at forward start                        */
  int64_t E;             /* embedding-forward delta                                  */
  int64_t Hd;            /* head-forward delta                                       */
  int64_t Th, Tb, Te;    /* max top-region bytes in head / layer / embedding backward */
  int64_t a[64];         /* pass-1 (save mode) delta per layer                       */
  int64_t y[64];         /* pass-2 (no-save mode) delta per layer                    */
  float   t_ms[64];      /* pass-1 forward time per layer (cudaEvent; 0 host-only)   */
  int64_t xt;            /* encoder-decoder: the target input size (2-D key); else 0  */
} mimose_sample;

typedef struct {
  int64_t live_bytes, peak_bytes;      /* arena now / peak of the last step           */
  int64_t max_peak_bytes;              /* over the ctx lifetime                        */
  int64_t persistent_bytes;            /* C                                            */
  int64_t budget_bytes;
  int64_t violations;                  /* MIMOSE_E_BUDGET events                       */
  int64_t steps, collect_steps, shuttled_steps;
  int64_t plan_calls, plan_cache_hits, plan_cache_misses;
  int64_t n_samples;
  int32_t phase, last_n_dropped;
  uint64_t last_drop_mask;
  int64_t last_predicted_peak;
  double planner_us_total;             /* host time in estimator+planner on misses     */
  double collector_ms_total;           /* host wall time of shuttled collect calls     */
  int64_t kernel_launches;             /* our kernels launched since init              */
  int64_t allreduce_calls;             /* ncclAllReduce of gradient buckets issued      */
  int64_t allreduce_bytes;             /* their fp32 bytes                             */
  int64_t plan_checks;                 /* cross-rank plan-hash checks passed (X4)      */
  int32_t comm_nranks;                 /* communicator size (0: no communicator)       */
  int32_t pad_;
} mimose_stats;

mimose_status mimose_init(const mimose_config* cfg, mimose_ctx** out);
void mimose_destroy(mimose_ctx* ctx);
const char* mimose_last_error(const mimose_ctx* ctx);
const char* mimose_status_str(mimose_status s);

/* Parameters: a host fp32 blob of every parameter tensor concatenated in the
   documented order (workload.param_spec), no
   padding.  bf16 mode: the fp32 values become the master copy and are rounded
   (RNE) to the bf16 working copy.  Also resets AdamW state and the step count. */
mimose_status mimose_num_params(const mimose_ctx* ctx, int64_t* n);
mimose_status mimose_set_params(mimose_ctx* ctx, const float* host_blob, int64_t n);
/* Reads the working copy (bf16 mode: bf16 values widened to fp32). */
mimose_status mimose_get_params(mimose_ctx* ctx, float* host_blob, int64_t n);
/* Reads the fp32 master copy AdamW updates (bf16 mode; fp32 mode: the weights). */
mimose_status mimose_get_master(mimose_ctx* ctx, float* host_blob, int64_t n);
/* fp32 gradients of the last backward (after the DP all-reduce, before the
   1/world scale), same order.  Test hook; synchronises the stream. */
mimose_status mimose_get_grads(mimose_ctx* ctx, float* host_blob, int64_t n);

/* Sheltered phase (Fig. 7): a forward in which every layer runs twice —
   pass 1 normal (deltas -> a_l, time -> t_l, then discarded), pass 2 keeping
   only the layer output (delta -> y_l).  Only unseen x are shuttled;
   seen x run the conservative all-dropped forward.  Backward then recomputes
   every layer and measures the transients.  After collect_iters calls (at least
   3 distinct x, at most 30 calls, reading A17) the estimator is fitted and the
   phase becomes RESPONSIVE.  loss_out (host, may be NULL) receives the loss. */
mimose_status mimose_collect(mimose_ctx* ctx, const mimose_batch* batch, float* loss_out);

/* Algorithm 1 (our reading): (M, x, L) -> L'.  Served from the plan
   cache when x was planned before.  Host only, no device work.
   Returns MIMOSE_E_NOT_READY in the sheltered phase; MIMOSE_E_INFEASIBLE if even
   the deepest plan predicts a peak above M - reserve (out->status set too). */
mimose_status mimose_plan(mimose_ctx* ctx, int64_t input_size, mimose_plan_t* out);
/* Encoder-decoder (reading A32): the plan for the 2-D input size
   (x = numel(source ids), x_t = numel(target ids)); the estimator behind it is
   the bivariate quadratic of the collector's samples (P:162-164 per input
   tensor).  Same cache / errors as mimose_plan; out->input_size = x. */
mimose_status mimose_plan2(mimose_ctx* ctx, int64_t x_src, int64_t x_tgt, mimose_plan_t* out);

/* Selects the scheduler behind mimose_plan (Mimose "reserves a
   flexible interface for users to experiment with other scheduling algorithms,
   such as the Knapsack optimization").  kind 0 = Algorithm 1 greedy (default);
   kind 1 = exact: the fewest recomputed layers whose position-aware predicted
   peak fits M - reserve, then the lowest peak, then the lexicographically
   smallest layer list (reading A29); kind 2 = time-weighted exact
   (the Knapsack): the least total recompute cost, cost_l(x) = the collector's
   forward time t_l regressed on x (integer ns, >= 1; averaged over the
   ranks before the fit when a communicator exists), then the lowest peak, then
   lexicographic (reading A31).  Clears the plan cache when the kind changes.
   MIMOSE_E_INVALID for an unknown kind; host only. */
mimose_status mimose_set_planner(mimose_ctx* ctx, int32_t kind);

/* Responsive forward under plan (NULL -> no layer dropped).  Dropped layers
   keep only their output.  The whole step's allocation sequence is
   checked against M before any launch (MIMOSE_E_BUDGET on breach). */
mimose_status mimose_forward(mimose_ctx* ctx, const mimose_batch* batch,
                             const mimose_plan_t* plan, float* loss_out);
/* Backward: recompute each dropped layer with the same kernels, launch
   configuration and Philox sites right before its gradient kernels (P:21,
   P:217); per-layer NCCL all-reduce overlapped with the remaining backward. */
mimose_status mimose_backward(mimose_ctx* ctx);
/* AdamW (torch semantics, reading A25) on the fp32 master weights. */
mimose_status mimose_step(mimose_ctx* ctx, float lr, float beta1, float beta2, float eps, float wd);
/* Register the optimizer.  fused = 1: mimose_backward launches AdamW for every
   gradient bucket (encoder layer, head, embeddings) on a separate stream as
   soon as that bucket is final (after its all-reduce under DP), overlapping the
   rest of the backward; mimose_step then only orders the next forward after the
   updates and must be called with the same arguments.  Same arithmetic as the
   unfused step. */
mimose_status mimose_set_optimizer(mimose_ctx* ctx, float lr, float beta1, float beta2, float eps, float wd,
                                   int32_t fused);

mimose_status mimose_get_stats(const mimose_ctx* ctx, mimose_stats* out);
mimose_status mimose_phase(const mimose_ctx* ctx, int32_t* phase);
mimose_status mimose_get_sample(const mimose_ctx* ctx, int32_t i, mimose_sample* out);

/* Host-only accounting of one full step (no launch): peak arena bytes for a
   batch shape and plan, using the same allocation sequence as the real step.
   Used to size budgets and by tests; never consulted by the planner (c-F). */
mimose_status mimose_dry_run(mimose_ctx* ctx, int32_t n_seqs, int32_t seq_len,
                             uint64_t drop_mask, int64_t* peak_out);
/* Shuttling-collector accounting alone (no launch): the sample a sheltered
   iteration at this shape would record (t_ms = 0). */
mimose_status mimose_dry_collect(mimose_ctx* ctx, int32_t n_seqs, int32_t seq_len,
                                 mimose_sample* out);
/* The same two for an encoder-decoder batch shape (source seq_len, target dec_len). */
mimose_status mimose_dry_run2(mimose_ctx* ctx, int32_t n_seqs, int32_t seq_len, int32_t dec_len,
                              uint64_t drop_mask, int64_t* peak_out);
mimose_status mimose_dry_collect2(mimose_ctx* ctx, int32_t n_seqs, int32_t seq_len, int32_t dec_len,
                                  mimose_sample* out);

/* Writes a fresh 128-byte ncclUniqueId (rank 0 calls it and broadcasts the
   bytes through the caller's process group before mimose_init on every rank). */
mimose_status mimose_nccl_unique_id(void* out128);

/* Kernel probe for the roofline report: when enabled (kind = 1: every GEMM
   launch of the step) the library records a cudaEvent pair around each probed
   launch on cfg.stream and accumulates the algorithmic FLOPs (2 M N K).
   mimose_probe_read synchronises, returns the summed device time (ms), FLOPs
   and launch count since the last enable, and keeps the probe running. */
mimose_status mimose_probe(mimose_ctx* ctx, int32_t kind);
mimose_status mimose_probe_read(mimose_ctx* ctx, double* total_ms, double* total_flops, int64_t* launches);

/* Test hook: one bf16 GEMM of the library, C[m,n] = sum_k A(m,k) B(n,k) with
   A(m,k) = A[m*a_sm + k*a_sk], B(n,k) = B[n*b_sn + k*b_sk] (element strides),
   epilogue `epi` (0 store bf16, 1 +bias bf16, 6 fp32; split-K writes `split`
   fp32 partials at C + z*M*ldc), tensor-core path if use_tc.  Device pointers;
   enqueued on `stream`. */
mimose_status mimose_debug_gemm(int32_t epi, int32_t M, int32_t N, int32_t K, const void* A, int64_t a_sm,
                                int64_t a_sk, const void* B, int64_t b_sn, int64_t b_sk, void* C, int64_t ldc,
                                const void* bias, int32_t split, int32_t use_tc, void* stream);
/* Same, every epilogue (0 store, 1 bias, 2 bias+GELU -> C, C2, 3 bias+dropout(p=0.1, seed 7)+residual
   -> fp32 C, 4 GELU' with aux, 5 fp32 C = acc + res, 6 fp32, 7 none (benchmark), 8 bias+tanh-GELU
   -> C, C2, 9 tanh-GELU' with aux, 10 bias+dropout+fp32 residual -> fp32 C, 11 fp32 C += acc);
   MIMOSE_E_INVALID for any other epi. */
mimose_status mimose_debug_gemm_ex(int32_t epi, int32_t M, int32_t N, int32_t K, const void* A, int64_t a_sm,
                                   int64_t a_sk, const void* B, int64_t b_sn, int64_t b_sk, void* C, int64_t ldc,
                                   void* C2, const void* bias, const void* res, int64_t ldr, const void* aux,
                                   int64_t ldx, int32_t split, int32_t use_tc, void* stream);

/* Test hook: two fp32-output bf16 GEMMs (as mimose_debug_gemm with epi 6, split 1)
   in ONE grouped persistent tcgen05 launch, 128 x 256 tiles (the grouped wgrad of
   the FFN block).  Returns MIMOSE_E_INVALID if the pair cannot be grouped (N % 256,
   more tiles than SMs). */
mimose_status mimose_debug_gemm_grouped(int32_t M1, int32_t N1, int32_t K1, const void* A1, int64_t a_sm1,
                                        int64_t a_sk1, const void* B1, int64_t b_sn1, int64_t b_sk1, void* C1,
                                        int32_t M2, int32_t N2, int32_t K2, const void* A2, int64_t a_sm2,
                                        int64_t a_sk2, const void* B2, int64_t b_sn2, int64_t b_sk2, void* C2,
                                        void* stream);

/* Test hook: process-wide kernel options. gemm_mode 1 = the default persistent
   tcgen05 GEMM (tile width and CTA pairs chosen per shape, grouped weight
   gradients), 12 / 13 = single-CTA tiles of width 256 / 128 for every shape and
   no grouped launches, 15 = LSU instead of TMA stores in the epilogues, 17 = the
   CTA-pair kernel (cta_group::2, 256 x 256 tiles) wherever N % 256 == 0; attn_tc
   0/1 routes bf16 attention with S <= 128 to the SIMT / tcgen05 kernels.
   Negative = unchanged. */
void mimose_debug_options(int32_t gemm_mode, int32_t attn_tc);

/* 1 if this build routes bf16 GEMMs to the tcgen05/TMEM/TMA kernels. */
int32_t mimose_tc_available(void);

/* ---- stateless host helpers (tests; same code the ctx uses) ---- */
/* Predicted series for one x: arrays a,y of n_layers entries. */
typedef struct {
  int64_t C, E, Hd, Th, Tb, Te;
  const int64_t* a;
  const int64_t* y;
  int32_t n_layers;
} mimose_series;
/* Position-aware predicted peak of a plan (reading A13). */
int64_t mimose_predicted_peak(const mimose_series* s, uint64_t drop_mask);
/* Full planner (Alg. 1 + A12 + A13) on given predictions. */
mimose_status mimose_plan_series(const mimose_series* s, int64_t budget, int64_t reserve,
                                 int32_t bucket_num, int32_t bucket_den,
                                 uint64_t* drop_mask, int64_t* predicted_peak);
/* (bucket_num == 0 selects the exact planner of mimose_set_planner kind 1.) */
/* The time-weighted exact planner (kind 2) on given predictions and per-layer
   integer costs cost[0..n_layers) (each clamped to >= 1). */
mimose_status mimose_plan_series_cost(const mimose_series* s, const int64_t* cost, int64_t budget,
                                      int64_t reserve, uint64_t* drop_mask, int64_t* predicted_peak);
/* Quadratic least squares (reading A18): fit ys(xs), predict at x_eval[i]. */
mimose_status mimose_fit_predict(const int64_t* xs, const int64_t* ys, int32_t n, int32_t degree,
                                 const int64_t* x_eval, int32_t n_eval, int64_t* out);

#ifdef __cplusplus
}
#endif
#endif /* MIMOSE_H_ */
