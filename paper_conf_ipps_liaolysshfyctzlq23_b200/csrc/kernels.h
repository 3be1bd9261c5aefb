// Launchers of the sm_100a kernels (internal).  All pointers are device
// pointers; all launches go on `st`.  Tensors are row-major; T = tokens, H =
// hidden, F = ffn width.  "E" storage is fp32 or bf16 per DType; statistics,
// gradients flowing between layers and weight gradients are fp32.
#pragma once
#include "common.h"

namespace mimose {

// Count of kernels launched by this library (bench "gpu_launches").
void note_launch(int n);
int64_t kernel_launch_count();

// ---------------------------------------------------------------- GEMM ----
// C[m, n] = sum_k A(m, k) * B(n, k) followed by an epilogue.
//   A(m,k) = A[m*a_sm + k*a_sk]   B(n,k) = B[n*b_sn + k*b_sk]   (element strides)
enum Epi : int {
  EPI_STORE = 0,          // C(E) = acc
  EPI_BIAS = 1,           // C(E) = acc + bias
  EPI_BIAS_GELU = 2,      // C(E) = u = acc + bias ; C2(E) = gelu(u)
  EPI_BIAS_DROP_RES = 3,  // C(f32) = res(E) + drop(acc + bias)   element e = m*ldc + n
  EPI_GELU_BWD = 4,       // C(E) = acc * gelu'(aux(E))
  EPI_ACC_RES_F32 = 5,    // C(f32) = acc + res(f32)  (res may alias C)
  EPI_F32 = 6,            // C(f32) = acc ; split-K: C + z*split_stride
  EPI_NONE = 7,           // benchmark only: accumulator read from TMEM, nothing stored
  EPI_BIAS_GELUT = 8,     // C(E) = u = acc + bias ; C2(E) = gelu_tanh(u)        (GPT-2)
  EPI_GELUT_BWD = 9,      // C(E) = acc * gelu_tanh'(aux(E))
  EPI_BIAS_DROP_RESF32 = 10,  // C(f32) = res(f32) + drop(acc + bias)  (pre-LN residual stream)
  EPI_ACC_F32 = 11        // C(f32) += acc  (fixed-order accumulation across launches)
};
struct GemmArgs {
  int M = 0, N = 0, K = 0;
  const void* A = nullptr; int64_t a_sm = 0, a_sk = 0;
  const void* B = nullptr; int64_t b_sn = 0, b_sk = 0;
  void* C = nullptr; int64_t ldc = 0;
  void* C2 = nullptr;
  const void* bias = nullptr;
  const void* res = nullptr; int64_t ldr = 0;
  const void* aux = nullptr; int64_t ldx = 0;
  Drop drop{};
  int split = 1; int64_t split_stride = 0;
  int bn = 0;              // forced tile width (0 = heuristic)
};
void gemm(DType dt, Epi epi, const GemmArgs& g, cudaStream_t st, bool use_tc);
bool tc_available();
// Two independent fp32-output (EPI_F32, split 1) bf16 GEMMs in one persistent
// tcgen05 launch with tile width bn (128 or 256; N % bn == 0).  Returns false
// (nothing launched) when the shapes / mode do not allow it.
bool gemm_tc_grouped(const GemmArgs& g1, const GemmArgs& g2, int bn, cudaStream_t st);
// 0: one tile per CTA; 1: persistent double-buffered (default).
void set_gemm_mode(int m);
// Deterministic split-K reduction: out[i] = sum_s part[s*n + i] (fixed order).
void splitk_reduce(const float* part, int splits, int64_t n, float* out, cudaStream_t st);

// ----------------------------------------------------------- attention ----
// qkv [B*S, 3H] (q | k | v, head-major columns), O [B*S, H], lse [B, h, S].
void attn_fwd(DType dt, const void* qkv, const int32_t* lengths, void* O, float* lse,
              int B, int S, int H, int h, Drop drop, cudaStream_t st, bool causal = false);
// bf16 with head dim 64 and S <= 128 runs on tcgen05 unless disabled (tests).
void set_attn_tc(bool on);
bool attn_tc_enabled();
// D [B,h,S] = rowsum(dO * O); dqkv [B*S, 3H].
void attn_bwd(DType dt, const void* qkv, const void* O, const void* dO, const float* lse,
              const int32_t* lengths, float* Dbuf, void* dqkv, int B, int S, int H, int h,
              Drop drop, cudaStream_t st, bool causal = false);

// Cross-attention (encoder-decoder): q [B*Sq, H], kv [B*Sk, 2H] (k | v); key
// padding by klens; tcgen05, head dim 64: the one-tile kernels when Sq, Sk <=
// 128, else the tiled ones (<= 1024; Dbuf [B, h, Sq] fp32 scratch for D).
// false: not launched.
bool attn_cross_fwd_tc(const void* q, const void* kv, const int32_t* qlens, const int32_t* klens, void* O, float* lse,
                       int B, int Sq, int Sk, int H, int h, Drop drop, cudaStream_t st);
bool attn_cross_bwd_tc(const void* q, const void* kv, const void* O, const void* dO, const float* lse,
                       const int32_t* qlens, const int32_t* klens, float* Dbuf, void* dq, void* dkv, int B, int Sq,
                       int Sk, int H, int h, Drop drop, cudaStream_t st);
bool attn_cross_fwd_tcl(const void* q, const void* kv, const int32_t* qlens, const int32_t* klens, void* O, float* lse,
                        int B, int Sq, int Sk, int H, int h, Drop drop, cudaStream_t st);
bool attn_cross_bwd_tcl(const void* q, const void* kv, const void* O, const void* dO, const float* lse,
                        const int32_t* qlens, const int32_t* klens, float* Dbuf, void* dq, void* dkv, int B, int Sq,
                        int Sk, int H, int h, Drop drop, cudaStream_t st);

// ----------------------------------------------------------- layernorm ----
// y = LN(z) (y may be null: recompute with the output store gated off); st = (mu, rstd).
// z (pre-LN sum) is fp32 in every mode.
void ln_fwd(DType dt, const float* z, const void* g, const void* b, void* y, float2* st,
            int T, int H, float eps, cudaStream_t st_);
// dz = LN'(dy [* premask]); dt = dz * mask (if dt != null);
// partials: pg, pb (dgamma, dbeta) and pbias (= colsum dt, if non-null), [NPART][H].
// res (nullable, may alias dz): dz = LN'(dy) + res before the dropout/bias step.
void ln_bwd(DType dt, const float* dy, Drop premask, const float* z, const float2* st,
            const void* g, float* dz, void* dtout, Drop mask, float* pg, float* pb,
            float* pbias, int T, int H, cudaStream_t st_, const float* res = nullptr);
// out(E) = in(f32) * mask ; part [NPART][N] = column sums of the stored out
void drop_cast_colsum(DType dt, const float* in, Drop mask, void* out, int T, int N, float* part, cudaStream_t st);
// out[c] = sum_p part[p*ld + c], p = 0..NPART-1 (fixed order)
void reduce_partials(const float* part, int64_t ld, int n, float* out, cudaStream_t st);
// Up to three such reductions in one launch (p1/p2 may be null), `rows` partial rows.
void reduce_rows3(const float* p0, float* o0, const float* p1, float* o1, const float* p2, float* o2, int rows,
                  int64_t ld, int n, cudaStream_t st);
// partials [NPART][N] of column sums of X [T, N] (E)
void colsum(DType dt, const void* X, int T, int N, float* part, cudaStream_t st);

// ----------------------------------------------------------- embedding ----
void embed_fwd(DType dt, const int32_t* ids, const int32_t* tt, const void* Ww, const void* Wp,
               const void* Wt, const void* g, const void* b, float* z0, float2* st0, void* x1,
               int B, int S, int H, int pos_offset, float eps, Drop drop, cudaStream_t st);
// Deterministic keyed row-sum: out[key[t]] = sum over tokens with that key, in
// token order, of rows of X [T, H] (fp32).  out rows not present, and the row of
// key `skip` (the padding id: HF padding_idx semantics), are untouched.
// X is clobbered (piece sums are written in place).  work: 4*T int32 + hist.
void keyed_rowsum(const int32_t* keys, int key_bits, float* X, int T, int H, float* out,
                  int32_t* work, int32_t* hist, int max_tiles, int skip, cudaStream_t st,
                  bool accumulate = false);
// GPT-2 embedding: x1(f32) = drop(wte[ids] + wpe[pos_offset + s])
void embed_fwd_pre(DType dt, const int32_t* ids, const void* Ww, const void* Wp, float* x1, int B, int S, int H,
                   int pos_offset, Drop drop, cudaStream_t st);
// dz0(f32) = dy * mask
void drop_f32(const float* dy, Drop mask, float* out, int64_t n, cudaStream_t st);
// dWt[k] = sum over tokens with token_type k of dz0 rows (fixed-order partials)
void type_grad(const float* dz0, const int32_t* tt, int T, int H, int TV, float* part, float* dWt, cudaStream_t st);
// dWp[pos_offset + s] = sum_b dz0[b*S + s]
void pos_grad(const float* dz0, int B, int S, int H, int pos_offset, float* dWp, cudaStream_t st,
              bool accumulate = false);

// ---------------------------------------------------------------- heads ----
// seq-cls / MC: pooled p [B,H] (E), logits [B,n_out] f32, loss -> misc[0]
void head_cls_fwd(DType dt, const void* y, int B, int S, int H, const void* Wp, const void* bp,
                  const void* Wc, const void* bc, int n_out, void* p, float* logits,
                  const int32_t* labels, int n_choices, int head_kind, float* loss, Drop drop,
                  cudaStream_t st);
// backward: scratch = dlogits [B*n_out] | dpd [B,H] f32 | dpre [B,H] f32
void head_cls_bwd(DType dt, const void* y, int B, int S, int H, const void* Wp, const void* Wc,
                  int n_out, const void* p, const float* logits, const int32_t* labels,
                  int n_choices, int head_kind, float* scratch, float* dWp, float* dbp,
                  float* dWc, float* dbc, float* dy, Drop drop, cudaStream_t st);
void head_qa_fwd(DType dt, const void* y, int B, int S, int H, const void* Wq, const void* bq,
                 float* logits, const int32_t* lengths, const int32_t* labels, float* loss,
                 cudaStream_t st);
void head_qa_bwd(DType dt, const void* y, int B, int S, int H, const void* Wq, const float* logits,
                 const int32_t* lengths, const int32_t* labels, float* dlog, float* part,
                 float* dWq, float* dbq, float* dy, cudaStream_t st);

// LM head (next-token CE over s < len-1).  logits: fp32 [nrows, ldv] of tokens
// row0..row0+nrows; tokstat[t] = (lse, nll).
void lm_ce_fwd(const float* logits, int64_t ldv, int V, int row0, int nrows, const int32_t* ids,
               const int32_t* lengths, int S, float2* tokstat, cudaStream_t st);
void lm_loss(const float2* tokstat, int T, const int32_t* lengths, int B, int S, float* loss, cudaStream_t st);
// dlog(E) = valid ? (softmax - onehot) / n_valid : 0
void lm_ce_bwd(DType dt, const float* logits, int64_t ldv, int V, int row0, int nrows, const int32_t* ids,
               const int32_t* lengths, int B, int S, const float2* tokstat, void* dlog, cudaStream_t st);

// ----------------------------------------------------------- optimizer ----
// AdamW (torch semantics).  master == nullptr: fp32 mode, w is the master.
void adamw(DType dt, void* w, float* master, const float* g, float* m, float* v, int64_t n,
           float lr, float b1, float b2, float eps, float wd, float bc1, float bc2,
           float grad_scale, cudaStream_t st);
// fp32 -> storage copy (set_params) and storage -> fp32 (get_params)
void cast_from_f32(DType dt, const float* src, void* dst, int64_t n, cudaStream_t st);
void cast_to_f32(DType dt, const void* src, float* dst, int64_t n, cudaStream_t st);

}  // namespace mimose
