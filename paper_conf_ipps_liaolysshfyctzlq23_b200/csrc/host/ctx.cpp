// libmimose host runtime: the C ABI of include/mimose.h.
//
//   arena      budget-enforcing two-ended LIFO arena over the caller's slab
//              (DESIGN "Memory model"; the paper's caching allocator loses
//              0.5-1 GB to fragmentation, P:296 — a LIFO arena cannot fragment)
//   schedule   forward / backward / recompute / optimizer launch order of one
//              step, run either for real or as a host-only dry run (identical
//              allocation sequence)
//   collector  shuttling double forward of the sheltered phase
//   estimator  + planner + plan cache (planning.cpp)
//   comm       per-layer NCCL gradient all-reduce overlapped with backward
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <array>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <unordered_map>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "../../../include/mimose.h"
#include "../kernels.h"
#include "planning.h"

using namespace mimose;

namespace {

inline int64_t a16(int64_t n) { return (n + 15) / 16 * 16; }

// NVTX ranges for Nsight timelines (MIMOSE_NVTX=1): the public calls and every
// layer / unit forward, recompute and backward.  Header-only NVTX v3; off by default.
bool nvtx_on() {
  static const bool v = [] {
    const char* e = std::getenv("MIMOSE_NVTX");
    return e && std::atoi(e) != 0;
  }();
  return v;
}
struct Range {
  bool on;
  explicit Range(const char* name) : on(nvtx_on()) { if (on) nvtxRangePushA(name); }
  Range(const char* what, int idx) : on(nvtx_on()) {
    if (on) {
      char buf[64];
      std::snprintf(buf, sizeof(buf), "%s %d", what, idx);
      nvtxRangePushA(buf);
    }
  }
  ~Range() { if (on) nvtxRangePop(); }
};

struct ParamInfo {
  int64_t numel, off;  // off in elements of the padded flat layout
};

// The documented parameter order (DESIGN "Parameter layout").
constexpr int LM_CHUNK = 2048;   // tokens per LM-head chunk (DESIGN "Memory model")
inline int64_t vpad(int64_t v) { return (v + 7) / 8 * 8; }

// Every tensor is padded to 64 elements.  The gradient buckets (embedding,
// one per layer, head; in layout order) end on a multiple of `unit` elements:
// 64, or 64 x world with ZeRO-1 so that every bucket splits into world equal
// shards.
std::vector<ParamInfo> build_layout(const mimose_config& c, int64_t* npad, int64_t unit = 64) {
  std::vector<int64_t> n;
  const int64_t H = c.hidden;
  auto Fof = [&](int l) -> int64_t { return c.ffn_layers ? c.ffn_layers[l] : c.ffn; };
  auto lay = [&](int n_emb) {
    std::vector<ParamInfo> out;
    int64_t off = 0;
    for (size_t i = 0; i < n.size(); ++i) {
      out.push_back({n[i], off});
      off += (n[i] + 63) / 64 * 64;
      const int64_t j = (int64_t)i + 1 - n_emb;          // params completed past the embedding bucket
      if (j == 0 || (j > 0 && j % 12 == 0 && j <= 12LL * c.n_layers) || i + 1 == n.size())
        off = (off + unit - 1) / unit * unit;             // bucket end
    }
    *npad = off;
    return out;
  };
  if (c.arch == 2) {             // encoder-decoder: wte, wpe, encoder layers, enc LNf, decoder layers, LNf
    n.push_back((int64_t)c.vocab * H);
    n.push_back((int64_t)c.max_pos * H);
    const int64_t F = c.ffn;
    for (int l = 0; l < c.n_layers; ++l) {
      const int64_t v[12] = {H, H, 3 * H * H, 3 * H, H * H, H, H, H, F * H, F, H * F, H};
      for (int64_t x : v) n.push_back(x);
    }
    n.push_back(H);
    n.push_back(H);
    for (int j = 0; j < c.n_dec_layers; ++j) {
      const int64_t v[20] = {H, H, 3 * H * H, 3 * H, H * H, H, H, H, H * H, H, 2 * H * H, 2 * H, H * H, H,
                             H, H, F * H, F, H * F, H};
      for (int64_t x : v) n.push_back(x);
    }
    n.push_back(H);
    n.push_back(H);
    std::vector<ParamInfo> out;
    int64_t off = 0;
    for (int64_t x : n) { out.push_back({x, off}); off += (x + 63) / 64 * 64; }
    *npad = (off + unit - 1) / unit * unit;
    return out;
  }
  if (c.arch == 1) {             // GPT-2: wte, wpe, pre-LN layers, lnf
    n.push_back((int64_t)c.vocab * H);
    n.push_back((int64_t)c.max_pos * H);
    for (int l = 0; l < c.n_layers; ++l) {
      const int64_t F = Fof(l);
      const int64_t v[12] = {H, H, 3 * H * H, 3 * H, H * H, H, H, H, F * H, F, H * F, H};
      for (int64_t x : v) n.push_back(x);
    }
    n.push_back(H);
    n.push_back(H);
    return lay(2);
  }
  n.push_back((int64_t)c.vocab * H);
  n.push_back((int64_t)c.max_pos * H);
  n.push_back((int64_t)c.type_vocab * H);
  n.push_back(H);
  n.push_back(H);
  for (int l = 0; l < c.n_layers; ++l) {
    const int64_t F = Fof(l);
    const int64_t v[12] = {3 * H * H, 3 * H, H * H, H, H, H, F * H, F, H * F, H, H, H};
    for (int64_t x : v) n.push_back(x);
  }
  if (c.head == MIMOSE_HEAD_QA) {
    n.push_back(2 * H);
    n.push_back(2);
  } else {
    const int64_t no = c.head == MIMOSE_HEAD_MC ? 1 : c.n_labels;
    n.push_back(H * H);
    n.push_back(H);
    n.push_back(no * H);
    n.push_back(no);
  }
  return lay(5);
}

enum { P_WORD = 0, P_POS, P_TYPE, P_LN0G, P_LN0B, P_LAYER0 };
enum { L_QKVW = 0, L_QKVB, L_OW, L_OB, L_LN1G, L_LN1B, L_F1W, L_F1B, L_F2W, L_F2B, L_LN2G, L_LN2B };

// ------------------------------------------------------------------ arena --
struct Arena {
  char* base = nullptr;
  int64_t cap = 0, budget = 0;
  bool enforce = true;
  int64_t C = 0;                 // persistent bytes (bottom)
  int64_t stack = 0;             // stack bytes above C
  int64_t top = 0;               // top-region bytes (grow down from cap)
  std::vector<int64_t> sstack, stop;
  int64_t peak = 0, top_phase_peak = 0;
  bool breach = false;

  int64_t live() const { return C + stack + top; }
  void tick() {
    peak = std::max(peak, live());
    top_phase_peak = std::max(top_phase_peak, top);
    if (live() > budget && enforce) breach = true;
    if (C + stack + top > cap) breach = true;   // physical collision: never allowed
  }
  char* push(int64_t n) {
    n = a16(n);
    char* p = base + C + stack;
    stack += n;
    sstack.push_back(n);
    tick();
    return p;
  }
  void pop(int64_t n) {
    n = a16(n);
    if (sstack.empty() || sstack.back() != n) { breach = true; return; }
    sstack.pop_back();
    stack -= n;
  }
  char* talloc(int64_t n) {
    n = a16(n);
    top += n;
    stop.push_back(n);
    tick();
    return base + cap - top;
  }
  void tfree(int64_t n) {
    n = a16(n);
    if (stop.empty() || stop.back() != n) { breach = true; return; }
    stop.pop_back();
    top -= n;
  }
  void reset_step() {
    stack = top = 0;
    sstack.clear();
    stop.clear();
    peak = live();
    breach = false;
  }
};

struct DecBufs {
  char *a = nullptr, *qkv = nullptr, *O = nullptr, *c = nullptr, *qc = nullptr, *kvc = nullptr, *oc = nullptr,
       *m = nullptr, *u = nullptr, *g = nullptr;
  float2 *st1 = nullptr, *st2 = nullptr, *st3 = nullptr;
  float *lse = nullptr, *lsec = nullptr, *r1 = nullptr, *r2 = nullptr;
};

struct LayerBufs {
  char *qkv = nullptr, *O = nullptr, *h1 = nullptr, *u = nullptr, *g = nullptr;
  float *z1 = nullptr, *z2 = nullptr;   // pre-LN sums, fp32 (reading R-P)
  char *a = nullptr, *m = nullptr;      // GPT-2: LN1 / LN2 outputs (GEMM operands)
  float* r1 = nullptr;                  // GPT-2: mid-layer residual stream (fp32)
  float *lse = nullptr;
  float2 *st1 = nullptr, *st2 = nullptr;
};

}  // namespace

struct mimose_ctx {
  mimose_config cfg{};
  DType dt = DT_F32;
  int e = 4;
  bool device = false;
  std::string err;
  mimose_status sticky = MIMOSE_OK;
  cudaStream_t st = nullptr, comm_st = nullptr, opt_st = nullptr;
  ncclComm_t comm = nullptr;
  cudaEvent_t ev_comm_done = nullptr, ev_opt_done = nullptr;
  std::vector<cudaEvent_t> ev_layer, ev_ar;
  // fused optimizer: per-bucket AdamW on opt_st as soon as the bucket's gradients are final
  bool opt_fused = false;
  float opt_lr = 0.f, opt_b1 = 0.9f, opt_b2 = 0.999f, opt_eps = 1e-8f, opt_wd = 0.f;

  std::vector<ParamInfo> layout;
  int64_t npad = 0;
  Arena ar;
  // persistent device buffers
  char* w = nullptr;
  float *grad = nullptr, *master = nullptr, *m = nullptr, *v = nullptr;
  int32_t *ids = nullptr, *tt = nullptr, *lens = nullptr, *labels = nullptr;
  float* misc = nullptr;
  float* ws = nullptr;        // split-K workspace (4 H H fp32)
  float* part = nullptr;      // NPART * 2 * max(3H, F) fp32
  int64_t ws_elems = 0;
  int planner = PLANNER_GREEDY;   // mimose_set_planner

  // step state
  int B = 0, S = 0, T = 0;
  uint64_t drop_mask = 0;
  bool fwd_done = false, bwd_done = false, collecting = false;
  bool step_pending = false;   // fused optimizer: backward applied the update, mimose_step not yet called
  // ZeRO-1: optimizer state (master, m, v) sharded over the ranks
  std::vector<int> ffn_l;                    // per-layer FFN widths (empty: uniform cfg.ffn)
  // Side stream for the weight-gradient reductions that nothing on the
  // backward's critical path reads (LN-partial and bias column sums)
  cudaStream_t aux_st = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  bool aux_pending = false;
  bool zero1 = false;
  int64_t nshard = 0;                        // elements of master / m / v on this rank
  std::vector<int64_t> bk_b0, bk_b1, bk_sh;  // per bucket (event index): [b0, b1) and shard offset
  std::vector<cudaEvent_t> ev_upd;           // ZeRO-1: shard update done (opt stream)
  int64_t stats_allreduce_calls = 0, stats_allreduce_bytes = 0;
  int64_t stats_plan_checks = 0;
  float* z0 = nullptr;
  char* x1 = nullptr;
  float2* st0 = nullptr;
  std::vector<LayerBufs> lb;
  std::vector<char*> y;
  char* hp = nullptr;         // pooled (cls) or LM: LNf output hf
  float* logits = nullptr;
  float2 *lm_stf = nullptr, *lm_tok = nullptr;   // LM head: LNf stats, per-token (lse, nll)
  // encoder-decoder: the two stacks' lengths / ids, the encoder output bundle, decoder buffers
  int Ss = 0, St = 0;
  int32_t *ids_src = nullptr, *ids_tgt = nullptr, *lens_src = nullptr, *lens_tgt = nullptr;
  char *enc_out = nullptr, *x1t = nullptr;
  float2* enc_st = nullptr;
  std::vector<DecBufs> dlb;
  int64_t it = 0;             // dropout step counter (forward calls)
  int64_t adam_t = 0;

  // Mimose
  int phase = MIMOSE_PHASE_SHELTERED;
  std::vector<Sample> samples;
  std::vector<int64_t> seen_x;
  Estimator est;
  std::unordered_map<int64_t, mimose_plan_t> cache;
  mimose_stats stats{};
  std::vector<cudaEvent_t> ev_t0, ev_t1;
  bool pending_times = false;
  // GEMM probe (roofline): event pairs around probed launches
  int probe = 0;
  std::vector<cudaEvent_t> probe_ev;
  size_t probe_used = 0;
  double probe_flops = 0.0;
  std::vector<std::array<int64_t, 4>> probe_shape;   // per probed launch: M, N, K, epi (grouped: -1)
};

namespace {

mimose_status fail(mimose_ctx* c, mimose_status s, const std::string& msg) {
  if (c) {
    c->err = msg;
    if (s == MIMOSE_E_CUDA || s == MIMOSE_E_NCCL) c->sticky = s;
  }
  return s;
}

#define CK(x)                                                                               \
  do {                                                                                      \
    cudaError_t e_ = (x);                                                                   \
    if (e_ != cudaSuccess) return fail(c, MIMOSE_E_CUDA, std::string(#x ": ") + cudaGetErrorString(e_)); \
  } while (0)
#define NK(x)                                                                               \
  do {                                                                                      \
    ncclResult_t r_ = (x);                                                                  \
    if (r_ != ncclSuccess) return fail(c, MIMOSE_E_NCCL, std::string(#x ": ") + ncclGetErrorString(r_)); \
  } while (0)

// ---------------------------------------------------------------- sizes ---
// Exactly DESIGN "Memory model" (and oracle/memsim.py, written independently).
struct Sz {
  int64_t z0, st0, x1;
  int64_t qkv, O, lse, z1, st1, h1, u, g, z2, st2;
  int64_t y;
  int64_t head0, head1, head2;   // QA: logits; cls: pooled, logits; LM: hf, stf, tokstat
  int64_t head_fwd;               // LM: fp32 logits chunk during the head forward
  int64_t dy, head_scr, layer_scr, emb_scr;
  // pre-LN (GPT-2) internals
  int64_t a, r1, m;
  int64_t r_dres, r_du, r_dt;  // carve offsets inside layer scratch
};

Sz sizes(const mimose_ctx* c, int B, int S) {
  const int64_t T = (int64_t)B * S, H = c->cfg.hidden, F = c->cfg.ffn, h = c->cfg.heads, e = c->e;
  Sz z{};
  const bool pre = c->cfg.arch != 0;
  z.z0 = a16(T * H * 4); z.st0 = a16(T * 8); z.x1 = pre ? a16(T * H * 4) : a16(T * H * e);
  z.a = a16(T * H * e); z.r1 = a16(T * H * 4); z.m = a16(T * H * e);
  z.qkv = a16(T * 3 * H * e); z.O = a16(T * H * e); z.lse = a16((int64_t)B * h * S * 4);
  z.z1 = a16(T * H * 4); z.st1 = a16(T * 8); z.h1 = a16(T * H * e);
  z.u = a16(T * F * e); z.g = a16(T * F * e); z.z2 = a16(T * H * 4); z.st2 = a16(T * 8);
  z.y = pre ? a16(T * H * 4) : a16(T * H * e);
  z.head2 = 0;
  z.head_fwd = 0;
  if (c->cfg.head == 3) {                     // LM head (GPT-2)
    const int64_t VP = vpad(c->cfg.vocab);
    z.head0 = a16(T * H * e); z.head1 = a16(T * 8); z.head2 = a16(T * 8);
    z.head_fwd = a16((int64_t)LM_CHUNK * VP * 4);
    z.head_scr = a16((int64_t)LM_CHUNK * VP * 4) + a16((int64_t)LM_CHUNK * VP * e);
  } else if (c->cfg.head == MIMOSE_HEAD_QA) {
    z.head0 = a16(T * 2 * 4); z.head1 = 0;
    z.head_scr = a16(T * 2 * 4);
  } else {
    const int64_t no = c->cfg.head == MIMOSE_HEAD_MC ? 1 : c->cfg.n_labels;
    z.head0 = a16((int64_t)B * H * e); z.head1 = a16((int64_t)B * no * 4);
    z.head_scr = a16((int64_t)B * no * 4) + 2 * a16((int64_t)B * H * 4);
  }
  z.dy = a16(T * H * 4);
  z.r_dres = 0;
  z.r_du = a16(T * H * 4);
  z.r_dt = z.r_du + a16(T * F * e);
  z.layer_scr = z.r_dt + a16(T * 3 * H * e) + a16((int64_t)B * h * S * 4);
  const int64_t maxT = (int64_t)c->cfg.max_seqs * c->cfg.max_seq_len;
  const int64_t ntiles = (maxT + 1023) / 1024;
  z.emb_scr = a16(T * H * 4) + a16(16 * T) + a16(4 * 256 * ntiles);
  return z;
}

int64_t persistent_bytes(const mimose_ctx* c) {
  const int64_t H = c->cfg.hidden, F = c->cfg.ffn;
  int64_t C = a16(c->npad * c->e) + a16(c->npad * 4) + 2 * a16(c->nshard * 4);   // w, grad, m, v
  if (c->dt != DT_F32) C += a16(c->nshard * 4);                                  // master
  const int64_t maxT = (int64_t)c->cfg.max_seqs * c->cfg.max_seq_len;
  C += 2 * a16(maxT * 4) + a16((int64_t)c->cfg.max_seqs * 4) + a16(2LL * c->cfg.max_seqs * 4);
  C += a16(256);
  C += a16(c->ws_elems * 4);                                   // wgrad split-K workspace
  C += a16((int64_t)NPART * 2 * std::max(3 * H, F) * 4);
  return C;
}

Drop make_drop(const mimose_ctx* c, uint32_t kind, uint32_t layer) {
  Drop d{};
  const double p = c->cfg.p_drop;
  d.enabled = p > 0.0;
  d.seed_lo = (uint32_t)(c->cfg.seed & 0xFFFFFFFFu);
  d.seed_hi = (uint32_t)(c->cfg.seed >> 32);
  d.site = site_word(kind, layer, (uint32_t)c->cfg.rank);
  d.step = (uint32_t)c->it;
  d.thresh = d.enabled ? (uint32_t)std::floor((1.0 - p) * 4294967296.0) : 0xFFFFFFFFu;
  d.scale = d.enabled ? (float)(1.0 / (1.0 - p)) : 1.0f;
  drop_set_keys(d);
  return d;
}
Drop no_drop() { Drop d{}; d.enabled = 0; return d; }

inline char* W(mimose_ctx* c, int i) { return c->w + c->layout[i].off * c->e; }
// FFN width of layer l (heterogeneous stages: mimose_config.ffn_layers).
inline int Fl(const mimose_ctx* c, int l) { return c->ffn_l.empty() ? c->cfg.ffn : c->ffn_l[l]; }

// Off-critical-path reductions: fork() orders the side stream after the work
// issued so far on `st` and returns it; join() makes `st` wait for everything
// issued on the side stream (called before a buffer the side stream reads or
// writes is reused: the LN partials, the bias-colsum partials, R2 / R3).
// MIMOSE_AUX=0 keeps every reduction on the compute stream (A/B).
bool aux_enabled(const mimose_ctx* c) {
  static const int v = [] {
    const char* e = std::getenv("MIMOSE_AUX");
    return e ? std::atoi(e) : 1;
  }();
  return v != 0 && c->aux_st != nullptr;
}
cudaStream_t fork(mimose_ctx* c, cudaStream_t st) {
  if (!aux_enabled(c)) return st;
  cudaEventRecord(c->ev_fork, st);
  cudaStreamWaitEvent(c->aux_st, c->ev_fork, 0);
  c->aux_pending = true;
  return c->aux_st;
}
void join(mimose_ctx* c, cudaStream_t st) {
  if (!c->aux_pending) return;
  cudaEventRecord(c->ev_join, c->aux_st);
  cudaStreamWaitEvent(st, c->ev_join, 0);
  c->aux_pending = false;
}
// Weight-gradient GEMMs of the post-LN layer on the side stream too, beside the
// next dgrad (MIMOSE_AUX_WGRAD=0: on the compute stream).
bool aux_wgrad(const mimose_ctx* c) {
  static const int v = [] {
    const char* e = std::getenv("MIMOSE_AUX_WGRAD");
    return e ? std::atoi(e) : 1;
  }();
  return v != 0 && aux_enabled(c) && c->dt == DT_BF16 && c->cfg.use_tc;
}
// The LN partials use the first NPART x max(3H, F) floats of c->part, the
// bias column-sum partials the second.
inline float* part_cs(const mimose_ctx* c) {
  return c->part + (int64_t)NPART * std::max<int64_t>(3LL * c->cfg.hidden, (int64_t)c->cfg.ffn);
}
inline float* G(mimose_ctx* c, int i) { return c->grad + c->layout[i].off; }
// Parameter index of semantic slot k (L_*) of layer l.  Post-LN order is the
// L_* enum order; GPT-2 (pre-LN) stores [ln1, qkv, o, ln2, f1, f2].
inline int layer_base(const mimose_ctx* c) { return c->cfg.arch != 0 ? 2 : P_LAYER0; }
inline int LP(mimose_ctx* c, int l, int k) {
  static const int pre_pos[12] = {2, 3, 4, 5, 0, 1, 8, 9, 10, 11, 6, 7};
  return layer_base(c) + 12 * l + (c->cfg.arch != 0 ? pre_pos[k] : k);
}
inline int HP(mimose_ctx* c, int k) {
  if (c->cfg.arch == 2) return 2 + 12 * c->cfg.n_layers + 2 + 20 * c->cfg.n_dec_layers + k;   // decoder final LN
  return layer_base(c) + 12 * c->cfg.n_layers + k;
}
// Checkpoint units: L layers, or 2L sub-layer blocks (granularity 1).
inline int n_units(const mimose_ctx* c) {
  return (c->cfg.granularity == 1 ? 2 * c->cfg.n_layers : c->cfg.n_layers) + (c->cfg.arch == 2 ? c->cfg.n_dec_layers : 0);
}

// ------------------------------------------------------------- probe ------
bool probe_begin(mimose_ctx* c, cudaStream_t st) {
  const bool on = c->probe == 1 && c->device;
  if (on) {
    if (c->probe_used + 2 > c->probe_ev.size()) {
      for (int i = 0; i < 256; ++i) {
        cudaEvent_t e;
        cudaEventCreate(&e);
        c->probe_ev.push_back(e);
      }
    }
    cudaEventRecord(c->probe_ev[c->probe_used], st);
  }
  return on;
}
void probe_end(mimose_ctx* c, cudaStream_t st, double flops, std::array<int64_t, 4> shape) {
  cudaEventRecord(c->probe_ev[c->probe_used + 1], st);
  c->probe_used += 2;
  c->probe_flops += flops;
  c->probe_shape.push_back(shape);
}
void pgemm(mimose_ctx* c, Epi epi, const GemmArgs& g, cudaStream_t st) {
  const bool on = probe_begin(c, st);
  gemm(c->dt, epi, g, st, c->cfg.use_tc != 0);
  if (on) probe_end(c, st, 2.0 * g.M * (double)g.N * g.K, {g.M, g.N, g.K, (int64_t)epi});
}

// ------------------------------------------------------------- schedule ---
// `real` = launch kernels; otherwise only the arena accounting runs.

struct Run {
  mimose_ctx* c;
  bool real;
  Sz z;
  cudaStream_t st;
};

// Attention block of a post-LN layer: x -> QKV, O, LSE, z1, st1 -> h1 = LN1(z1).
// h1out == nullptr (sub-layer recompute after h1 was released): the LN1 output
// store is gated off, the statistics are still written.
void att_forward(Run& r, int l, const char* x, LayerBufs& b, char* h1out) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  const int T = c->T, H = c->cfg.hidden;
  GemmArgs g;
  // QKV = x Wqkv^T + b
  g = GemmArgs();
  g.M = T; g.N = 3 * H; g.K = H;
  g.A = x; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, LP(c, l, L_QKVW)); g.b_sn = H; g.b_sk = 1;
  g.C = b.qkv; g.ldc = 3 * H; g.bias = W(c, LP(c, l, L_QKVB));
  pgemm(c, EPI_BIAS, g, r.st);
  attn_fwd(c->dt, b.qkv, c->lens, b.O, b.lse, c->B, c->S, H, c->cfg.heads, make_drop(c, KIND_ATTN_PROBS, l), r.st);
  // z1 = x + drop(O Wo^T + bo)
  g = GemmArgs();
  g.M = T; g.N = H; g.K = H;
  g.A = b.O; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, LP(c, l, L_OW)); g.b_sn = H; g.b_sk = 1;
  g.C = b.z1; g.ldc = H; g.bias = W(c, LP(c, l, L_OB)); g.res = x; g.ldr = H;
  g.drop = make_drop(c, KIND_ATTN_OUT, l);
  pgemm(c, EPI_BIAS_DROP_RES, g, r.st);
  ln_fwd(c->dt, b.z1, W(c, LP(c, l, L_LN1G)), W(c, LP(c, l, L_LN1B)), h1out, b.st1, T, H, c->cfg.ln_eps, r.st);
}

// FFN block: h1 (b.h1) -> u, g, z2, st2 -> y = LN2(z2) (store gated off when yout == nullptr).
void ffn_forward(Run& r, int l, LayerBufs& b, char* yout) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  const int T = c->T, H = c->cfg.hidden, F = Fl(c, l);
  GemmArgs g;
  // u = h1 W1^T + b1, g = gelu(u)
  g = GemmArgs();
  g.M = T; g.N = F; g.K = H;
  g.A = b.h1; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, LP(c, l, L_F1W)); g.b_sn = H; g.b_sk = 1;
  g.C = b.u; g.C2 = b.g; g.ldc = F; g.bias = W(c, LP(c, l, L_F1B));
  pgemm(c, EPI_BIAS_GELU, g, r.st);
  // z2 = h1 + drop(g W2^T + b2)
  g = GemmArgs();
  g.M = T; g.N = H; g.K = F;
  g.A = b.g; g.a_sm = F; g.a_sk = 1;
  g.B = W(c, LP(c, l, L_F2W)); g.b_sn = F; g.b_sk = 1;
  g.C = b.z2; g.ldc = H; g.bias = W(c, LP(c, l, L_F2B)); g.res = b.h1; g.ldr = H;
  g.drop = make_drop(c, KIND_FFN_OUT, l);
  pgemm(c, EPI_BIAS_DROP_RES, g, r.st);
  // y = LN2(z2); the store is gated off during recompute (yout == nullptr)
  ln_fwd(c->dt, b.z2, W(c, LP(c, l, L_LN2G)), W(c, LP(c, l, L_LN2B)), yout, b.st2, T, H, c->cfg.ln_eps, r.st);
}

void layer_forward(Run& r, int l, const char* x, LayerBufs& b, char* yout) {
  att_forward(r, l, x, b, b.h1);
  ffn_forward(r, l, b, yout);
}

void alloc_internals(Run& r, LayerBufs& b, bool on_stack) {
  Arena& a = r.c->ar;
  auto al = [&](int64_t n) { return on_stack ? a.push(n) : a.talloc(n); };
  if (r.c->cfg.arch != 0) {   // [a, st1, QKV, O, LSE, r1, st2, m, u, g]
    b.a = al(r.z.a); b.st1 = (float2*)al(r.z.st1); b.qkv = al(r.z.qkv); b.O = al(r.z.O);
    b.lse = (float*)al(r.z.lse); b.r1 = (float*)al(r.z.r1); b.st2 = (float2*)al(r.z.st2); b.m = al(r.z.m);
    b.u = al(r.z.u); b.g = al(r.z.g);
    return;
  }
  b.qkv = al(r.z.qkv); b.O = al(r.z.O); b.lse = (float*)al(r.z.lse);
  b.z1 = (float*)al(r.z.z1); b.st1 = (float2*)al(r.z.st1); b.h1 = al(r.z.h1);
  b.u = al(r.z.u); b.g = al(r.z.g); b.z2 = (float*)al(r.z.z2); b.st2 = (float2*)al(r.z.st2);
}
// Sub-layer units (granularity 1, post-LN; DESIGN reading A30): the attention
// block's internals [QKV, O, LSE, z1, st1] and the FFN block's [u, g, z2, st2],
// in the layer's push order (h1 sits between them).
// Pre-LN (GPT-2): attention [a, st1, QKV, O, LSE] -> r1, FFN [st2, m, u, g] -> y.
void alloc_att(Run& r, LayerBufs& b, bool on_stack) {
  Arena& a = r.c->ar;
  auto al = [&](int64_t n) { return on_stack ? a.push(n) : a.talloc(n); };
  if (r.c->cfg.arch != 0) {
    b.a = al(r.z.a); b.st1 = (float2*)al(r.z.st1); b.qkv = al(r.z.qkv); b.O = al(r.z.O);
    b.lse = (float*)al(r.z.lse);
    return;
  }
  b.qkv = al(r.z.qkv); b.O = al(r.z.O); b.lse = (float*)al(r.z.lse);
  b.z1 = (float*)al(r.z.z1); b.st1 = (float2*)al(r.z.st1);
}
void free_att(Run& r, bool on_stack) {
  Arena& a = r.c->ar;
  const int64_t s0[5] = {r.z.qkv, r.z.O, r.z.lse, r.z.z1, r.z.st1};
  const int64_t s1[5] = {r.z.a, r.z.st1, r.z.qkv, r.z.O, r.z.lse};
  const int64_t* s = r.c->cfg.arch != 0 ? s1 : s0;
  for (int i = 4; i >= 0; --i) on_stack ? a.pop(s[i]) : a.tfree(s[i]);
}
void alloc_ffn(Run& r, LayerBufs& b, bool on_stack) {
  Arena& a = r.c->ar;
  auto al = [&](int64_t n) { return on_stack ? a.push(n) : a.talloc(n); };
  if (r.c->cfg.arch != 0) {
    b.st2 = (float2*)al(r.z.st2); b.m = al(r.z.m); b.u = al(r.z.u); b.g = al(r.z.g);
    return;
  }
  b.u = al(r.z.u); b.g = al(r.z.g); b.z2 = (float*)al(r.z.z2); b.st2 = (float2*)al(r.z.st2);
}
void free_ffn(Run& r, bool on_stack) {
  Arena& a = r.c->ar;
  const int64_t s0[4] = {r.z.u, r.z.g, r.z.z2, r.z.st2};
  const int64_t s1[4] = {r.z.st2, r.z.m, r.z.u, r.z.g};
  const int64_t* s = r.c->cfg.arch != 0 ? s1 : s0;
  for (int i = 3; i >= 0; --i) on_stack ? a.pop(s[i]) : a.tfree(s[i]);
}

// Per-layer sizes: only the FFN internals u, g depend on the layer (its FFN
// width F_l, heterogeneous stages); the layer scratch is sized for max F.
void set_layer(Run& r, int l) {
  const int64_t T = (int64_t)r.c->B * r.c->S;
  r.z.u = r.z.g = a16(T * Fl(r.c, l) * r.c->e);
}

void free_internals(Run& r, bool on_stack) {
  Arena& a = r.c->ar;
  const int64_t s0[10] = {r.z.qkv, r.z.O, r.z.lse, r.z.z1, r.z.st1, r.z.h1, r.z.u, r.z.g, r.z.z2, r.z.st2};
  const int64_t s1[10] = {r.z.a, r.z.st1, r.z.qkv, r.z.O, r.z.lse, r.z.r1, r.z.st2, r.z.m, r.z.u, r.z.g};
  const int64_t* s = r.c->cfg.arch != 0 ? s1 : s0;
  for (int i = 9; i >= 0; --i) on_stack ? a.pop(s[i]) : a.tfree(s[i]);
}

void wgrad(Run& r, const void* dY, int N, const void* X, int K, float* out) {
  // dW[N, K] = sum_t dY[t, n] X[t, k]; deterministic split-K over t.
  mimose_ctx* c = r.c;
  const int T = c->T;
  const int tiles = ((N + 127) / 128) * ((K + 127) / 128);
  int split = std::max(1, std::min(4, 148 / std::max(1, tiles)));
  while (split > 1 && (int64_t)split * N * K > c->ws_elems) --split;
  while (split > 1 && T / split < 64) --split;
  GemmArgs g;
  g.M = N; g.N = K; g.K = T;
  g.A = dY; g.a_sm = 1; g.a_sk = N;
  g.B = X; g.b_sn = 1; g.b_sk = K;
  g.ldc = K;
  g.split = split;
  if (split == 1) {
    g.C = out;
    pgemm(c, EPI_F32, g, r.st);
  } else {
    g.C = c->ws; g.split_stride = (int64_t)N * K;
    pgemm(c, EPI_F32, g, r.st);
    splitk_reduce(c->ws, split, (int64_t)N * K, out, r.st);
  }
}

// dW1 = dY1^T X1 and dW2 = dY2^T X2 (both deterministic, fp32 out): one grouped
// tcgen05 launch with 128 x bn tiles when the two fit one wave of SMs (BERT-base:
// the FFN pair 72 + 72 tiles at bn 256, the attention pair 36 + 108 at bn 128;
// H = 1024: the attention pair 32 + 96 at bn 256), else two wgrad() calls.
void wgrad2(Run& r, const void* dY1, int N1, const void* X1, int K1, float* out1, const void* dY2, int N2,
            const void* X2, int K2, float* out2, int bn = 0) {
  mimose_ctx* c = r.c;
  const int T = c->T;
  if (bn == 0) {
    // tile width: the one whose single wave keeps more SMs busy, weighting a
    // 128-wide tile at 0.58 of a 256-wide one (its measured mainloop rate);
    // more tiles than SMs cannot be grouped (-> two launches)
    auto tiles = [&](int w) {
      return (K1 % w || K2 % w) ? 1 << 30 : ((N1 + 127) / 128) * (K1 / w) + ((N2 + 127) / 128) * (K2 / w);
    };
    const double e256 = tiles(256) <= 148 ? tiles(256) : 0.0, e128 = tiles(128) <= 148 ? 0.58 * tiles(128) : 0.0;
    bn = e256 >= e128 ? 256 : 128;
  }
  if (c->dt == DT_BF16 && c->cfg.use_tc && K1 % bn == 0 && K2 % bn == 0) {
    GemmArgs g[2];
    const void* dY[2] = {dY1, dY2};
    const void* X[2] = {X1, X2};
    const int N[2] = {N1, N2}, K[2] = {K1, K2};
    float* out[2] = {out1, out2};
    for (int i = 0; i < 2; ++i) {
      g[i].M = N[i]; g[i].N = K[i]; g[i].K = T;
      g[i].A = dY[i]; g[i].a_sm = 1; g[i].a_sk = N[i];
      g[i].B = X[i]; g[i].b_sn = 1; g[i].b_sk = K[i];
      g[i].C = out[i]; g[i].ldc = K[i];
    }
    const bool on = probe_begin(c, r.st);
    const bool done = gemm_tc_grouped(g[0], g[1], bn, r.st);
    if (on) {
      if (done) probe_end(c, r.st, 2.0 * T * ((double)N1 * K1 + (double)N2 * K2), {T, N1 * K1 + N2 * K2, bn, -1});
      else cudaEventRecord(c->probe_ev[c->probe_used + 1], r.st);
    }
    if (done) {
      note_launch(1);
      return;
    }
  }
  wgrad(r, dY1, N1, X1, K1, out1);
  wgrad(r, dY2, N2, X2, K2, out2);
}

void dgrad(Run& r, Epi epi, const void* dY, int Nout, const void* Wt, int Kin, void* out, const void* res_or_aux) {
  mimose_ctx* c = r.c;
  GemmArgs g;
  g.M = c->T; g.N = Kin; g.K = Nout;
  g.A = dY; g.a_sm = Nout; g.a_sk = 1;
  g.B = Wt; g.b_sn = 1; g.b_sk = Kin;
  g.C = out; g.ldc = Kin;
  if (epi == EPI_GELU_BWD) { g.aux = res_or_aux; g.ldx = Kin; }
  if (epi == EPI_ACC_RES_F32) { g.res = res_or_aux; g.ldr = Kin; }
  pgemm(c, epi, g, r.st);
}

// FFN-block gradients of a post-LN layer: dy -> dz2 -> ... -> dres = dh1;
// scratch carve: dres (dz / dh1), R2 (du, later dO), R3 (dt2 / dt1, later dQKV).
void ffn_backward(Run& r, int l, LayerBufs& b, float* dy, char* scr) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  const int T = c->T, H = c->cfg.hidden, F = Fl(c, l);
  float* dres = (float*)(scr + r.z.r_dres);
  char* R2 = scr + r.z.r_du;     // du, later dO
  char* R3 = scr + r.z.r_dt;     // dt2 / dt1, later dQKV
  float* pg = c->part;
  float* pb = c->part + (int64_t)NPART * H;
  float* pbias = c->part + 2LL * NPART * H;
  join(c, r.st);                 // the previous layer's side reductions read R3 and the partials
  // LN2 backward + dropout backward -> dz2 (dres), dt2 (R3), partials
  ln_bwd(c->dt, dy, no_drop(), b.z2, b.st2, W(c, LP(c, l, L_LN2G)), dres, R3, make_drop(c, KIND_FFN_OUT, l),
         pg, pb, pbias, T, H, r.st);
  reduce_rows3(pg, G(c, LP(c, l, L_LN2G)), pb, G(c, LP(c, l, L_LN2B)), pbias, G(c, LP(c, l, L_F2B)), NPART, H, H,
               fork(c, r.st));
  // FFN2: du = (dt2 W2) * gelu'(u)
  dgrad(r, EPI_GELU_BWD, R3, H, W(c, LP(c, l, L_F2W)), F, R2, b.u);
  // db1 = colsum du and (aux_wgrad) the weight gradients dW2 = dt2^T g, dW1 = du^T h1
  // on the side stream, beside the FFN1 dgrad (dt2 in R3 lives until LN1 backward)
  {
    cudaStream_t sa = fork(c, r.st);
    colsum(c->dt, R2, T, F, part_cs(c), sa);
    reduce_partials(part_cs(c), F, F, G(c, LP(c, l, L_F1B)), sa);
    if (aux_wgrad(c)) {
      Run ra = r;
      ra.st = sa;
      wgrad2(ra, R3, H, b.g, F, G(c, LP(c, l, L_F2W)), R2, F, b.h1, H, G(c, LP(c, l, L_F1W)));
    }
  }
  // FFN1: dh1 = du W1 + dz2 (in place in dres)
  dgrad(r, EPI_ACC_RES_F32, R2, F, W(c, LP(c, l, L_F1W)), H, dres, dres);
  if (!aux_wgrad(c)) wgrad2(r, R3, H, b.g, F, G(c, LP(c, l, L_F2W)), R2, F, b.h1, H, G(c, LP(c, l, L_F1W)));
}

// Attention-block gradients of a post-LN layer (after ffn_backward; dres = dh1).
void att_backward(Run& r, int l, const char* x, LayerBufs& b, float* dy, char* scr) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  const int T = c->T, H = c->cfg.hidden, h = c->cfg.heads;
  float* dres = (float*)(scr + r.z.r_dres);
  char* R2 = scr + r.z.r_du;
  char* R3 = scr + r.z.r_dt;
  float* Dbuf = (float*)(scr + r.z.r_dt + a16((int64_t)T * 3 * H * c->e));
  float* pg = c->part;
  float* pb = c->part + (int64_t)NPART * H;
  float* pbias = c->part + 2LL * NPART * H;
  // dt1 goes to the spare tail of R2 (R2 holds T x F, dO uses its first T x H) so
  // that it outlives the attention backward and dWo can be grouped with dWqkv
  const bool spare = c->cfg.ffn >= 2 * H;
  char* DT1 = spare ? R2 + a16((int64_t)T * H * c->e) : R3;
  join(c, r.st);                 // LN2 partials reduced and du summed before LN1 / dO reuse them
  // LN1 backward + dropout backward -> dz1 (dres, in place), dt1 (DT1)
  ln_bwd(c->dt, dres, no_drop(), b.z1, b.st1, W(c, LP(c, l, L_LN1G)), dres, DT1, make_drop(c, KIND_ATTN_OUT, l),
         pg, pb, pbias, T, H, r.st);
  reduce_rows3(pg, G(c, LP(c, l, L_LN1G)), pb, G(c, LP(c, l, L_LN1B)), pbias, G(c, LP(c, l, L_OB)), NPART, H, H,
               fork(c, r.st));
  // out-proj: dO = dt1 Wo (R2)
  dgrad(r, EPI_STORE, DT1, H, W(c, LP(c, l, L_OW)), H, R2, nullptr);
  if (!spare) wgrad(r, DT1, H, b.O, H, G(c, LP(c, l, L_OW)));     // dWo = dt1^T O before R3 is reused
  // attention backward -> dQKV (R3)
  attn_bwd(c->dt, b.qkv, b.O, R2, b.lse, c->lens, Dbuf, R3, c->B, c->S, H, h, make_drop(c, KIND_ATTN_PROBS, l), r.st);
  // dbqkv = colsum dQKV and (aux_wgrad) dWo = dt1^T O with dWqkv = dQKV^T x on the
  // side stream, beside the QKV dgrad
  const bool side_w = spare && aux_wgrad(c);
  {
    cudaStream_t sa = fork(c, r.st);
    colsum(c->dt, R3, T, 3 * H, part_cs(c), sa);
    reduce_partials(part_cs(c), 3 * H, 3 * H, G(c, LP(c, l, L_QKVB)), sa);
    if (side_w) {
      Run ra = r;
      ra.st = sa;
      wgrad2(ra, DT1, H, b.O, H, G(c, LP(c, l, L_OW)), R3, 3 * H, x, H, G(c, LP(c, l, L_QKVW)));
    }
  }
  // QKV: dx = dQKV Wqkv + dz1 -> dy buffer
  dgrad(r, EPI_ACC_RES_F32, R3, 3 * H, W(c, LP(c, l, L_QKVW)), H, dy, dres);
  // dWo = dt1^T O and dWqkv = dQKV^T x
  if (spare && !side_w)
    wgrad2(r, DT1, H, b.O, H, G(c, LP(c, l, L_OW)), R3, 3 * H, x, H, G(c, LP(c, l, L_QKVW)));
  else if (!spare)
    wgrad(r, R3, 3 * H, x, H, G(c, LP(c, l, L_QKVW)));
}

void layer_backward(Run& r, int l, const char* x, LayerBufs& b, float* dy, char* scr) {
  ffn_backward(r, l, b, dy, scr);
  att_backward(r, l, x, b, dy, scr);
}

// ---------------------------------------------------------------------------
// GPT-2 pre-LN layer (causal): a = LN1(x); r1 = x + drop(Attn(a) Wo + bo);
// m = LN2(r1); y = r1 + drop(gelu_tanh(m W1 + b1) W2 + b2).  x, r1, y fp32.
// In recompute (yout == nullptr) the FFN2 GEMM is skipped: y is not needed.
// ---------------------------------------------------------------------------
// Attention block of a pre-LN layer: x -> a = LN1(x), QKV, O, LSE -> r1 = x + drop(O Wo^T + bo).
// r1out == nullptr (sub-layer recompute after r1 was released): the out-proj GEMM is skipped.
void att_forward_pre(Run& r, int l, const float* x, LayerBufs& b, float* r1out) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  const int T = c->T, H = c->cfg.hidden;
  ln_fwd(c->dt, x, W(c, LP(c, l, L_LN1G)), W(c, LP(c, l, L_LN1B)), b.a, b.st1, T, H, c->cfg.ln_eps, r.st);
  GemmArgs g;
  g.M = T; g.N = 3 * H; g.K = H;
  g.A = b.a; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, LP(c, l, L_QKVW)); g.b_sn = H; g.b_sk = 1;
  g.C = b.qkv; g.ldc = 3 * H; g.bias = W(c, LP(c, l, L_QKVB));
  pgemm(c, EPI_BIAS, g, r.st);
  attn_fwd(c->dt, b.qkv, c->lens, b.O, b.lse, c->B, c->S, H, c->cfg.heads, make_drop(c, KIND_ATTN_PROBS, l), r.st,
           c->cfg.arch == 1);   // GPT-2 causal; the encoder-decoder's encoder is bidirectional
  if (!r1out) return;
  g = GemmArgs();
  g.M = T; g.N = H; g.K = H;
  g.A = b.O; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, LP(c, l, L_OW)); g.b_sn = H; g.b_sk = 1;
  g.C = r1out; g.ldc = H; g.bias = W(c, LP(c, l, L_OB)); g.res = x; g.ldr = H;
  g.drop = make_drop(c, KIND_ATTN_OUT, l);
  pgemm(c, EPI_BIAS_DROP_RESF32, g, r.st);
}

// FFN block of a pre-LN layer: r1 (b.r1) -> m = LN2(r1), u, g -> y = r1 + drop(g W2^T + b2);
// yout == nullptr (recompute): the FFN2 GEMM is skipped, y is not needed.
void ffn_forward_pre(Run& r, int l, LayerBufs& b, float* yout) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  const int T = c->T, H = c->cfg.hidden, F = Fl(c, l);
  GemmArgs g;
  ln_fwd(c->dt, b.r1, W(c, LP(c, l, L_LN2G)), W(c, LP(c, l, L_LN2B)), b.m, b.st2, T, H, c->cfg.ln_eps, r.st);
  g = GemmArgs();
  g.M = T; g.N = F; g.K = H;
  g.A = b.m; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, LP(c, l, L_F1W)); g.b_sn = H; g.b_sk = 1;
  g.C = b.u; g.C2 = b.g; g.ldc = F; g.bias = W(c, LP(c, l, L_F1B));
  pgemm(c, EPI_BIAS_GELUT, g, r.st);
  if (!yout) return;
  g = GemmArgs();
  g.M = T; g.N = H; g.K = F;
  g.A = b.g; g.a_sm = F; g.a_sk = 1;
  g.B = W(c, LP(c, l, L_F2W)); g.b_sn = F; g.b_sk = 1;
  g.C = yout; g.ldc = H; g.bias = W(c, LP(c, l, L_F2B)); g.res = b.r1; g.ldr = H;
  g.drop = make_drop(c, KIND_FFN_OUT, l);
  pgemm(c, EPI_BIAS_DROP_RESF32, g, r.st);
}

void layer_forward_pre(Run& r, int l, const float* x, LayerBufs& b, float* yout) {
  att_forward_pre(r, l, x, b, b.r1);
  ffn_forward_pre(r, l, b, yout);
}

// FFN-block gradients of a pre-LN layer, through LN2: dy -> dr1 (in place), dt1 (R3).
void ffn_backward_pre(Run& r, int l, LayerBufs& b, float* dy, char* scr) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  const int T = c->T, H = c->cfg.hidden, F = Fl(c, l);
  float* dres = (float*)(scr + r.z.r_dres);
  char* R2 = scr + r.z.r_du;     // du, later dO
  char* R3 = scr + r.z.r_dt;     // dt2 / dt1, later dQKV
  float* Dbuf = (float*)(scr + r.z.r_dt + a16((int64_t)T * 3 * H * c->e));
  float* pg = c->part;
  float* pb = c->part + (int64_t)NPART * H;
  float* pbias = c->part + 2LL * NPART * H;
  join(c, r.st);                 // the previous layer's side reductions read R3 and the partials
  // dt2 = dy * mask (bf16), db2 = colsum dt2
  drop_cast_colsum(c->dt, dy, make_drop(c, KIND_FFN_OUT, l), R3, T, H, pbias, r.st);
  reduce_partials(pbias, H, H, G(c, LP(c, l, L_F2B)), fork(c, r.st));
  // FFN2: du = (dt2 W2) * gelu_tanh'(u); dW2 = dt2^T g
  {
    GemmArgs g;
    g.M = T; g.N = F; g.K = H;
    g.A = R3; g.a_sm = H; g.a_sk = 1;
    g.B = W(c, LP(c, l, L_F2W)); g.b_sn = 1; g.b_sk = F;
    g.C = R2; g.ldc = F; g.aux = b.u; g.ldx = F;
    pgemm(c, EPI_GELUT_BWD, g, r.st);
  }
  wgrad(r, R3, H, b.g, F, G(c, LP(c, l, L_F2W)));
  // FFN1: dm = du W1 (fp32, dres); dW1 = du^T m; db1
  dgrad(r, EPI_F32, R2, F, W(c, LP(c, l, L_F1W)), H, dres, nullptr);
  {
    cudaStream_t sa = fork(c, r.st);
    colsum(c->dt, R2, T, F, part_cs(c), sa);
    reduce_partials(part_cs(c), F, F, G(c, LP(c, l, L_F1B)), sa);
  }
  wgrad(r, R2, F, b.m, H, G(c, LP(c, l, L_F1W)));
  join(c, r.st);                 // pbias reduced, du summed before LN2 / DT1 reuse them
  // LN2 backward + residual: dr1 = dy + LN2'(dm) (in place in dy); dt1 = dr1 * mask (DT1: the
  // spare tail of R2 when F >= 2H, so it outlives the dQKV write into R3, else R3)
  char* DT1 = F >= 2 * H ? R2 + a16((int64_t)T * H * c->e) : R3;
  ln_bwd(c->dt, dres, no_drop(), b.r1, b.st2, W(c, LP(c, l, L_LN2G)), dy, DT1, make_drop(c, KIND_ATTN_OUT, l),
         pg, pb, pbias, T, H, r.st, dy);
  reduce_rows3(pg, G(c, LP(c, l, L_LN2G)), pb, G(c, LP(c, l, L_LN2B)), pbias, G(c, LP(c, l, L_OB)), NPART, H, H,
               fork(c, r.st));
}

// Attention-block gradients of a pre-LN layer (after ffn_backward_pre: dy = dr1, R3 = dt1).
void att_backward_pre(Run& r, int l, const float* x, LayerBufs& b, float* dy, char* scr) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  const int T = c->T, H = c->cfg.hidden, h = c->cfg.heads;
  float* dres = (float*)(scr + r.z.r_dres);
  char* R2 = scr + r.z.r_du;
  char* R3 = scr + r.z.r_dt;
  float* Dbuf = (float*)(scr + r.z.r_dt + a16((int64_t)T * 3 * H * c->e));
  float* pg = c->part;
  float* pb = c->part + (int64_t)NPART * H;
  const bool spare = c->cfg.ffn >= 2 * H;          // dt1 in the spare tail of R2 (ffn_backward_pre)
  char* DT1 = spare ? R2 + a16((int64_t)T * H * c->e) : R3;
  // out-proj: dO = dt1 Wo (R2)
  dgrad(r, EPI_STORE, DT1, H, W(c, LP(c, l, L_OW)), H, R2, nullptr);
  if (!spare) wgrad(r, DT1, H, b.O, H, G(c, LP(c, l, L_OW)));
  attn_bwd(c->dt, b.qkv, b.O, R2, b.lse, c->lens, Dbuf, R3, c->B, c->S, H, h, make_drop(c, KIND_ATTN_PROBS, l),
           r.st, c->cfg.arch == 1);
  // QKV: da = dQKV Wqkv (fp32, dres); dWo = dt1^T O with dWqkv = dQKV^T a (grouped); dbqkv on the side
  {
    cudaStream_t sa = fork(c, r.st);
    colsum(c->dt, R3, T, 3 * H, part_cs(c), sa);
    reduce_partials(part_cs(c), 3 * H, 3 * H, G(c, LP(c, l, L_QKVB)), sa);
  }
  dgrad(r, EPI_F32, R3, 3 * H, W(c, LP(c, l, L_QKVW)), H, dres, nullptr);
  if (spare)
    wgrad2(r, DT1, H, b.O, H, G(c, LP(c, l, L_OW)), R3, 3 * H, b.a, H, G(c, LP(c, l, L_QKVW)));
  else
    wgrad(r, R3, 3 * H, b.a, H, G(c, LP(c, l, L_QKVW)));
  join(c, r.st);                 // LN2 partials reduced before LN1's partials overwrite them
  // LN1 backward + residual: dx = dr1 + LN1'(da) (in place in dy)
  ln_bwd(c->dt, dres, no_drop(), x, b.st1, W(c, LP(c, l, L_LN1G)), dy, nullptr, no_drop(), pg, pb, nullptr, T, H,
         r.st, dy);
  reduce_rows3(pg, G(c, LP(c, l, L_LN1G)), pb, G(c, LP(c, l, L_LN1B)), nullptr, nullptr, NPART, H, H,
               fork(c, r.st));
}

void layer_backward_pre(Run& r, int l, const float* x, LayerBufs& b, float* dy, char* scr) {
  ffn_backward_pre(r, l, b, dy, scr);
  att_backward_pre(r, l, x, b, dy, scr);
}

// LM head (GPT-2): hf = LNf(y); chunks of LM_CHUNK tokens: logits = hf W_e^T (fp32),
// per-token (lse, nll); loss = sum nll / #targets.
void lm_head_forward(Run& r, float* yL, char* hf, float2* stf, float2* tok, float* logits) {
  mimose_ctx* c = r.c;
  const int T = c->T, H = c->cfg.hidden, V = c->cfg.vocab;
  const int64_t VP = vpad(V);
  ln_fwd(c->dt, yL, W(c, HP(c, 0)), W(c, HP(c, 1)), hf, stf, T, H, c->cfg.ln_eps, r.st);
  for (int r0 = 0; r0 < T; r0 += LM_CHUNK) {
    const int nc = std::min(LM_CHUNK, T - r0);
    GemmArgs g;
    g.M = nc; g.N = V; g.K = H;
    g.A = hf + (int64_t)r0 * H * c->e; g.a_sm = H; g.a_sk = 1;
    g.B = W(c, P_WORD); g.b_sn = H; g.b_sk = 1;
    g.C = logits; g.ldc = VP;
    pgemm(c, EPI_F32, g, r.st);
    lm_ce_fwd(logits, VP, V, r0, nc, c->ids, c->lens, c->S, tok, r.st);
  }
  lm_loss(tok, T, c->lens, c->B, c->S, c->misc, r.st);
}

// Backward of the LM head into dy (fp32 [T, H]); dW_e accumulates chunk by chunk.
void lm_head_backward(Run& r, float* yL, char* hf, float2* stf, float2* tok, char* scr, float* dy) {
  mimose_ctx* c = r.c;
  const int T = c->T, H = c->cfg.hidden, V = c->cfg.vocab;
  const int64_t VP = vpad(V);
  float* logits = (float*)scr;
  char* dlog = scr + a16((int64_t)LM_CHUNK * VP * 4);
  for (int r0 = 0; r0 < T; r0 += LM_CHUNK) {
    const int nc = std::min(LM_CHUNK, T - r0);
    GemmArgs g;
    g.M = nc; g.N = V; g.K = H;
    g.A = hf + (int64_t)r0 * H * c->e; g.a_sm = H; g.a_sk = 1;
    g.B = W(c, P_WORD); g.b_sn = H; g.b_sk = 1;
    g.C = logits; g.ldc = VP;
    pgemm(c, EPI_F32, g, r.st);                                  // recompute the chunk's logits
    lm_ce_bwd(c->dt, logits, VP, V, r0, nc, c->ids, c->lens, c->B, c->S, tok, dlog, r.st);
    // dh = dlog W_e: K = V but only nc/128 x H/256 output tiles, so the K range is
    // split in two (fp32 partials in the chunk's logits region, dead once dlog is
    // written; fixed-order sum): twice the tiles at the 256-wide tile rate.
    g = GemmArgs();
    g.M = nc; g.N = H; g.K = V;
    g.A = dlog; g.a_sm = VP; g.a_sk = 1;
    g.B = W(c, P_WORD); g.b_sn = 1; g.b_sk = H;
    g.C = logits; g.ldc = H;
    g.split = 2; g.split_stride = (int64_t)nc * H;
    pgemm(c, EPI_F32, g, r.st);
    splitk_reduce(logits, 2, (int64_t)nc * H, dy + (int64_t)r0 * H, r.st);
    g = GemmArgs();                                               // dW_e += dlog^T hf
    g.M = V; g.N = H; g.K = nc;
    g.A = dlog; g.a_sm = 1; g.a_sk = VP;
    g.B = hf + (int64_t)r0 * H * c->e; g.b_sn = 1; g.b_sk = H;
    g.C = G(c, P_WORD); g.ldc = H;
    pgemm(c, EPI_ACC_F32, g, r.st);
  }
  float* pg = c->part;
  float* pb = c->part + (int64_t)NPART * H;
  ln_bwd(c->dt, dy, no_drop(), yL, stf, W(c, HP(c, 0)), dy, nullptr, no_drop(), pg, pb, nullptr, T, H, r.st);
  reduce_rows3(pg, G(c, HP(c, 0)), pb, G(c, HP(c, 1)), nullptr, nullptr, NPART, H, H, r.st);
}

int64_t bucket_begin(mimose_ctx* c, int first_param) { return c->layout[first_param].off; }
int64_t bucket_end(mimose_ctx* c, int last_param) {
  return c->layout[last_param].off + (c->layout[last_param].numel + 63) / 64 * 64;
}

// A gradient bucket (params first..last) is final: all-reduce it (DP) on the
// comm stream and, with the fused optimizer, update it on the optimizer stream,
// both overlapping the rest of the backward.
// ZeRO-1: reduce-scatter the bucket (this rank's shard of the
// summed gradient lands in its own slice, in place), AdamW on that shard
// (master, m, v hold shards only), all-gather the updated working weights.
// `st_rs` runs the collectives, `st_opt` the update; the all-gather waits on it.
mimose_status zero_bucket(mimose_ctx* c, int evi, cudaStream_t st_rs, cudaStream_t st_opt, bool update) {
  const int W = c->cfg.world, r = c->cfg.rank;
  const int64_t b0 = c->bk_b0[evi], cb = (c->bk_b1[evi] - b0) / W, sh = c->bk_sh[evi];
  float* gsh = c->grad + b0 + r * cb;
  NK(ncclReduceScatter(c->grad + b0, gsh, (size_t)cb, ncclFloat, ncclSum, c->comm, st_rs));
  c->stats_allreduce_calls++;
  c->stats_allreduce_bytes += cb * W * 4;
  if (!update) return MIMOSE_OK;
  if (st_opt != st_rs) {
    CK(cudaEventRecord(c->ev_ar[evi], st_rs));
    CK(cudaStreamWaitEvent(st_opt, c->ev_ar[evi], 0));
  }
  const double t = (double)(c->adam_t + 1);
  const double bc1 = 1.0 - std::pow((double)c->opt_b1, t), bc2 = 1.0 - std::pow((double)c->opt_b2, t);
  char* wsh = c->w + (b0 + r * cb) * c->e;
  adamw(c->dt, wsh, c->master ? c->master + sh : nullptr, gsh, c->m + sh, c->v + sh, cb, c->opt_lr, c->opt_b1,
        c->opt_b2, c->opt_eps, c->opt_wd, (float)bc1, (float)bc2, 1.0f / (float)W, st_opt);
  if (st_opt != st_rs) {
    CK(cudaEventRecord(c->ev_upd[evi], st_opt));
    CK(cudaStreamWaitEvent(st_rs, c->ev_upd[evi], 0));
  }
  NK(ncclAllGather(wsh, c->w + b0 * c->e, (size_t)cb, c->dt == DT_F32 ? ncclFloat : ncclBfloat16, c->comm, st_rs));
  return MIMOSE_OK;
}

mimose_status allreduce_bucket(mimose_ctx* c, int first, int last, int evi) {
  if (!c->device || (!c->comm && !c->opt_fused)) return MIMOSE_OK;
  // the bucket is final once the compute stream AND the side reductions
  // (its bias / LN gradients) are done
  const bool side = c->aux_pending;
  if (side) CK(cudaEventRecord(c->ev_join, c->aux_st));
  if (c->zero1) {
    CK(cudaEventRecord(c->ev_layer[evi], c->st));
    CK(cudaStreamWaitEvent(c->comm_st, c->ev_layer[evi], 0));
    if (side) CK(cudaStreamWaitEvent(c->comm_st, c->ev_join, 0));
    return zero_bucket(c, evi, c->comm_st, c->opt_st, c->opt_fused);
  }
  const int64_t b0 = bucket_begin(c, first), b1 = bucket_end(c, last);
  CK(cudaEventRecord(c->ev_layer[evi], c->st));
  cudaEvent_t ready = c->ev_layer[evi];
  if (side) CK(cudaStreamWaitEvent(c->comm ? c->comm_st : c->opt_st, c->ev_join, 0));
  if (c->comm) {
    c->stats_allreduce_calls++;
    c->stats_allreduce_bytes += (b1 - b0) * 4;
    CK(cudaStreamWaitEvent(c->comm_st, c->ev_layer[evi], 0));
    NK(ncclAllReduce(c->grad + b0, c->grad + b0, (size_t)(b1 - b0), ncclFloat, ncclSum, c->comm, c->comm_st));
    CK(cudaEventRecord(c->ev_ar[evi], c->comm_st));
    ready = c->ev_ar[evi];
  }
  if (c->opt_fused) {
    CK(cudaStreamWaitEvent(c->opt_st, ready, 0));
    const double t = (double)(c->adam_t + 1);
    const double bc1 = 1.0 - std::pow((double)c->opt_b1, t), bc2 = 1.0 - std::pow((double)c->opt_b2, t);
    adamw(c->dt, c->w + b0 * c->e, c->master ? c->master + b0 : nullptr, c->grad + b0, c->m + b0, c->v + b0, b1 - b0,
          c->opt_lr, c->opt_b1, c->opt_b2, c->opt_eps, c->opt_wd, (float)bc1, (float)bc2, 1.0f / (float)c->cfg.world,
          c->opt_st);
  }
  return MIMOSE_OK;
}

mimose_status copy_batch(mimose_ctx* c, const mimose_batch* bt) {
  const int64_t T = (int64_t)bt->n_seqs * bt->seq_len;
  const cudaMemcpyKind k = bt->on_host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
  int nl;
  if (c->cfg.head == MIMOSE_HEAD_MC) nl = bt->n_seqs / c->cfg.n_choices;
  else if (c->cfg.head == MIMOSE_HEAD_QA) nl = 2 * bt->n_seqs;
  else if (c->cfg.head == 3) nl = 0;            // LM targets are the next input tokens
  else nl = bt->n_seqs;
  if (c->cfg.arch == 2) {   // source ids / lengths; decoder ids / lengths in the tt / labels buffers
    CK(cudaMemcpyAsync(c->ids_src, bt->input_ids, T * 4, k, c->st));
    CK(cudaMemcpyAsync(c->lens_src, bt->lengths, (int64_t)bt->n_seqs * 4, k, c->st));
    CK(cudaMemcpyAsync(c->ids_tgt, bt->dec_ids, (int64_t)bt->n_seqs * bt->dec_len * 4, k, c->st));
    CK(cudaMemcpyAsync(c->lens_tgt, bt->dec_lengths, (int64_t)bt->n_seqs * 4, k, c->st));
    return MIMOSE_OK;
  }
  CK(cudaMemcpyAsync(c->ids, bt->input_ids, T * 4, k, c->st));
  CK(cudaMemcpyAsync(c->tt, bt->token_type, T * 4, k, c->st));
  CK(cudaMemcpyAsync(c->lens, bt->lengths, (int64_t)bt->n_seqs * 4, k, c->st));
  if (nl) CK(cudaMemcpyAsync(c->labels, bt->labels, (int64_t)nl * 4, k, c->st));
  return MIMOSE_OK;
}

mimose_status check_batch(mimose_ctx* c, const mimose_batch* bt) {
  if (!bt || bt->n_seqs <= 0 || bt->seq_len <= 0 || bt->n_seqs > c->cfg.max_seqs || bt->seq_len > c->cfg.max_seq_len)
    return fail(c, MIMOSE_E_INVALID, "batch shape outside [1, max_seqs] x [1, max_seq_len]");
  if (c->cfg.head == MIMOSE_HEAD_MC && bt->n_seqs % c->cfg.n_choices)
    return fail(c, MIMOSE_E_INVALID, "MC batch: n_seqs must be a multiple of n_choices");
  if (bt->seq_len + c->cfg.pos_offset > c->cfg.max_pos)
    return fail(c, MIMOSE_E_INVALID, "seq_len + pos_offset exceeds max_pos");
  if (c->cfg.arch == 2 && (bt->dec_len <= 0 || bt->dec_len > c->cfg.max_seq_len ||
                           bt->dec_len + c->cfg.pos_offset > c->cfg.max_pos ||
                           (c->device && bt->input_ids && (!bt->dec_ids || !bt->dec_lengths))))
    return fail(c, MIMOSE_E_INVALID, "encoder-decoder batch: decoder ids / lengths / dec_len in [1, max_seq_len]");
  return MIMOSE_OK;
}

void layer_fwd_any(Run& r, int l, const char* x, LayerBufs& b, char* yout) {
  Range rg(yout ? "layer fwd" : "layer recompute", l);
  if (r.c->cfg.arch != 0) layer_forward_pre(r, l, (const float*)x, b, (float*)yout);
  else layer_forward(r, l, x, b, yout);
}
void layer_bwd_any(Run& r, int l, const char* x, LayerBufs& b, float* dy, char* scr) {
  Range rg("layer bwd", l);
  if (r.c->cfg.arch != 0) layer_backward_pre(r, l, (const float*)x, b, dy, scr);
  else layer_backward(r, l, x, b, dy, scr);
}

// Sub-layer unit steps for either architecture; the unit boundary tensor ("mid")
// is h1 = LN1(z1) (post-LN) or r1 = x + drop(attn) (pre-LN).
int64_t mid_size(const Run& r) { return r.c->cfg.arch != 0 ? r.z.r1 : r.z.h1; }
char* mid_of(const Run& r, const LayerBufs& b) { return r.c->cfg.arch != 0 ? (char*)b.r1 : b.h1; }
void set_mid(const Run& r, LayerBufs& b, char* p) {
  if (r.c->cfg.arch != 0) b.r1 = (float*)p;
  else b.h1 = p;
}
void att_fwd_u(Run& r, int l, const char* x, LayerBufs& b, char* mid_out) {
  if (r.c->cfg.arch != 0) att_forward_pre(r, l, (const float*)x, b, (float*)mid_out);
  else att_forward(r, l, x, b, mid_out);
}
void ffn_fwd_u(Run& r, int l, LayerBufs& b, char* yout) {
  if (r.c->cfg.arch != 0) ffn_forward_pre(r, l, b, (float*)yout);
  else ffn_forward(r, l, b, yout);
}
void ffn_bwd_u(Run& r, int l, LayerBufs& b, float* dy, char* scr) {
  if (r.c->cfg.arch != 0) ffn_backward_pre(r, l, b, dy, scr);
  else ffn_backward(r, l, b, dy, scr);
}
void att_bwd_u(Run& r, int l, const char* x, LayerBufs& b, float* dy, char* scr) {
  if (r.c->cfg.arch != 0) att_backward_pre(r, l, (const float*)x, b, dy, scr);
  else att_backward(r, l, x, b, dy, scr);
}

// ===========================================================================
// Encoder-decoder (reading A32; DESIGN §3 "Encoder-decoder").
// Units: encoder layers 0..Le-1 (pre-LN, bidirectional: the GPT-2 layer code
// with a non-causal mask), decoder layers Le..Le+Ld-1 (pre-LN: causal
// self-attention, cross-attention on the encoder output, FFN).  The last
// encoder unit's output bundle is [x_L, enc_out = LN_enc(x_L), enc_st, x1_t].
// Arena order and sizes follow oracle/memsim.py sizes_encdec exactly.
// ===========================================================================
inline int EL(const mimose_ctx* c, int k) { return 2 + 12 * c->cfg.n_layers + k; }   // encoder final LN
inline int DP(const mimose_ctx* c, int j, int k) { return 2 + 12 * c->cfg.n_layers + 2 + 20 * j + k; }
enum { D_LN1G = 0, D_LN1B, D_QKVW, D_QKVB, D_OW, D_OB, D_LN2G, D_LN2B, D_CQW, D_CQB, D_CKVW, D_CKVB, D_COW, D_COB,
       D_LN3G, D_LN3B, D_F1W, D_F1B, D_F2W, D_F2B };
constexpr uint32_t DEC_EMB_LAYER = 0xFFE;
constexpr uint32_t KIND_CROSS_PROBS = 5, KIND_CROSS_OUT = 6;

struct SzD {                 // decoder-side and shared sizes of one (B, Ss, St)
  int64_t a, st, qkv, O, lse, r, c, qc, kvc, m, u, g, y;   // decoder internals (st/r/lse shared shapes)
  int64_t xL, enc_out, enc_st, x1t;                         // the bundle
  int64_t head0, head1, head2, head_fwd, head_scr;
  int64_t dy, denc, U, embU;
  int64_t scr_enc_off, scr_kv_off;                          // carve offsets inside U
};

SzD sizes_dec(const mimose_ctx* c, int B, int Ss, int St) {
  const int64_t Ts = (int64_t)B * Ss, Tt = (int64_t)B * St, H = c->cfg.hidden, F = c->cfg.ffn, h = c->cfg.heads,
                e = c->e;
  SzD z{};
  z.a = a16(Tt * H * e); z.st = a16(Tt * 8); z.qkv = a16(Tt * 3 * H * e); z.O = a16(Tt * H * e);
  z.lse = a16((int64_t)B * h * St * 4); z.r = a16(Tt * H * 4); z.c = a16(Tt * H * e); z.qc = a16(Tt * H * e);
  z.kvc = a16(Ts * 2 * H * e); z.m = a16(Tt * H * e); z.u = a16(Tt * F * e); z.g = a16(Tt * F * e);
  z.y = a16(Tt * H * 4);
  z.xL = a16(Ts * H * 4); z.enc_out = a16(Ts * H * e); z.enc_st = a16(Ts * 8); z.x1t = a16(Tt * H * 4);
  const int64_t VP = vpad(c->cfg.vocab);
  z.head0 = a16(Tt * H * e); z.head1 = a16(Tt * 8); z.head2 = a16(Tt * 8);
  z.head_fwd = a16((int64_t)LM_CHUNK * VP * 4);
  z.head_scr = a16((int64_t)LM_CHUNK * VP * 4) + a16((int64_t)LM_CHUNK * VP * e);
  z.dy = a16(Tt * H * 4); z.denc = a16(Ts * H * 4);
  auto lscr = [&](int64_t T, int64_t S) {
    return a16(T * H * 4) + a16(T * F * e) + a16(T * 3 * H * e) + a16((int64_t)B * h * S * 4);
  };
  z.scr_kv_off = lscr(Tt, St);
  z.scr_enc_off = z.scr_kv_off + a16(Ts * 2 * H * e);
  z.U = z.scr_enc_off + lscr(Ts, Ss);
  const int64_t maxT = (int64_t)c->cfg.max_seqs * c->cfg.max_seq_len;
  const int64_t ntiles = (maxT + 1023) / 1024;
  auto escr = [&](int64_t T) { return a16(T * H * 4) + a16(16 * T) + a16(4 * 256 * ntiles); };
  z.embU = escr(Ts) + escr(Tt);
  return z;
}



// The decoder internals in the order of oracle/memsim.py sizes_encdec:
// a st1 QKV O LSE r1 st2 c Qc KVc Oc LSEc r2 st3 m u g
void dec_sizes_list(const SzD& z, int64_t* s) {
  const int64_t v[17] = {z.a, z.st, z.qkv, z.O, z.lse, z.r, z.st, z.c, z.qc, z.kvc, z.O, z.lse, z.r, z.st, z.m, z.u, z.g};
  for (int i = 0; i < 17; ++i) s[i] = v[i];
}
void alloc_dec(mimose_ctx* c, const SzD& z, DecBufs& b, bool on_stack) {
  Arena& a = c->ar;
  auto al = [&](int64_t n) { return on_stack ? a.push(n) : a.talloc(n); };
  b.a = al(z.a); b.st1 = (float2*)al(z.st); b.qkv = al(z.qkv); b.O = al(z.O); b.lse = (float*)al(z.lse);
  b.r1 = (float*)al(z.r); b.st2 = (float2*)al(z.st); b.c = al(z.c); b.qc = al(z.qc); b.kvc = al(z.kvc);
  b.oc = al(z.O); b.lsec = (float*)al(z.lse); b.r2 = (float*)al(z.r); b.st3 = (float2*)al(z.st); b.m = al(z.m);
  b.u = al(z.u); b.g = al(z.g);
}
void free_dec(mimose_ctx* c, const SzD& z, bool on_stack) {
  int64_t s[17];
  dec_sizes_list(z, s);
  for (int i = 16; i >= 0; --i) on_stack ? c->ar.pop(s[i]) : c->ar.tfree(s[i]);
}

// Point the step state at one stack: the layer kernels read c->S, c->T and the
// key/query lengths through c->lens, the LM head the ids through c->ids.
void use_enc(mimose_ctx* c) {
  c->S = c->Ss; c->T = c->B * c->Ss;
  c->lens = c->lens_src; c->ids = c->ids_src;
}
void use_dec(mimose_ctx* c) {
  c->S = c->St; c->T = c->B * c->St;
  c->lens = c->lens_tgt; c->ids = c->ids_tgt;
}

void dec_layer_forward(Run& r, const SzD& z, int j, const float* x, DecBufs& b, float* yout) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  use_dec(c);
  const int Tt = c->T, Ts = c->B * c->Ss, H = c->cfg.hidden, F = c->cfg.ffn, h = c->cfg.heads;
  const uint32_t site = (uint32_t)(c->cfg.n_layers + j);
  ln_fwd(c->dt, x, W(c, DP(c, j, D_LN1G)), W(c, DP(c, j, D_LN1B)), b.a, b.st1, Tt, H, c->cfg.ln_eps, r.st);
  GemmArgs g;
  g.M = Tt; g.N = 3 * H; g.K = H;
  g.A = b.a; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, DP(c, j, D_QKVW)); g.b_sn = H; g.b_sk = 1;
  g.C = b.qkv; g.ldc = 3 * H; g.bias = W(c, DP(c, j, D_QKVB));
  pgemm(c, EPI_BIAS, g, r.st);
  attn_fwd(c->dt, b.qkv, c->lens_tgt, b.O, b.lse, c->B, c->St, H, h, make_drop(c, KIND_ATTN_PROBS, site), r.st, true);
  g = GemmArgs();
  g.M = Tt; g.N = H; g.K = H;
  g.A = b.O; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, DP(c, j, D_OW)); g.b_sn = H; g.b_sk = 1;
  g.C = b.r1; g.ldc = H; g.bias = W(c, DP(c, j, D_OB)); g.res = x; g.ldr = H;
  g.drop = make_drop(c, KIND_ATTN_OUT, site);
  pgemm(c, EPI_BIAS_DROP_RESF32, g, r.st);
  // cross-attention: Q from LN2(r1), K / V from the encoder output
  ln_fwd(c->dt, b.r1, W(c, DP(c, j, D_LN2G)), W(c, DP(c, j, D_LN2B)), b.c, b.st2, Tt, H, c->cfg.ln_eps, r.st);
  g = GemmArgs();
  g.M = Tt; g.N = H; g.K = H;
  g.A = b.c; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, DP(c, j, D_CQW)); g.b_sn = H; g.b_sk = 1;
  g.C = b.qc; g.ldc = H; g.bias = W(c, DP(c, j, D_CQB));
  pgemm(c, EPI_BIAS, g, r.st);
  g = GemmArgs();
  g.M = Ts; g.N = 2 * H; g.K = H;
  g.A = c->enc_out; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, DP(c, j, D_CKVW)); g.b_sn = H; g.b_sk = 1;
  g.C = b.kvc; g.ldc = 2 * H; g.bias = W(c, DP(c, j, D_CKVB));
  pgemm(c, EPI_BIAS, g, r.st);
  attn_cross_fwd_tc(b.qc, b.kvc, c->lens_tgt, c->lens_src, b.oc, b.lsec, c->B, c->St, c->Ss, H, h,
                    make_drop(c, KIND_CROSS_PROBS, site), r.st);
  note_launch(1);
  g = GemmArgs();
  g.M = Tt; g.N = H; g.K = H;
  g.A = b.oc; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, DP(c, j, D_COW)); g.b_sn = H; g.b_sk = 1;
  g.C = b.r2; g.ldc = H; g.bias = W(c, DP(c, j, D_COB)); g.res = b.r1; g.ldr = H;
  g.drop = make_drop(c, KIND_CROSS_OUT, site);
  pgemm(c, EPI_BIAS_DROP_RESF32, g, r.st);
  // FFN
  ln_fwd(c->dt, b.r2, W(c, DP(c, j, D_LN3G)), W(c, DP(c, j, D_LN3B)), b.m, b.st3, Tt, H, c->cfg.ln_eps, r.st);
  g = GemmArgs();
  g.M = Tt; g.N = F; g.K = H;
  g.A = b.m; g.a_sm = H; g.a_sk = 1;
  g.B = W(c, DP(c, j, D_F1W)); g.b_sn = H; g.b_sk = 1;
  g.C = b.u; g.C2 = b.g; g.ldc = F; g.bias = W(c, DP(c, j, D_F1B));
  pgemm(c, EPI_BIAS_GELUT, g, r.st);
  if (!yout) return;                            // recompute: y is not needed
  g = GemmArgs();
  g.M = Tt; g.N = H; g.K = F;
  g.A = b.g; g.a_sm = F; g.a_sk = 1;
  g.B = W(c, DP(c, j, D_F2W)); g.b_sn = F; g.b_sk = 1;
  g.C = yout; g.ldc = H; g.bias = W(c, DP(c, j, D_F2B)); g.res = b.r2; g.ldr = H;
  g.drop = make_drop(c, KIND_FFN_OUT, site);
  pgemm(c, EPI_BIAS_DROP_RESF32, g, r.st);
}

// Decoder layer backward: dy (fp32 [Tt, H]) in place -> dx; denc (fp32 [Ts, H]) += the
// cross-attention K / V path.  scr = the uniform layer scratch.
void dec_layer_backward(Run& r, const SzD& z, int j, const float* x, DecBufs& b, float* dy, float* denc, char* scr) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  use_dec(c);
  const int Tt = c->T, Ts = c->B * c->Ss, H = c->cfg.hidden, F = c->cfg.ffn, h = c->cfg.heads;
  const uint32_t site = (uint32_t)(c->cfg.n_layers + j);
  const Sz zt = sizes(c, c->B, c->St);
  float* dres = (float*)(scr + zt.r_dres);
  char* R2 = scr + zt.r_du;                     // du; then dOc / dO in its head, dtc / dt1 in its tail
  char* R3 = scr + zt.r_dt;                     // dt3; then dQc; then dQKV
  float* Dbuf = (float*)(scr + zt.r_dt + a16((int64_t)Tt * 3 * H * c->e));
  char* dKV = scr + z.scr_kv_off;
  char* TAIL = R2 + a16((int64_t)Tt * H * c->e);
  float* pg = c->part;
  float* pb = c->part + (int64_t)NPART * H;
  float* pbias = c->part + 2LL * NPART * H;
  // FFN: dt3 = dy * mask (bf16) with db2; du = (dt3 W2) * gelu_tanh'(u); dW2; dm = du W1; dW1; db1
  drop_cast_colsum(c->dt, dy, make_drop(c, KIND_FFN_OUT, site), R3, Tt, H, pbias, r.st);
  reduce_partials(pbias, H, H, G(c, DP(c, j, D_F2B)), r.st);
  {
    GemmArgs g;
    g.M = Tt; g.N = F; g.K = H;
    g.A = R3; g.a_sm = H; g.a_sk = 1;
    g.B = W(c, DP(c, j, D_F2W)); g.b_sn = 1; g.b_sk = F;
    g.C = R2; g.ldc = F; g.aux = b.u; g.ldx = F;
    pgemm(c, EPI_GELUT_BWD, g, r.st);
  }
  wgrad(r, R3, H, b.g, F, G(c, DP(c, j, D_F2W)));
  dgrad(r, EPI_F32, R2, F, W(c, DP(c, j, D_F1W)), H, dres, nullptr);
  wgrad(r, R2, F, b.m, H, G(c, DP(c, j, D_F1W)));
  colsum(c->dt, R2, Tt, F, part_cs(c), r.st);
  reduce_partials(part_cs(c), F, F, G(c, DP(c, j, D_F1B)), r.st);
  // LN3 backward + residual: dr2 = dy + LN3'(dm) (in place in dy); dtc = dr2 * mask (TAIL); dbco
  ln_bwd(c->dt, dres, no_drop(), b.r2, b.st3, W(c, DP(c, j, D_LN3G)), dy, TAIL, make_drop(c, KIND_CROSS_OUT, site),
         pg, pb, pbias, Tt, H, r.st, dy);
  reduce_rows3(pg, G(c, DP(c, j, D_LN3G)), pb, G(c, DP(c, j, D_LN3B)), pbias, G(c, DP(c, j, D_COB)), NPART, H, H,
               r.st);
  // cross-attention: dOc = dtc Wco (R2 head); dWco; attention backward -> dQc (R3), dKV
  dgrad(r, EPI_STORE, TAIL, H, W(c, DP(c, j, D_COW)), H, R2, nullptr);
  wgrad(r, TAIL, H, b.oc, H, G(c, DP(c, j, D_COW)));
  attn_cross_bwd_tc(b.qc, b.kvc, b.oc, R2, b.lsec, c->lens_tgt, c->lens_src, Dbuf, R3, dKV, c->B, c->St, c->Ss, H, h,
                    make_drop(c, KIND_CROSS_PROBS, site), r.st);
  note_launch(std::max(c->St, c->Ss) > 128 ? 2 : 1);
  // dc = dQc Wcq (dres); dWcq; dbcq
  dgrad(r, EPI_F32, R3, H, W(c, DP(c, j, D_CQW)), H, dres, nullptr);
  wgrad(r, R3, H, b.c, H, G(c, DP(c, j, D_CQW)));
  colsum(c->dt, R3, Tt, H, part_cs(c), r.st);
  reduce_partials(part_cs(c), H, H, G(c, DP(c, j, D_CQB)), r.st);
  // denc += dKV Wckv (M = Ts); dWckv = dKV^T enc_out; dbckv
  {
    GemmArgs g;
    g.M = Ts; g.N = H; g.K = 2 * H;
    g.A = dKV; g.a_sm = 2 * H; g.a_sk = 1;
    g.B = W(c, DP(c, j, D_CKVW)); g.b_sn = 1; g.b_sk = H;
    g.C = denc; g.ldc = H; g.res = denc; g.ldr = H;
    pgemm(c, EPI_ACC_RES_F32, g, r.st);
  }
  {
    const int sT = c->T;
    c->T = Ts;                                   // the weight gradient contracts over the source tokens
    wgrad(r, dKV, 2 * H, c->enc_out, H, G(c, DP(c, j, D_CKVW)));
    c->T = sT;
  }
  colsum(c->dt, dKV, Ts, 2 * H, part_cs(c), r.st);
  reduce_partials(part_cs(c), 2 * H, 2 * H, G(c, DP(c, j, D_CKVB)), r.st);
  // LN2 backward + residual: dr1 = dr2 + LN2'(dc) (in place in dy); dt1 = dr1 * mask (TAIL)
  ln_bwd(c->dt, dres, no_drop(), b.r1, b.st2, W(c, DP(c, j, D_LN2G)), dy, TAIL, make_drop(c, KIND_ATTN_OUT, site),
         pg, pb, pbias, Tt, H, r.st, dy);
  reduce_rows3(pg, G(c, DP(c, j, D_LN2G)), pb, G(c, DP(c, j, D_LN2B)), pbias, G(c, DP(c, j, D_OB)), NPART, H, H,
               r.st);
  // self-attention: dO = dt1 Wo (R2 head); dWo; attention backward -> dQKV (R3); da = dQKV Wqkv
  dgrad(r, EPI_STORE, TAIL, H, W(c, DP(c, j, D_OW)), H, R2, nullptr);
  wgrad(r, TAIL, H, b.O, H, G(c, DP(c, j, D_OW)));
  attn_bwd(c->dt, b.qkv, b.O, R2, b.lse, c->lens_tgt, Dbuf, R3, c->B, c->St, H, h, make_drop(c, KIND_ATTN_PROBS, site),
           r.st, true);
  dgrad(r, EPI_F32, R3, 3 * H, W(c, DP(c, j, D_QKVW)), H, dres, nullptr);
  wgrad(r, R3, 3 * H, b.a, H, G(c, DP(c, j, D_QKVW)));
  colsum(c->dt, R3, Tt, 3 * H, part_cs(c), r.st);
  reduce_partials(part_cs(c), 3 * H, 3 * H, G(c, DP(c, j, D_QKVB)), r.st);
  // LN1 backward + residual: dx = dr1 + LN1'(da) (in place in dy)
  ln_bwd(c->dt, dres, no_drop(), x, b.st1, W(c, DP(c, j, D_LN1G)), dy, nullptr, no_drop(), pg, pb, nullptr, Tt, H,
         r.st, dy);
  reduce_rows3(pg, G(c, DP(c, j, D_LN1G)), pb, G(c, DP(c, j, D_LN1B)), nullptr, nullptr, NPART, H, H, r.st);
}

// The last encoder unit's extra output: enc_out = LN_enc(x_L) and the decoder embedding x1_t.
void enc_tail_forward(Run& r, const float* xL, char* enc_out, float2* enc_st, float* x1t) {
  mimose_ctx* c = r.c;
  if (!r.real) return;
  const int H = c->cfg.hidden;
  ln_fwd(c->dt, xL, W(c, EL(c, 0)), W(c, EL(c, 1)), enc_out, enc_st, c->B * c->Ss, H, c->cfg.ln_eps, r.st);
  embed_fwd_pre(c->dt, c->ids_tgt, W(c, P_WORD), W(c, P_POS), x1t, c->B, c->St, H, c->cfg.pos_offset,
                make_drop(c, KIND_EMB, DEC_EMB_LAYER), r.st);
}

void run_forward_ed(Run& r, uint64_t mask, bool collect, Sample* sample) {
  mimose_ctx* c = r.c;
  Arena& a = c->ar;
  const int Le = c->cfg.n_layers, Ld = c->cfg.n_dec_layers, H = c->cfg.hidden;
  const SzD zd = sizes_dec(c, c->B, c->Ss, c->St);
  r.z = sizes(c, c->B, c->Ss);                       // encoder-layer sizes (GPT-2 layer list at T_s)
  const int64_t base = a.live();
  use_enc(c);
  c->x1 = a.push(r.z.x1);                            // x1_s
  if (sample) sample->E = a.live() - base;
  if (r.real)
    embed_fwd_pre(c->dt, c->ids_src, W(c, P_WORD), W(c, P_POS), (float*)c->x1, c->B, c->Ss, H, c->cfg.pos_offset,
                  make_drop(c, KIND_EMB, LAYER_NONE), r.st);
  c->lb.assign(Le, LayerBufs());
  c->dlb.assign(Ld, DecBufs());
  c->y.assign(Le + Ld, nullptr);
  const char* x = c->x1;
  for (int l = 0; l < Le; ++l) {
    use_enc(c);
    const int64_t b0 = a.live();
    const bool last = l == Le - 1;
    if (collect && sample) {                         // pass 1 (save mode), timed, discarded
      LayerBufs tmp;
      alloc_internals(r, tmp, true);
      char* yt = a.push(r.z.y);
      char *eo = nullptr, *x1t = nullptr;
      float2* es = nullptr;
      if (last) { eo = a.push(zd.enc_out); es = (float2*)a.push(zd.enc_st); x1t = a.push(zd.x1t); }
      if (r.real) cudaEventRecord(c->ev_t0[l], r.st);
      layer_fwd_any(r, l, x, tmp, yt);
      if (last) { char* so = c->enc_out; c->enc_out = eo; enc_tail_forward(r, (float*)yt, eo, es, (float*)x1t); c->enc_out = so; }
      if (r.real) cudaEventRecord(c->ev_t1[l], r.st);
      sample->a[l] = a.live() - b0;
      if (last) { a.pop(zd.x1t); a.pop(zd.enc_st); a.pop(zd.enc_out); }
      a.pop(r.z.y);
      free_internals(r, true);
    }
    const bool dropped = collect || ((mask >> l) & 1);
    alloc_internals(r, c->lb[l], !dropped);
    c->y[l] = a.push(r.z.y);
    if (last) {
      c->enc_out = a.push(zd.enc_out);
      c->enc_st = (float2*)a.push(zd.enc_st);
      c->x1t = a.push(zd.x1t);
    }
    layer_fwd_any(r, l, x, c->lb[l], c->y[l]);
    if (last) enc_tail_forward(r, (float*)c->y[l], c->enc_out, c->enc_st, (float*)c->x1t);
    if (dropped) free_internals(r, false);
    if (sample) sample->y[l] = a.live() - b0;
    x = c->y[l];
  }
  x = c->x1t;
  for (int j = 0; j < Ld; ++j) {
    const int u = Le + j;
    const int64_t b0 = a.live();
    if (collect && sample) {
      DecBufs tmp;
      alloc_dec(c, zd, tmp, true);
      char* yt = a.push(zd.y);
      if (r.real) cudaEventRecord(c->ev_t0[u], r.st);
      dec_layer_forward(r, zd, j, (const float*)x, tmp, (float*)yt);
      if (r.real) cudaEventRecord(c->ev_t1[u], r.st);
      sample->a[u] = a.live() - b0;
      a.pop(zd.y);
      free_dec(c, zd, true);
    }
    const bool dropped = collect || ((mask >> u) & 1);
    alloc_dec(c, zd, c->dlb[j], !dropped);
    c->y[u] = a.push(zd.y);
    dec_layer_forward(r, zd, j, (const float*)x, c->dlb[j], (float*)c->y[u]);
    if (dropped) free_dec(c, zd, false);
    if (sample) sample->y[u] = a.live() - b0;
    x = c->y[u];
  }
  use_dec(c);
  const int64_t h0 = a.live();
  c->hp = a.push(zd.head0);
  c->lm_stf = (float2*)a.push(zd.head1);
  c->lm_tok = (float2*)a.push(zd.head2);
  if (sample) sample->Hd = a.live() - h0;
  float* lg = (float*)a.talloc(zd.head_fwd);
  if (r.real) lm_head_forward(r, (float*)c->y[Le + Ld - 1], c->hp, c->lm_stf, c->lm_tok, lg);
  a.tfree(zd.head_fwd);
}

mimose_status run_backward_ed(Run& r, Sample* sample) {
  mimose_ctx* c = r.c;
  Arena& a = c->ar;
  const int Le = c->cfg.n_layers, Ld = c->cfg.n_dec_layers, H = c->cfg.hidden;
  const SzD zd = sizes_dec(c, c->B, c->Ss, c->St);
  r.z = sizes(c, c->B, c->Ss);
  const int Ts = c->B * c->Ss, Tt = c->B * c->St;
  float* denc = (float*)a.talloc(zd.denc);
  float* dy = (float*)a.talloc(zd.dy);
  if (r.real) CK(cudaMemsetAsync(denc, 0, (size_t)Ts * H * 4, r.st));
  // ---- LM head on the decoder ----
  use_dec(c);
  a.top_phase_peak = a.top;
  char* hs = a.talloc(zd.head_scr);
  if (r.real) {
    CK(cudaMemsetAsync(G(c, P_WORD), 0, (size_t)c->layout[P_WORD].numel * 4, r.st));
    lm_head_backward(r, (float*)c->y[Le + Ld - 1], c->hp, c->lm_stf, c->lm_tok, hs, dy);
  }
  a.tfree(zd.head_scr);
  if (sample) sample->Th = a.top_phase_peak;
  a.pop(zd.head2);
  a.pop(zd.head1);
  a.pop(zd.head0);
  a.pop(zd.y);                                        // the last decoder output
  // ---- decoder layers ----
  a.top_phase_peak = a.top;
  int64_t tb = 0, te = 0;
  for (int j = Ld - 1; j >= 0; --j) {
    const int u = Le + j;
    const float* x = j > 0 ? (const float*)c->y[u - 1] : (const float*)c->x1t;
    if ((c->drop_mask >> u) & 1) {
      if (r.real) join(c, r.st);
      alloc_dec(c, zd, c->dlb[j], true);
      dec_layer_forward(r, zd, j, x, c->dlb[j], nullptr);
    }
    char* scr = a.talloc(zd.U);
    dec_layer_backward(r, zd, j, x, c->dlb[j], dy, denc, scr);
    a.tfree(zd.U);
    free_dec(c, zd, true);
    if (j > 0) a.pop(zd.y);
  }
  tb = a.top_phase_peak;
  // ---- decoder embedding (tied wte accumulates onto the LM head's dW_e) ----
  a.top_phase_peak = a.top;
  char* es = a.talloc(zd.embU);
  if (r.real) {
    float* dz0 = (float*)es;
    int32_t* work = (int32_t*)(es + a16((int64_t)Tt * H * 4));
    int32_t* hist = (int32_t*)(es + a16((int64_t)Tt * H * 4) + a16(16LL * Tt));
    drop_f32(dy, make_drop(c, KIND_EMB, DEC_EMB_LAYER), dz0, (int64_t)Tt * H, r.st);
    pos_grad(dz0, c->B, c->St, H, c->cfg.pos_offset, G(c, P_POS), r.st);    // (writes every row below St)
    const int64_t maxT = (int64_t)c->cfg.max_seqs * c->cfg.max_seq_len;
    keyed_rowsum(c->ids_tgt, c->cfg.vocab <= 256 ? 8 : 16, dz0, Tt, H, G(c, P_WORD), work, hist,
                 (int)((maxT + 1023) / 1024), c->cfg.pad_id, r.st, /*accumulate=*/true);
  }
  a.tfree(zd.embU);
  te = a.top_phase_peak;
  a.pop(zd.x1t);
  // ---- encoder final LN (in place in denc) ----
  use_enc(c);
  if (r.real) {
    float* pg = c->part;
    float* pb = c->part + (int64_t)NPART * H;
    ln_bwd(c->dt, denc, no_drop(), (const float*)c->y[Le - 1], c->enc_st, W(c, EL(c, 0)), denc, nullptr, no_drop(),
           pg, pb, nullptr, Ts, H, r.st);
    reduce_rows3(pg, G(c, EL(c, 0)), pb, G(c, EL(c, 1)), nullptr, nullptr, NPART, H, H, r.st);
  }
  a.pop(zd.enc_st);
  a.pop(zd.enc_out);
  a.pop(r.z.y);                                       // x_L
  // ---- encoder layers (GPT-2 layer code, bidirectional) ----
  a.top_phase_peak = a.top;
  for (int l = Le - 1; l >= 0; --l) {
    use_enc(c);
    const char* x = l > 0 ? c->y[l - 1] : c->x1;
    if ((c->drop_mask >> l) & 1) {
      if (r.real) join(c, r.st);
      alloc_internals(r, c->lb[l], true);
      layer_fwd_any(r, l, x, c->lb[l], nullptr);
    }
    char* scr = a.talloc(zd.U);
    layer_bwd_any(r, l, x, c->lb[l], denc, scr);
    a.tfree(zd.U);
    free_internals(r, true);
    if (l > 0) a.pop(r.z.y);
  }
  tb = std::max(tb, a.top_phase_peak);
  if (r.real) join(c, r.st);
  // ---- encoder embedding ----
  a.top_phase_peak = a.top;
  es = a.talloc(zd.embU);
  if (r.real) {
    float* dz0 = (float*)es;
    int32_t* work = (int32_t*)(es + a16((int64_t)Ts * H * 4));
    int32_t* hist = (int32_t*)(es + a16((int64_t)Ts * H * 4) + a16(16LL * Ts));
    drop_f32(denc, make_drop(c, KIND_EMB, LAYER_NONE), dz0, (int64_t)Ts * H, r.st);
    if (c->St < c->cfg.max_pos)                      // rows the decoder did not write
      CK(cudaMemsetAsync(G(c, P_POS) + (int64_t)(c->cfg.pos_offset + c->St) * H, 0,
                         (size_t)(c->cfg.max_pos - c->cfg.pos_offset - c->St) * H * 4, r.st));
    pos_grad(dz0, c->B, c->Ss, H, c->cfg.pos_offset, G(c, P_POS), r.st, /*accumulate=*/true);
    const int64_t maxT = (int64_t)c->cfg.max_seqs * c->cfg.max_seq_len;
    keyed_rowsum(c->ids_src, c->cfg.vocab <= 256 ? 8 : 16, dz0, Ts, H, G(c, P_WORD), work, hist,
                 (int)((maxT + 1023) / 1024), c->cfg.pad_id, r.st, /*accumulate=*/true);
  }
  a.tfree(zd.embU);
  te = std::max(te, a.top_phase_peak);
  if (sample) { sample->Tb = tb; sample->Te = te; }
  a.pop(r.z.x1);
  a.tfree(zd.dy);
  a.tfree(zd.denc);
  if (r.real) {
    mimose_status s = allreduce_bucket(c, 0, (int)c->layout.size() - 1, Le + 1);   // one bucket: every tensor
    if (s) return s;
  }
  return MIMOSE_OK;
}

// Forward of one step.  mode 0: plan-driven; mode 1: shuttling collector.
// When `sample` is non-null the collector deltas are recorded.
void run_forward(Run& r, uint64_t mask, bool collect, Sample* sample) {
  mimose_ctx* c = r.c;
  if (c->cfg.arch == 2) return run_forward_ed(r, mask, collect, sample);
  Arena& a = c->ar;
  const int L = c->cfg.n_layers, H = c->cfg.hidden;
  const int64_t base = a.live();
  if (c->cfg.arch == 1) {                       // GPT-2: x1 = drop(wte[ids] + wpe[pos]) (fp32)
    c->z0 = nullptr;
    c->st0 = nullptr;
    c->x1 = a.push(r.z.x1);
    if (sample) sample->E = a.live() - base;
    if (r.real)
      embed_fwd_pre(c->dt, c->ids, W(c, P_WORD), W(c, P_POS), (float*)c->x1, c->B, c->S, H, c->cfg.pos_offset,
                    make_drop(c, KIND_EMB, LAYER_NONE), r.st);
  } else {
    c->z0 = (float*)a.push(r.z.z0);
    c->st0 = (float2*)a.push(r.z.st0);
    c->x1 = a.push(r.z.x1);
    if (sample) sample->E = a.live() - base;
    if (r.real)
      embed_fwd(c->dt, c->ids, c->tt, W(c, P_WORD), W(c, P_POS), W(c, P_TYPE), W(c, P_LN0G), W(c, P_LN0B), c->z0,
                c->st0, c->x1, c->B, c->S, H, c->cfg.pos_offset, c->cfg.ln_eps, make_drop(c, KIND_EMB, LAYER_NONE),
                r.st);
  }
  c->lb.assign(L, LayerBufs());
  c->y.assign(L, nullptr);
  const char* x = c->x1;
  for (int l = 0; l < L && c->cfg.granularity == 1; ++l) {   // sub-layer units 2l (attention), 2l+1 (FFN)
    set_layer(r, l);
    LayerBufs& b = c->lb[l];
    const int ua = 2 * l, uf = 2 * l + 1;
    int64_t b0 = a.live();
    if (collect && sample) {                  // pass 1 (save mode), timed, discarded
      LayerBufs tmp;
      alloc_att(r, tmp, true);
      char* ht = a.push(mid_size(r));
      set_mid(r, tmp, ht);
      if (r.real) cudaEventRecord(c->ev_t0[ua], r.st);
      att_fwd_u(r, l, x, tmp, ht);
      if (r.real) cudaEventRecord(c->ev_t1[ua], r.st);
      sample->a[ua] = a.live() - b0;
      a.pop(mid_size(r));
      free_att(r, true);
    }
    const bool da = collect || ((mask >> ua) & 1);
    alloc_att(r, b, !da);
    set_mid(r, b, a.push(mid_size(r)));
    att_fwd_u(r, l, x, b, mid_of(r, b));
    if (da) free_att(r, false);
    if (sample) sample->y[ua] = a.live() - b0;
    b0 = a.live();
    if (collect && sample) {
      LayerBufs tmp;
      set_mid(r, tmp, mid_of(r, b));
      alloc_ffn(r, tmp, true);
      char* yt = a.push(r.z.y);
      if (r.real) cudaEventRecord(c->ev_t0[uf], r.st);
      ffn_fwd_u(r, l, tmp, yt);
      if (r.real) cudaEventRecord(c->ev_t1[uf], r.st);
      sample->a[uf] = a.live() - b0;
      a.pop(r.z.y);
      free_ffn(r, true);
    }
    const bool df = collect || ((mask >> uf) & 1);
    alloc_ffn(r, b, !df);
    c->y[l] = a.push(r.z.y);
    ffn_fwd_u(r, l, b, c->y[l]);
    if (df) free_ffn(r, false);
    if (sample) sample->y[uf] = a.live() - b0;
    x = c->y[l];
  }
  for (int l = 0; l < L && c->cfg.granularity == 0; ++l) {
    set_layer(r, l);
    const int64_t b0 = a.live();
    if (collect && sample) {
      // pass 1: normal forward (save mode), timed; output and activations discarded
      LayerBufs tmp;
      alloc_internals(r, tmp, true);
      char* yt = a.push(r.z.y);
      if (r.real) cudaEventRecord(c->ev_t0[l], r.st);
      layer_fwd_any(r, l, x, tmp, yt);
      if (r.real) cudaEventRecord(c->ev_t1[l], r.st);
      sample->a[l] = a.live() - b0;
      a.pop(r.z.y);
      free_internals(r, true);
    }
    const bool dropped = collect || ((mask >> l) & 1);
    alloc_internals(r, c->lb[l], !dropped);
    c->y[l] = a.push(r.z.y);
    layer_fwd_any(r, l, x, c->lb[l], c->y[l]);
    if (dropped) free_internals(r, false);
    if (sample) sample->y[l] = a.live() - b0;
    x = c->y[l];
  }
  const int64_t h0 = a.live();
  if (c->cfg.head == 3) {                       // LM head: hf, stf, tokstat; fp32 logits chunk transient
    c->hp = a.push(r.z.head0);
    c->lm_stf = (float2*)a.push(r.z.head1);
    c->lm_tok = (float2*)a.push(r.z.head2);
    if (sample) sample->Hd = a.live() - h0;
    float* lg = (float*)a.talloc(r.z.head_fwd);
    if (r.real) lm_head_forward(r, (float*)c->y[L - 1], c->hp, c->lm_stf, c->lm_tok, lg);
    a.tfree(r.z.head_fwd);
    return;
  } else if (c->cfg.head == MIMOSE_HEAD_QA) {
    c->logits = (float*)a.push(r.z.head0);
    if (r.real)
      head_qa_fwd(c->dt, c->y[L - 1], c->B, c->S, H, W(c, HP(c, 0)), W(c, HP(c, 1)), c->logits, c->lens,
                  c->labels, c->misc, r.st);
  } else {
    c->hp = a.push(r.z.head0);
    c->logits = (float*)a.push(r.z.head1);
    const int no = c->cfg.head == MIMOSE_HEAD_MC ? 1 : c->cfg.n_labels;
    if (r.real)
      head_cls_fwd(c->dt, c->y[L - 1], c->B, c->S, H, W(c, HP(c, 0)), W(c, HP(c, 1)), W(c, HP(c, 2)),
                   W(c, HP(c, 3)), no, c->hp, c->logits, c->labels, c->cfg.n_choices, c->cfg.head, c->misc,
                   make_drop(c, KIND_HEAD, LAYER_NONE), r.st);
  }
  if (sample) sample->Hd = a.live() - h0;
}

mimose_status run_backward(Run& r, Sample* sample) {
  mimose_ctx* c = r.c;
  if (c->cfg.arch == 2) return run_backward_ed(r, sample);
  Arena& a = c->ar;
  const int L = c->cfg.n_layers, H = c->cfg.hidden;
  const int T = c->T;
  float* dy = (float*)a.talloc(r.z.dy);
  // ---- head ----
  a.top_phase_peak = a.top;
  char* hs = a.talloc(r.z.head_scr);
  if (r.real) {
    if (c->cfg.head == 3) {
      // the tied wte gradient accumulates: LM head chunks now, the embedding lookup later
      CK(cudaMemsetAsync(G(c, P_WORD), 0, (size_t)c->layout[P_WORD].numel * 4, r.st));
      lm_head_backward(r, (float*)c->y[L - 1], c->hp, c->lm_stf, c->lm_tok, hs, dy);
    } else if (c->cfg.head == MIMOSE_HEAD_QA) {
      head_qa_bwd(c->dt, c->y[L - 1], c->B, c->S, H, W(c, HP(c, 0)), c->logits, c->lens, c->labels, (float*)hs,
                  c->part, G(c, HP(c, 0)), G(c, HP(c, 1)), dy, r.st);
    } else {
      CK(cudaMemsetAsync(dy, 0, (size_t)T * H * 4, r.st));
      const int no = c->cfg.head == MIMOSE_HEAD_MC ? 1 : c->cfg.n_labels;
      head_cls_bwd(c->dt, c->y[L - 1], c->B, c->S, H, W(c, HP(c, 0)), W(c, HP(c, 2)), no, c->hp, c->logits,
                   c->labels, c->cfg.n_choices, c->cfg.head, (float*)hs, G(c, HP(c, 0)), G(c, HP(c, 1)),
                   G(c, HP(c, 2)), G(c, HP(c, 3)), dy, make_drop(c, KIND_HEAD, LAYER_NONE), r.st);
    }
  }
  a.tfree(r.z.head_scr);
  if (sample) sample->Th = a.top_phase_peak;
  if (r.real) {
    const int nh = (c->cfg.head == MIMOSE_HEAD_QA || c->cfg.head == 3) ? 2 : 4;
    mimose_status s = allreduce_bucket(c, HP(c, 0), HP(c, nh - 1), L);
    if (s) return s;
  }
  if (c->cfg.head == 3) {
    a.pop(r.z.head2);
    a.pop(r.z.head1);
    a.pop(r.z.head0);
  } else if (c->cfg.head == MIMOSE_HEAD_QA) {
    a.pop(r.z.head0);
  } else {
    a.pop(r.z.head1);
    a.pop(r.z.head0);
  }
  a.pop(r.z.y);                                       // y_L
  // ---- layers ----
  a.top_phase_peak = a.top;
  for (int l = L - 1; l >= 0 && c->cfg.granularity == 1; --l) {   // sub-layer units
    set_layer(r, l);
    LayerBufs& b = c->lb[l];
    const char* x = l > 0 ? c->y[l - 1] : c->x1;
    if ((c->drop_mask >> (2 * l + 1)) & 1) {          // recompute the FFN block from h1 / r1
      if (r.real) join(c, r.st);                      // side-stream readers of the popped region first
      alloc_ffn(r, b, true);
      ffn_fwd_u(r, l, b, nullptr);
    }
    char* scr = a.talloc(r.z.layer_scr);
    ffn_bwd_u(r, l, b, dy, scr);
    free_ffn(r, true);
    a.pop(mid_size(r));                               // h1 / r1: dead after the FFN block's gradients
    if ((c->drop_mask >> (2 * l)) & 1) {              // recompute the attention block from y_{l-1}
      if (r.real) join(c, r.st);                      // the FFN block's side wgrad reads g, h1 (popped)
      alloc_att(r, b, true);
      att_fwd_u(r, l, x, b, nullptr);
    }
    att_bwd_u(r, l, x, b, dy, scr);
    a.tfree(r.z.layer_scr);
    if (r.real) {
      mimose_status s = allreduce_bucket(c, layer_base(c) + 12 * l, layer_base(c) + 12 * l + 11, l);
      if (s) return s;
    }
    free_att(r, true);
    if (l > 0) a.pop(r.z.y);                          // y_{l-1}: input of layer l
  }
  for (int l = L - 1; l >= 0 && c->cfg.granularity == 0; --l) {
    set_layer(r, l);
    const bool dropped = (c->drop_mask >> l) & 1;
    const char* x = l > 0 ? c->y[l - 1] : c->x1;
    if (dropped) {                                    // recompute right before the gradients
      if (r.real) join(c, r.st);                      // the side wgrads of layer l+1 read x = y_l, O (popped)
      alloc_internals(r, c->lb[l], true);
      layer_fwd_any(r, l, x, c->lb[l], nullptr);
    }
    char* scr = a.talloc(r.z.layer_scr);
    layer_bwd_any(r, l, x, c->lb[l], dy, scr);
    a.tfree(r.z.layer_scr);
    if (r.real) {
      mimose_status s = allreduce_bucket(c, layer_base(c) + 12 * l, layer_base(c) + 12 * l + 11, l);
      if (s) return s;
    }
    free_internals(r, true);
    if (l > 0) a.pop(r.z.y);                          // y_{l-1}: input of layer l
  }
  if (sample) sample->Tb = a.top_phase_peak;
  if (r.real) join(c, r.st);                          // the partials buffer is reused below
  // ---- embedding ----
  a.top_phase_peak = a.top;
  char* es = a.talloc(r.z.emb_scr);
  if (r.real && c->cfg.arch == 1) {
    float* dz0 = (float*)es;
    int32_t* work = (int32_t*)(es + a16((int64_t)T * H * 4));
    int32_t* hist = (int32_t*)(es + a16((int64_t)T * H * 4) + a16(16LL * T));
    drop_f32(dy, make_drop(c, KIND_EMB, LAYER_NONE), dz0, (int64_t)T * H, r.st);
    CK(cudaMemsetAsync(G(c, P_POS), 0, (size_t)c->layout[P_POS].numel * 4, r.st));
    pos_grad(dz0, c->B, c->S, H, c->cfg.pos_offset, G(c, P_POS), r.st);
    const int64_t maxT = (int64_t)c->cfg.max_seqs * c->cfg.max_seq_len;
    keyed_rowsum(c->ids, c->cfg.vocab <= 256 ? 8 : 16, dz0, T, H, G(c, P_WORD), work, hist,
                 (int)((maxT + 1023) / 1024), c->cfg.pad_id, r.st, /*accumulate=*/true);
  } else if (r.real) {
    float* dz0 = (float*)es;
    int32_t* work = (int32_t*)(es + a16((int64_t)T * H * 4));
    int32_t* hist = (int32_t*)(es + a16((int64_t)T * H * 4) + a16(16LL * T));
    float* pg = c->part;
    float* pb = c->part + (int64_t)NPART * H;
    ln_bwd(c->dt, dy, make_drop(c, KIND_EMB, LAYER_NONE), c->z0, c->st0, W(c, P_LN0G), dz0, nullptr, no_drop(), pg,
           pb, nullptr, T, H, r.st);
    reduce_rows3(pg, G(c, P_LN0G), pb, G(c, P_LN0B), nullptr, nullptr, NPART, H, H, r.st);
    const int64_t e0 = c->layout[P_WORD].off, e1 = bucket_end(c, P_TYPE);
    CK(cudaMemsetAsync(c->grad + e0, 0, (size_t)(e1 - e0) * 4, r.st));
    pos_grad(dz0, c->B, c->S, H, c->cfg.pos_offset, G(c, P_POS), r.st);
    type_grad(dz0, c->tt, T, H, c->cfg.type_vocab, c->part, G(c, P_TYPE), r.st);
    const int bits = c->cfg.vocab <= 256 ? 8 : 16;
    const int64_t maxT = (int64_t)c->cfg.max_seqs * c->cfg.max_seq_len;
    keyed_rowsum(c->ids, bits, dz0, T, H, G(c, P_WORD), work, hist, (int)((maxT + 1023) / 1024), c->cfg.pad_id,
                 r.st);
  }
  a.tfree(r.z.emb_scr);
  if (sample) sample->Te = a.top_phase_peak;
  if (r.real) {
    mimose_status s = allreduce_bucket(c, P_WORD, c->cfg.arch == 1 ? P_POS : P_LN0B, L + 1);
    if (s) return s;
  }
  a.pop(r.z.x1);
  if (c->cfg.arch != 1) {
    a.pop(r.z.st0);
    a.pop(r.z.z0);
  }
  a.tfree(r.z.dy);
  return MIMOSE_OK;
}

// Host-only accounting of a full step: peak bytes and breach flag.
void dry_step(mimose_ctx* c, int B, int S, uint64_t mask, bool collect, int64_t* peak, bool* breach, Sample* smp,
              int St = 0) {
  // Save the ctx step state that the dry run overwrites.
  const int sB = c->B, sS = c->S, sT = c->T, sSs = c->Ss, sSt = c->St;
  int32_t *sids = c->ids, *slens = c->lens;
  char *seo = c->enc_out, *sx1t = c->x1t;
  float2* sest = c->enc_st;
  std::vector<DecBufs> sdlb = c->dlb;
  const uint64_t sm = c->drop_mask;
  Arena saved = c->ar;
  float* sz0 = c->z0;
  char *sx1 = c->x1, *shp = c->hp;
  float2* sst0 = c->st0;
  float* slog = c->logits;
  float2 *slst = c->lm_stf, *sltk = c->lm_tok;
  std::vector<LayerBufs> slb = c->lb;
  std::vector<char*> sy = c->y;
  c->B = B; c->S = S; c->T = B * S;
  c->Ss = S; c->St = St;
  c->drop_mask = collect ? ~0ull : mask;
  c->ar.reset_step();
  c->ar.base = nullptr;
  Run r{c, false, sizes(c, B, S), nullptr};
  run_forward(r, mask, collect, smp);
  run_backward(r, smp);
  *peak = c->ar.peak;
  *breach = c->ar.breach;
  c->ar = saved;
  c->B = sB; c->S = sS; c->T = sT; c->drop_mask = sm;
  c->z0 = sz0; c->x1 = sx1; c->hp = shp; c->st0 = sst0; c->logits = slog;
  c->lm_stf = slst; c->lm_tok = sltk;
  c->lb = slb; c->y = sy;
  c->Ss = sSs; c->St = sSt; c->ids = sids; c->lens = slens;
  c->enc_out = seo; c->x1t = sx1t; c->enc_st = sest; c->dlb = sdlb;
}

mimose_status check_ready(mimose_ctx* c) {
  if (!c) return MIMOSE_E_INVALID;
  if (c->sticky) return c->sticky;
  return MIMOSE_OK;
}

void resolve_times(mimose_ctx* c) {
  if (!c->pending_times || !c->device) return;
  cudaStreamSynchronize(c->st);
  Sample& s = c->samples.back();
  for (int l = 0; l < n_units(c); ++l) {
    float ms = 0.f;
    cudaEventElapsedTime(&ms, c->ev_t0[l], c->ev_t1[l]);
    s.t_ms[l] = ms;
  }
  c->pending_times = false;
}

// Data parallel: every rank must derive the same plans, but the
// collector's forward times are per-rank measurements.  Before the estimator
// is fitted, the ranks average their time samples (same x sequence on every
// rank: the length schedule is shared), so the time-weighted planner's costs
// agree bit for bit.  Memory samples are exact integers and already agree.
mimose_status agree_times(mimose_ctx* c) {
  if (!c->comm || c->samples.empty()) return MIMOSE_OK;
  const int U = n_units(c);
  const size_t n = c->samples.size() * (size_t)U;
  std::vector<float> h(n);
  for (size_t i = 0; i < c->samples.size(); ++i)
    for (int l = 0; l < U; ++l) h[i * U + l] = c->samples[i].t_ms[l];
  float* d = nullptr;
  CK(cudaMallocAsync((void**)&d, n * 4, c->st));
  CK(cudaMemcpyAsync(d, h.data(), n * 4, cudaMemcpyHostToDevice, c->st));
  NK(ncclAllReduce(d, d, n, ncclFloat, ncclAvg, c->comm, c->st));
  CK(cudaMemcpyAsync(h.data(), d, n * 4, cudaMemcpyDeviceToHost, c->st));
  CK(cudaFreeAsync(d, c->st));
  CK(cudaStreamSynchronize(c->st));
  for (size_t i = 0; i < c->samples.size(); ++i)
    for (int l = 0; l < U; ++l) c->samples[i].t_ms[l] = h[i * U + l];
  return MIMOSE_OK;
}

mimose_status read_loss(mimose_ctx* c, float* loss_out) {
  if (!loss_out) return MIMOSE_OK;
  if (!c->device) { *loss_out = 0.f; return MIMOSE_OK; }
  const float* src = c->misc;
  if (c->comm) {   // the scalar loss is all-reduced (mean over ranks) for logging
    NK(ncclAllReduce(c->misc, c->misc + 1, 1, ncclFloat, ncclAvg, c->comm, c->st));
    src = c->misc + 1;
  }
  CK(cudaMemcpyAsync(loss_out, src, 4, cudaMemcpyDeviceToHost, c->st));
  CK(cudaStreamSynchronize(c->st));
  return MIMOSE_OK;
}

}  // namespace

// =================================================================== ABI ===
extern "C" {

void mimose_default_config(mimose_config* cfg) {
  std::memset(cfg, 0, sizeof(*cfg));
  cfg->arch = MIMOSE_ARCH_POST_LN;
  cfg->head = MIMOSE_HEAD_SEQCLS;
  cfg->dtype = MIMOSE_BF16;
  cfg->type_vocab = 2;
  cfg->n_choices = 4;
  cfg->n_labels = 2;
  cfg->p_drop = 0.1f;
  cfg->ln_eps = 1e-12f;
  cfg->enforce_budget = 1;
  cfg->collect_iters = 10;
  cfg->bucket_num = 9;
  cfg->bucket_den = 10;
  cfg->degree = 2;
  cfg->world = 1;
  cfg->use_tc = 1;
  cfg->pad_id = -1;
}

const char* mimose_status_str(mimose_status s) {
  switch (s) {
    case MIMOSE_OK: return "ok";
    case MIMOSE_E_INVALID: return "invalid argument";
    case MIMOSE_E_STATE: return "call out of order";
    case MIMOSE_E_NOT_READY: return "estimator not fitted (sheltered phase)";
    case MIMOSE_E_INFEASIBLE: return "budget infeasible";
    case MIMOSE_E_BUDGET: return "budget violation";
    case MIMOSE_E_CUDA: return "CUDA error";
    case MIMOSE_E_NCCL: return "NCCL error";
    case MIMOSE_E_NODEVICE: return "host-only context";
  }
  return "?";
}

const char* mimose_last_error(const mimose_ctx* c) { return c ? c->err.c_str() : "null ctx"; }

mimose_status mimose_init(const mimose_config* cfgp, mimose_ctx** out) {
  if (!cfgp || !out) return MIMOSE_E_INVALID;
  *out = nullptr;
  mimose_ctx* c = new mimose_ctx();
  c->cfg = *cfgp;
  const mimose_config& k = c->cfg;
  auto bad = [&](const char* m) { c->err = m; return MIMOSE_E_INVALID; };
  const bool arch_ok = (k.arch == MIMOSE_ARCH_POST_LN && k.head >= 0 && k.head <= 2) || (k.arch == 1 && k.head == 3) ||
                       (k.arch == 2 && k.head == 3 && k.n_dec_layers >= 1 && k.n_layers + k.n_dec_layers <= 64 &&
                        k.granularity == 0 && k.zero1 == 0 && !k.ffn_layers && k.max_seq_len <= 1024 &&
                        k.hidden / k.heads == 64 && k.ffn >= 2 * k.hidden &&
                        (!k.arena_base || (k.dtype == MIMOSE_BF16 && k.use_tc)));
  if (!arch_ok || k.n_layers < 1 || k.n_layers > 64 || k.hidden % 64 || k.heads < 1 ||
      k.hidden % k.heads || (k.hidden / k.heads != 32 && k.hidden / k.heads != 64) || k.ffn % 64 ||
      k.hidden > 1024 || k.ffn > 4096 || k.vocab < 1 || k.vocab > 65536 || (k.arch == 0 && (k.type_vocab < 1 || k.type_vocab > 4)) ||
      k.max_seqs < 1 || k.max_seq_len < 1 || (int64_t)k.max_seqs * k.max_seq_len > 32768 || k.max_pos < 1 ||
      (k.head == MIMOSE_HEAD_MC && k.n_choices < 1) ||
      (k.head == MIMOSE_HEAD_SEQCLS && (k.n_labels < 1 || k.n_labels > 32)) || k.world < 1 || k.rank < 0 ||
      k.rank >= k.world || k.bucket_den <= 0 || k.degree < 0 || k.degree > 2 || k.granularity < 0 ||
      k.granularity > 1 || (k.granularity == 1 && 2 * k.n_layers > 64)) {
    mimose_status s = bad("invalid model / sizing config");
    *out = c;   // returned so mimose_last_error works; caller destroys
    return s;
  }
  if (k.zero1 && k.arena_base && k.world == 1 && !k.comm_force) {
    mimose_status s = bad("zero1 needs a communicator (world > 1 or comm_force)");
    *out = c;
    return s;
  }
  if (c->cfg.collect_iters <= 0) c->cfg.collect_iters = 10;
  c->dt = k.dtype == MIMOSE_FP32 ? DT_F32 : DT_BF16;
  c->e = k.dtype == MIMOSE_FP32 ? 4 : 2;
  if (k.ffn_layers) {
    for (int l = 0; l < k.n_layers; ++l) {
      const int f = k.ffn_layers[l];
      if (f < 64 || f % 64 || f > k.ffn) {
        mimose_status s = bad("ffn_layers[l] must be a multiple of 64 in [64, ffn]");
        *out = c;
        return s;
      }
      c->ffn_l.push_back(f);
    }
  }
  c->zero1 = k.zero1 != 0;
  c->layout = build_layout(k, &c->npad, c->zero1 ? 64LL * k.world : 64);
  c->nshard = c->zero1 ? c->npad / k.world : c->npad;
  c->cfg.ffn_layers = nullptr;   // copied into ffn_l; the caller's array need not outlive init
  {  // gradient buckets by event index: layer l -> l, head -> L, embedding -> L + 1
    const int L = k.n_layers, lb = k.arch != 0 ? 2 : P_LAYER0;
    c->bk_b0.assign(L + 2, 0);
    c->bk_b1.assign(L + 2, 0);
    c->bk_sh.assign(L + 2, 0);
    for (int l = 0; l < L; ++l) {
      c->bk_b0[l] = c->layout[lb + 12 * l].off;
      c->bk_b1[l] = l + 1 < L ? c->layout[lb + 12 * (l + 1)].off : c->layout[lb + 12 * L].off;
    }
    c->bk_b0[L] = c->layout[lb + 12 * L].off;
    c->bk_b1[L] = c->npad;
    c->bk_b0[L + 1] = 0;
    c->bk_b1[L + 1] = c->layout[lb].off;
    const int W = c->zero1 ? k.world : 1;
    int64_t sh = 0;
    for (int i : {L + 1}) { c->bk_sh[i] = sh; sh += (c->bk_b1[i] - c->bk_b0[i]) / W; }
    for (int l = 0; l < L; ++l) { c->bk_sh[l] = sh; sh += (c->bk_b1[l] - c->bk_b0[l]) / W; }
    c->bk_sh[L] = sh;
    sh += (c->bk_b1[L] - c->bk_b0[L]) / W;
    if (sh != c->nshard) {
      *out = c;
      return bad("internal: ZeRO-1 shard layout mismatch");
    }
  }
  c->ws_elems = 4LL * k.hidden * k.hidden;   // wgrad split-K partials (oracle/memsim.py)
  c->device = k.arena_base != nullptr;
  Arena& a = c->ar;
  a.base = (char*)k.arena_base;
  // every allocation is a multiple of 16 B, so live <= M  <=>  live <= floor16(M):
  // flooring the slab end keeps top-region addresses 16-B aligned at no cost
  a.cap = k.arena_base ? (k.arena_bytes & ~(int64_t)15) : (int64_t)1 << 62;
  a.budget = k.budget_bytes > 0 ? k.budget_bytes : a.cap;
  a.enforce = k.enforce_budget != 0;
  if (c->device && a.enforce && a.cap < (a.budget & ~(int64_t)15)) {
    *out = c;
    return bad("arena_bytes < budget_bytes with enforce_budget");
  }
  // persistent region, in the documented order
  int64_t off = 0;
  auto take = [&](int64_t n) { char* p = a.base + off; off += a16(n); return p; };
  c->w = take(c->npad * c->e);
  c->grad = (float*)take(c->npad * 4);
  if (c->dt != DT_F32) c->master = (float*)take(c->nshard * 4);   // ZeRO-1: this rank's shards only
  c->m = (float*)take(c->nshard * 4);
  c->v = (float*)take(c->nshard * 4);
  const int64_t maxT = (int64_t)k.max_seqs * k.max_seq_len;
  c->ids = (int32_t*)take(maxT * 4);
  c->tt = (int32_t*)take(maxT * 4);
  c->lens = (int32_t*)take((int64_t)k.max_seqs * 4);
  c->labels = (int32_t*)take(2LL * k.max_seqs * 4);
  // encoder-decoder: source ids / lengths in ids / lens, decoder ids / lengths in tt / labels
  c->ids_src = c->ids; c->ids_tgt = c->tt; c->lens_src = c->lens; c->lens_tgt = c->labels;
  c->misc = (float*)take(256);
  c->ws = (float*)take(c->ws_elems * 4);
  c->part = (float*)take((int64_t)NPART * 2 * std::max<int64_t>(3LL * k.hidden, (int64_t)k.ffn) * 4);
  a.C = off;
  if (a.C != persistent_bytes(c)) {
    *out = c;
    return bad("internal: persistent layout mismatch");
  }
  a.reset_step();
  c->stats.persistent_bytes = a.C;
  c->stats.budget_bytes = a.budget;
  c->stats.phase = MIMOSE_PHASE_SHELTERED;
  if (a.C > a.budget || a.C > a.cap) {
    *out = c;
    c->err = "persistent state alone exceeds the budget / arena";
    return MIMOSE_E_INFEASIBLE;
  }
  if (c->device) {
    c->st = (cudaStream_t)k.stream;
    const int L = k.n_layers;
    const int U = n_units(c);
    c->ev_t0.resize(U);
    c->ev_t1.resize(U);
    for (int l = 0; l < U; ++l) {
      CK(cudaEventCreate(&c->ev_t0[l]));
      CK(cudaEventCreate(&c->ev_t1[l]));
    }
    CK(cudaMemsetAsync(a.base, 0, (size_t)a.C, c->st));
    c->ev_layer.resize(L + 2);
    c->ev_ar.resize(L + 2);
    c->ev_upd.resize(L + 2);
    for (auto& e : c->ev_upd) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    for (auto& e : c->ev_layer) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    for (auto& e : c->ev_ar) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    CK(cudaStreamCreateWithFlags(&c->opt_st, cudaStreamNonBlocking));
    CK(cudaStreamCreateWithFlags(&c->aux_st, cudaStreamNonBlocking));
    CK(cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&c->ev_opt_done, cudaEventDisableTiming));
    if (k.world > 1 || k.comm_force) {
      if (k.world > 1 && !k.nccl_id) { *out = c; return bad("world > 1 needs nccl_id"); }
      int lo, hi;
      CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
      CK(cudaStreamCreateWithPriority(&c->comm_st, cudaStreamNonBlocking, hi));
      ncclUniqueId id;
      if (k.nccl_id) std::memcpy(&id, k.nccl_id, sizeof(id));
      else NK(ncclGetUniqueId(&id));                // world == 1 with comm_force: own 1-rank communicator
      // Cap NCCL's CTAs: its kernels run on the comm stream next to the
      // persistent GEMMs (grid = SM count) and the fused AdamW; the GEMMs'
      // CTAs never wait on each other, so a cap only trades bandwidth for SMs.
      ncclConfig_t nc = NCCL_CONFIG_INITIALIZER;
      const int cap = k.nccl_max_ctas < 0 ? 0 : (k.nccl_max_ctas == 0 ? 16 : k.nccl_max_ctas);
      if (cap > 0) { nc.maxCTAs = cap; nc.minCTAs = std::min(cap, 4); }
      NK(ncclCommInitRankConfig(&c->comm, k.world, id, k.rank, &nc));
      CK(cudaEventCreateWithFlags(&c->ev_comm_done, cudaEventDisableTiming));
    }
  }
  *out = c;
  return MIMOSE_OK;
}

void mimose_destroy(mimose_ctx* c) {
  if (!c) return;
  if (c->device) {
    cudaStreamSynchronize(c->st);
    for (auto e : c->ev_t0) cudaEventDestroy(e);
    for (auto e : c->ev_t1) cudaEventDestroy(e);
    if (c->opt_st) cudaStreamSynchronize(c->opt_st);
    for (auto e : c->ev_layer) cudaEventDestroy(e);
    for (auto e : c->ev_ar) cudaEventDestroy(e);
    for (auto e : c->ev_upd) cudaEventDestroy(e);
    for (auto e : c->probe_ev) cudaEventDestroy(e);
    if (c->ev_opt_done) cudaEventDestroy(c->ev_opt_done);
    if (c->opt_st) cudaStreamDestroy(c->opt_st);
    if (c->aux_st) { cudaStreamSynchronize(c->aux_st); cudaStreamDestroy(c->aux_st); }
    if (c->ev_fork) cudaEventDestroy(c->ev_fork);
    if (c->ev_join) cudaEventDestroy(c->ev_join);
    if (c->ev_comm_done) cudaEventDestroy(c->ev_comm_done);
    if (c->comm) ncclCommDestroy(c->comm);
    if (c->comm_st) cudaStreamDestroy(c->comm_st);
  }
  delete c;
}

mimose_status mimose_num_params(const mimose_ctx* c, int64_t* n) {
  if (!c || !n) return MIMOSE_E_INVALID;
  int64_t s = 0;
  for (auto& p : c->layout) s += p.numel;
  *n = s;
  return MIMOSE_OK;
}

static mimose_status xfer_params(mimose_ctx* c, float* host, int64_t n, int which) {
  if (mimose_status s = check_ready(c)) return s;
  int64_t tot;
  mimose_num_params(c, &tot);
  if (n != tot || !host) return fail(c, MIMOSE_E_INVALID, "blob size mismatch");
  if (!c->device) return fail(c, MIMOSE_E_NODEVICE, "host-only context");
  if (which == 3 && c->zero1 && c->cfg.world > 1)
    return fail(c, MIMOSE_E_INVALID, "ZeRO-1: the master copy is sharded over the ranks");
  if (c->opt_st) CK(cudaStreamSynchronize(c->opt_st));
  float* tmp = nullptr;
  CK(cudaMallocAsync((void**)&tmp, (size_t)c->npad * 4, c->st));
  std::vector<float> img((size_t)c->npad, 0.f);
  if (which == 0) {  // set
    int64_t o = 0;
    for (auto& p : c->layout) { std::memcpy(&img[p.off], host + o, p.numel * 4); o += p.numel; }
    CK(cudaMemcpyAsync(tmp, img.data(), (size_t)c->npad * 4, cudaMemcpyHostToDevice, c->st));
    cast_from_f32(c->dt, tmp, c->w, c->npad, c->st);
    if (c->master) {
      if (!c->zero1) {
        CK(cudaMemcpyAsync(c->master, tmp, (size_t)c->npad * 4, cudaMemcpyDeviceToDevice, c->st));
      } else {   // this rank's shard of every bucket
        const int W = c->cfg.world, r = c->cfg.rank;
        for (size_t i = 0; i < c->bk_b0.size(); ++i) {
          const int64_t cb = (c->bk_b1[i] - c->bk_b0[i]) / W;
          CK(cudaMemcpyAsync(c->master + c->bk_sh[i], tmp + c->bk_b0[i] + r * cb, (size_t)cb * 4,
                             cudaMemcpyDeviceToDevice, c->st));
        }
      }
    }
    CK(cudaMemsetAsync(c->m, 0, (size_t)c->nshard * 4, c->st));
    CK(cudaMemsetAsync(c->v, 0, (size_t)c->nshard * 4, c->st));
    c->adam_t = 0;
  } else {
    if (which == 1 || (which == 3 && !c->master)) cast_to_f32(c->dt, c->w, tmp, c->npad, c->st);
    else if (which == 3) CK(cudaMemcpyAsync(tmp, c->master, (size_t)c->npad * 4, cudaMemcpyDeviceToDevice, c->st));
    else CK(cudaMemcpyAsync(tmp, c->grad, (size_t)c->npad * 4, cudaMemcpyDeviceToDevice, c->st));
    CK(cudaMemcpyAsync(img.data(), tmp, (size_t)c->npad * 4, cudaMemcpyDeviceToHost, c->st));
  }
  CK(cudaStreamSynchronize(c->st));
  CK(cudaFreeAsync(tmp, c->st));
  CK(cudaStreamSynchronize(c->st));
  if (which != 0) {
    int64_t o = 0;
    for (auto& p : c->layout) { std::memcpy(host + o, &img[p.off], p.numel * 4); o += p.numel; }
  }
  return MIMOSE_OK;
}

mimose_status mimose_set_params(mimose_ctx* c, const float* h, int64_t n) { return xfer_params(c, (float*)h, n, 0); }
mimose_status mimose_get_params(mimose_ctx* c, float* h, int64_t n) { return xfer_params(c, h, n, 1); }
mimose_status mimose_get_master(mimose_ctx* c, float* h, int64_t n) { return xfer_params(c, h, n, 3); }
mimose_status mimose_get_grads(mimose_ctx* c, float* h, int64_t n) {
  if (c && c->device && c->comm_st) cudaStreamSynchronize(c->comm_st);
  return xfer_params(c, h, n, 2);
}

// every rank must run the same plan for the same x (the
// plan is derived, never broadcast).  All-gather a 64-bit FNV-1a hash of
// (x, drop mask, peak) and compare; one 8-B-per-rank exchange + a host sync.
static mimose_status check_plan_consistency(mimose_ctx* c, int64_t x, uint64_t mask, int64_t peak) {
  uint64_t h = 1469598103934665603ull;
  for (uint64_t v : {(uint64_t)x, mask, (uint64_t)peak})
    for (int i = 0; i < 8; ++i) { h ^= (v >> (8 * i)) & 0xff; h *= 1099511628211ull; }
  int n = 1;
  NK(ncclCommCount(c->comm, &n));
  if (n > 15) return MIMOSE_OK;                             // misc[32..63] holds 16 hash words
  uint64_t* dev = (uint64_t*)(c->misc + 32);                // [0] own hash, [1..n] the gather
  uint64_t* gat = dev + 1;
  CK(cudaMemcpyAsync(dev, &h, 8, cudaMemcpyHostToDevice, c->st));
  NK(ncclAllGather(dev, gat, 1, ncclUint64, c->comm, c->st));
  uint64_t got[16];
  CK(cudaMemcpyAsync(got, gat, 8 * (size_t)n, cudaMemcpyDeviceToHost, c->st));
  CK(cudaStreamSynchronize(c->st));
  for (int r = 0; r < n; ++r)
    if (got[r] != h) return fail(c, MIMOSE_E_STATE, "plan mismatch across ranks (rank " + std::to_string(r) + ")");
  c->stats_plan_checks++;
  return MIMOSE_OK;
}

static mimose_status begin_step(mimose_ctx* c, const mimose_batch* bt, uint64_t mask, bool collect, Sample* smp) {
  if (mimose_status s = check_batch(c, bt)) return s;
  // whole-step accounting first: abandon before any launch on a breach
  int64_t peak;
  bool breach;
  const int St = c->cfg.arch == 2 ? bt->dec_len : 0;
  dry_step(c, bt->n_seqs, bt->seq_len, mask, collect, &peak, &breach, nullptr, St);
  if (breach) {
    c->stats.violations++;
    return fail(c, MIMOSE_E_BUDGET, "step would exceed the budget (predicted " + std::to_string(peak) +
                                        " B > M = " + std::to_string(c->ar.budget) + ")");
  }
  if (c->comm && c->cfg.check_plans) {
    if (mimose_status s = check_plan_consistency(c, (int64_t)bt->n_seqs * bt->seq_len, collect ? ~0ull : mask, peak))
      return s;
  }
  c->B = bt->n_seqs; c->S = bt->seq_len; c->T = c->B * c->S;
  c->Ss = bt->seq_len; c->St = St;
  c->drop_mask = collect ? ~0ull : mask;
  c->ar.reset_step();
  c->it++;
  if (c->device) {
    if (mimose_status s = copy_batch(c, bt)) return s;
  }
  Run r{c, c->device, sizes(c, c->B, c->S), c->st};
  run_forward(r, mask, collect, smp);
  c->fwd_done = true;
  c->bwd_done = false;
  return MIMOSE_OK;
}

mimose_status mimose_collect(mimose_ctx* c, const mimose_batch* bt, float* loss_out) {
  Range rg("mimose_collect");
  if (mimose_status s = check_ready(c)) return s;
  if (c->phase != MIMOSE_PHASE_SHELTERED) return fail(c, MIMOSE_E_STATE, "collect after the sheltered phase");
  if (c->fwd_done && !c->bwd_done) return fail(c, MIMOSE_E_STATE, "forward pending its backward");
  if (c->step_pending) return fail(c, MIMOSE_E_STATE, "fused optimizer: mimose_step must close the previous step");
  resolve_times(c);
  const int64_t x = bt ? (int64_t)bt->n_seqs * bt->seq_len : 0;
  const int64_t xt = bt && c->cfg.arch == 2 ? (int64_t)bt->n_seqs * bt->dec_len : 0;
  const int64_t key = (x << 32) | xt;           // 2-D key of an encoder-decoder (xt = 0 otherwise)
  const bool unseen = std::find(c->seen_x.begin(), c->seen_x.end(), key) == c->seen_x.end();
  auto t0 = std::chrono::steady_clock::now();
  c->collecting = unseen;
  Sample smp;
  const int U = n_units(c);
  smp.a.assign(U, 0); smp.y.assign(U, 0); smp.t_ms.assign(U, 0.f);
  mimose_status s = begin_step(c, bt, ~0ull, true, unseen ? &smp : nullptr);
  if (s) return s;
  if (unseen) {
    smp.x = x;
    smp.xt = xt;
    smp.C = c->ar.C;
    c->samples.push_back(smp);     // Th/Tb/Te filled by backward
    c->seen_x.push_back(key);
    c->pending_times = c->device;
    c->stats.shuttled_steps++;
  }
  c->stats.collect_steps++;
  if (mimose_status s2 = read_loss(c, loss_out)) return s2;
  c->stats.collector_ms_total +=
      std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return MIMOSE_OK;
}

mimose_status mimose_forward(mimose_ctx* c, const mimose_batch* bt, const mimose_plan_t* plan, float* loss_out) {
  Range rg("mimose_forward");
  if (mimose_status s = check_ready(c)) return s;
  if (c->fwd_done && !c->bwd_done) return fail(c, MIMOSE_E_STATE, "forward pending its backward");
  if (c->step_pending) return fail(c, MIMOSE_E_STATE, "fused optimizer: mimose_step must close the previous step");
  resolve_times(c);
  c->collecting = false;
  const uint64_t mask = plan ? plan->drop_mask : 0;
  if (mimose_status s = begin_step(c, bt, mask, false, nullptr)) return s;
  return read_loss(c, loss_out);
}

mimose_status mimose_backward(mimose_ctx* c) {
  Range rg("mimose_backward");
  if (mimose_status s = check_ready(c)) return s;
  if (!c->fwd_done || c->bwd_done) return fail(c, MIMOSE_E_STATE, "backward without a pending forward");
  Run r{c, c->device, sizes(c, c->B, c->S), c->st};
  Sample* smp = c->collecting ? &c->samples.back() : nullptr;
  if (mimose_status s = run_backward(r, smp)) return s;
  c->bwd_done = true;
  c->step_pending = c->device && c->opt_fused;   // the per-bucket updates are already applied
  c->stats.peak_bytes = c->ar.peak;
  c->stats.max_peak_bytes = std::max(c->stats.max_peak_bytes, c->ar.peak);
  c->stats.steps++;
  if (c->ar.breach) {   // cannot happen after the dry run; kept as a hard check
    c->stats.violations++;
    return fail(c, MIMOSE_E_BUDGET, "arena breach during backward");
  }
  if (c->phase == MIMOSE_PHASE_SHELTERED) {
    std::vector<int64_t> xs;
    for (auto& s : c->samples) xs.push_back((s.x << 32) | s.xt);
    std::sort(xs.begin(), xs.end());
    const int distinct = (int)(std::unique(xs.begin(), xs.end()) - xs.begin());
    const int64_t n = c->stats.collect_steps;
    const int need = c->cfg.arch == 2 ? 6 : 3;     // distinct keys for a quadratic (2-D: 6 coefficients)
    if (!c->samples.empty() && ((n >= c->cfg.collect_iters && distinct >= need) || n >= 30)) {
      resolve_times(c);
      if (mimose_status s2 = agree_times(c)) return s2;
      auto t0 = std::chrono::steady_clock::now();
      if (c->cfg.arch == 2) c->est.fit2(c->samples, c->cfg.degree);
      else c->est.fit(c->samples, c->cfg.degree);
      c->stats.planner_us_total +=
          std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count();
      c->phase = MIMOSE_PHASE_RESPONSIVE;
      c->stats.phase = c->phase;
    }
  }
  c->stats.n_samples = (int64_t)c->samples.size();
  return MIMOSE_OK;
}

mimose_status mimose_step(mimose_ctx* c, float lr, float b1, float b2, float eps, float wd) {
  Range rg("mimose_step");
  if (mimose_status s = check_ready(c)) return s;
  if (!c->bwd_done) return fail(c, MIMOSE_E_STATE, "step without a backward");
  if (!c->device) return MIMOSE_OK;
  if (c->opt_fused) {   // the per-bucket updates were launched during backward
    // The update has been applied with the mimose_set_optimizer arguments:
    // order the compute stream behind it and advance t whatever this call's
    // arguments say, then report a mismatch.
    CK(cudaEventRecord(c->ev_opt_done, c->opt_st));
    CK(cudaStreamWaitEvent(c->st, c->ev_opt_done, 0));
    if (c->zero1) {   // the weight all-gathers follow the shard updates on the comm stream
      CK(cudaEventRecord(c->ev_comm_done, c->comm_st));
      CK(cudaStreamWaitEvent(c->st, c->ev_comm_done, 0));
    }
    c->adam_t++;
    c->fwd_done = false;
    c->step_pending = false;
    if (lr != c->opt_lr || b1 != c->opt_b1 || b2 != c->opt_b2 || eps != c->opt_eps || wd != c->opt_wd)
      return fail(c, MIMOSE_E_INVALID,
                  "fused optimizer: step arguments differ from mimose_set_optimizer (the update used the latter)");
    return MIMOSE_OK;
  }
  if (c->comm) {
    CK(cudaEventRecord(c->ev_comm_done, c->comm_st));
    CK(cudaStreamWaitEvent(c->st, c->ev_comm_done, 0));
  }
  if (c->zero1) {   // unfused ZeRO-1: shard updates + all-gathers, bucket by bucket, on the compute stream
    c->opt_lr = lr; c->opt_b1 = b1; c->opt_b2 = b2; c->opt_eps = eps; c->opt_wd = wd;
    for (int evi = 0; evi < (int)c->bk_b0.size(); ++evi) {
      // the reduce-scatter already ran during backward; redo only the update + all-gather
      const int W = c->cfg.world, r = c->cfg.rank;
      const int64_t b0 = c->bk_b0[evi], cb = (c->bk_b1[evi] - b0) / W, sh = c->bk_sh[evi];
      const double t = (double)(c->adam_t + 1);
      const double bc1 = 1.0 - std::pow((double)b1, t), bc2 = 1.0 - std::pow((double)b2, t);
      char* wsh = c->w + (b0 + r * cb) * c->e;
      adamw(c->dt, wsh, c->master ? c->master + sh : nullptr, c->grad + b0 + r * cb, c->m + sh, c->v + sh, cb, lr, b1,
            b2, eps, wd, (float)bc1, (float)bc2, 1.0f / (float)W, c->st);
      NK(ncclAllGather(wsh, c->w + b0 * c->e, (size_t)cb, c->dt == DT_F32 ? ncclFloat : ncclBfloat16, c->comm,
                       c->st));
    }
    c->adam_t++;
    c->fwd_done = false;
    return MIMOSE_OK;
  }
  c->adam_t++;
  const double bc1 = 1.0 - std::pow((double)b1, (double)c->adam_t);
  const double bc2 = 1.0 - std::pow((double)b2, (double)c->adam_t);
  adamw(c->dt, c->w, c->master, c->grad, c->m, c->v, c->npad, lr, b1, b2, eps, wd, (float)bc1, (float)bc2,
        1.0f / (float)c->cfg.world, c->st);
  CK(cudaGetLastError());
  c->fwd_done = false;
  return MIMOSE_OK;
}

mimose_status mimose_set_optimizer(mimose_ctx* c, float lr, float b1, float b2, float eps, float wd, int32_t fused) {
  if (mimose_status s = check_ready(c)) return s;
  if (c->fwd_done && !c->bwd_done) return fail(c, MIMOSE_E_STATE, "set_optimizer inside a step");
  if (c->step_pending) return fail(c, MIMOSE_E_STATE, "set_optimizer before mimose_step closed the step");
  c->opt_fused = fused != 0;
  c->opt_lr = lr; c->opt_b1 = b1; c->opt_b2 = b2; c->opt_eps = eps; c->opt_wd = wd;
  return MIMOSE_OK;
}

mimose_status mimose_set_planner(mimose_ctx* c, int32_t kind) {
  if (mimose_status s = check_ready(c)) return s;
  if (kind != PLANNER_GREEDY && kind != PLANNER_EXACT && kind != PLANNER_EXACT_TIME)
    return fail(c, MIMOSE_E_INVALID, "unknown planner");
  if (kind != c->planner) c->cache.clear();      // cached plans belong to the previous planner
  c->planner = kind;
  return MIMOSE_OK;
}

static mimose_status plan_impl(mimose_ctx* c, int64_t x, int64_t xt, mimose_plan_t* out) {
  if (mimose_status s = check_ready(c)) return s;
  if (!out || x <= 0 || (c->cfg.arch == 2 && (xt <= 0 || x >= (1LL << 31) || xt >= (1LL << 31))))
    return fail(c, MIMOSE_E_INVALID, "bad plan arguments");
  if (c->phase != MIMOSE_PHASE_RESPONSIVE) return fail(c, MIMOSE_E_NOT_READY, "estimator not fitted yet");
  c->stats.plan_calls++;
  const int64_t key = c->cfg.arch == 2 ? (x << 32) | xt : x;
  auto it = c->cache.find(key);
  if (it != c->cache.end()) {
    c->stats.plan_cache_hits++;
    *out = it->second;
    out->from_cache = 1;
  } else {
    c->stats.plan_cache_misses++;
    auto t0 = std::chrono::steady_clock::now();
    const bool two = c->cfg.arch == 2;
    const Series s = two ? c->est.predict2(x, xt) : c->est.predict(x);
    const PlanResult pr =
        c->planner == PLANNER_EXACT ? plan_exact(s, c->ar.budget, c->cfg.reserve_bytes)
        : c->planner == PLANNER_EXACT_TIME
            ? plan_exact_cost(s, two ? c->est.predict_cost2(x, xt) : c->est.predict_cost(x), c->ar.budget,
                              c->cfg.reserve_bytes)
            : plan_greedy(s, c->ar.budget, c->cfg.reserve_bytes, c->cfg.bucket_num, c->cfg.bucket_den);
    c->stats.planner_us_total +=
        std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count();
    mimose_plan_t p{};
    p.drop_mask = pr.drop_mask;
    p.n_dropped = __builtin_popcountll(pr.drop_mask);
    p.from_cache = 0;
    p.input_size = x;
    p.predicted_peak = pr.peak;
    p.budget = c->ar.budget - c->cfg.reserve_bytes;
    p.status = pr.feasible ? MIMOSE_OK : MIMOSE_E_INFEASIBLE;
    c->cache[key] = p;
    *out = p;
  }
  c->stats.last_drop_mask = out->drop_mask;
  c->stats.last_n_dropped = out->n_dropped;
  c->stats.last_predicted_peak = out->predicted_peak;
  if (out->status != MIMOSE_OK) return fail(c, MIMOSE_E_INFEASIBLE, "no plan fits the budget");
  return MIMOSE_OK;
}

mimose_status mimose_plan(mimose_ctx* c, int64_t x, mimose_plan_t* out) {
  if (c && c->cfg.arch == 2) return fail(c, MIMOSE_E_INVALID, "encoder-decoder: use mimose_plan2 (2-D key)");
  return plan_impl(c, x, 0, out);
}

mimose_status mimose_plan2(mimose_ctx* c, int64_t x, int64_t xt, mimose_plan_t* out) {
  if (c && c->cfg.arch != 2) return fail(c, MIMOSE_E_INVALID, "mimose_plan2 is for encoder-decoder contexts");
  return plan_impl(c, x, xt, out);
}

int32_t mimose_tc_available(void) { return tc_available() ? 1 : 0; }

mimose_status mimose_debug_gemm_ex(int32_t epi, int32_t M, int32_t N, int32_t K, const void* A, int64_t a_sm,
                                   int64_t a_sk, const void* B, int64_t b_sn, int64_t b_sk, void* Cp, int64_t ldc,
                                   void* C2, const void* bias, const void* res, int64_t ldr, const void* aux,
                                   int64_t ldx, int32_t split, int32_t use_tc, void* stream) {
  if (epi < 0 || epi > (int)EPI_ACC_F32) return MIMOSE_E_INVALID;
  GemmArgs g;
  g.M = M; g.N = N; g.K = K;
  g.A = A; g.a_sm = a_sm; g.a_sk = a_sk;
  g.B = B; g.b_sn = b_sn; g.b_sk = b_sk;
  g.C = Cp; g.ldc = ldc; g.C2 = C2; g.bias = bias; g.res = res; g.ldr = ldr; g.aux = aux; g.ldx = ldx;
  g.split = split < 1 ? 1 : split;
  g.split_stride = (int64_t)M * ldc;
  g.drop.enabled = 1; g.drop.seed_lo = 7; g.drop.seed_hi = 0; g.drop.site = 0; g.drop.step = 1;
  drop_set_keys(g.drop);
  g.drop.thresh = 3865470566u; g.drop.scale = (float)(1.0 / 0.9);
  gemm(DT_BF16, (Epi)epi, g, (cudaStream_t)stream, use_tc != 0);
  return cudaGetLastError() == cudaSuccess ? MIMOSE_OK : MIMOSE_E_CUDA;
}

mimose_status mimose_debug_gemm_grouped(int32_t M1, int32_t N1, int32_t K1, const void* A1, int64_t a_sm1,
                                        int64_t a_sk1, const void* B1, int64_t b_sn1, int64_t b_sk1, void* C1,
                                        int32_t M2, int32_t N2, int32_t K2, const void* A2, int64_t a_sm2,
                                        int64_t a_sk2, const void* B2, int64_t b_sn2, int64_t b_sk2, void* C2,
                                        void* stream) {
  GemmArgs g1, g2;
  g1.M = M1; g1.N = N1; g1.K = K1; g1.A = A1; g1.a_sm = a_sm1; g1.a_sk = a_sk1;
  g1.B = B1; g1.b_sn = b_sn1; g1.b_sk = b_sk1; g1.C = C1; g1.ldc = N1;
  g2.M = M2; g2.N = N2; g2.K = K2; g2.A = A2; g2.a_sm = a_sm2; g2.a_sk = a_sk2;
  g2.B = B2; g2.b_sn = b_sn2; g2.b_sk = b_sk2; g2.C = C2; g2.ldc = N2;
  if (!gemm_tc_grouped(g1, g2, 256, (cudaStream_t)stream)) return MIMOSE_E_INVALID;
  return cudaGetLastError() == cudaSuccess ? MIMOSE_OK : MIMOSE_E_CUDA;
}

void mimose_debug_options(int32_t gemm_mode, int32_t attn_tc) {
  if (gemm_mode >= 0) set_gemm_mode(gemm_mode);
  if (attn_tc >= 0) set_attn_tc(attn_tc != 0);
}

mimose_status mimose_debug_gemm(int32_t epi, int32_t M, int32_t N, int32_t K, const void* A, int64_t a_sm,
                                int64_t a_sk, const void* B, int64_t b_sn, int64_t b_sk, void* Cp, int64_t ldc,
                                const void* bias, int32_t split, int32_t use_tc, void* stream) {
  if (epi != EPI_STORE && epi != EPI_BIAS && epi != EPI_F32) return MIMOSE_E_INVALID;
  GemmArgs g;
  g.M = M; g.N = N; g.K = K;
  g.A = A; g.a_sm = a_sm; g.a_sk = a_sk;
  g.B = B; g.b_sn = b_sn; g.b_sk = b_sk;
  g.C = Cp; g.ldc = ldc; g.bias = bias;
  g.split = split < 1 ? 1 : split;
  g.split_stride = (int64_t)M * ldc;
  gemm(DT_BF16, (Epi)epi, g, (cudaStream_t)stream, use_tc != 0);
  return cudaGetLastError() == cudaSuccess ? MIMOSE_OK : MIMOSE_E_CUDA;
}

mimose_status mimose_nccl_unique_id(void* out128) {
  if (!out128) return MIMOSE_E_INVALID;
  ncclUniqueId id;
  if (ncclGetUniqueId(&id) != ncclSuccess) return MIMOSE_E_NCCL;
  std::memcpy(out128, &id, sizeof(id));
  return MIMOSE_OK;
}

mimose_status mimose_probe(mimose_ctx* c, int32_t kind) {
  if (!c) return MIMOSE_E_INVALID;
  c->probe = kind;
  c->probe_used = 0;
  c->probe_flops = 0.0;
  c->probe_shape.clear();
  return MIMOSE_OK;
}

mimose_status mimose_probe_read(mimose_ctx* c, double* ms, double* flops, int64_t* launches) {
  if (!c || !ms || !flops || !launches) return MIMOSE_E_INVALID;
  double tot = 0.0;
  if (c->device && c->probe_used) {
    CK(cudaStreamSynchronize(c->st));
    // MIMOSE_PROBE_DUMP=<path>: one CSV line per probed launch (M, N, K, epi, us);
    // a grouped weight-gradient launch is (T, N1 K1 + N2 K2, tile width, -1)
    const char* dump = std::getenv("MIMOSE_PROBE_DUMP");
    FILE* f = dump ? std::fopen(dump, "a") : nullptr;
    for (size_t i = 0; i + 1 < c->probe_used; i += 2) {
      float t = 0.f;
      CK(cudaEventElapsedTime(&t, c->probe_ev[i], c->probe_ev[i + 1]));
      tot += t;
      if (f && i / 2 < c->probe_shape.size()) {
        const auto& sh = c->probe_shape[i / 2];
        std::fprintf(f, "%lld,%lld,%lld,%lld,%.3f\n", (long long)sh[0], (long long)sh[1], (long long)sh[2],
                     (long long)sh[3], 1000.0 * t);
      }
    }
    if (f) std::fclose(f);
  }
  *ms = tot;
  *flops = c->probe_flops;
  *launches = (int64_t)(c->probe_used / 2);
  return MIMOSE_OK;
}

mimose_status mimose_get_stats(const mimose_ctx* c, mimose_stats* out) {
  if (!c || !out) return MIMOSE_E_INVALID;
  *out = c->stats;
  out->live_bytes = c->ar.live();
  out->phase = c->phase;
  out->kernel_launches = kernel_launch_count();
  out->allreduce_calls = c->stats_allreduce_calls;
  out->allreduce_bytes = c->stats_allreduce_bytes;
  out->plan_checks = c->stats_plan_checks;
  out->comm_nranks = 0;
  if (c->comm) {
    int n = 0;
    if (ncclCommCount(c->comm, &n) == ncclSuccess) out->comm_nranks = n;
  }
  return MIMOSE_OK;
}

mimose_status mimose_phase(const mimose_ctx* c, int32_t* p) {
  if (!c || !p) return MIMOSE_E_INVALID;
  *p = c->phase;
  return MIMOSE_OK;
}

mimose_status mimose_get_sample(const mimose_ctx* c, int32_t i, mimose_sample* out) {
  if (!c || !out || i < 0 || i >= (int)c->samples.size()) return MIMOSE_E_INVALID;
  const_cast<mimose_ctx*>(c)->err.clear();
  resolve_times(const_cast<mimose_ctx*>(c));
  const Sample& s = c->samples[i];
  std::memset(out, 0, sizeof(*out));
  out->x = s.x; out->C = s.C; out->E = s.E; out->Hd = s.Hd; out->Th = s.Th; out->Tb = s.Tb; out->Te = s.Te;
  out->xt = s.xt;
  for (size_t l = 0; l < s.a.size(); ++l) { out->a[l] = s.a[l]; out->y[l] = s.y[l]; out->t_ms[l] = s.t_ms[l]; }
  return MIMOSE_OK;
}

mimose_status mimose_dry_run2(mimose_ctx* c, int32_t n_seqs, int32_t seq_len, int32_t dec_len, uint64_t mask,
                              int64_t* peak) {
  if (!c || !peak) return MIMOSE_E_INVALID;
  mimose_batch bt{nullptr, nullptr, nullptr, nullptr, n_seqs, seq_len, 1, nullptr, nullptr, dec_len, 0};
  if (mimose_status s = check_batch(c, &bt)) return s;
  bool breach;
  const bool enf = c->ar.enforce;
  c->ar.enforce = false;
  dry_step(c, n_seqs, seq_len, mask, false, peak, &breach, nullptr, c->cfg.arch == 2 ? dec_len : 0);
  c->ar.enforce = enf;
  return MIMOSE_OK;
}
mimose_status mimose_dry_run(mimose_ctx* c, int32_t n_seqs, int32_t seq_len, uint64_t mask, int64_t* peak) {
  return mimose_dry_run2(c, n_seqs, seq_len, c && c->cfg.arch == 2 ? seq_len : 0, mask, peak);
}

mimose_status mimose_dry_collect2(mimose_ctx* c, int32_t n_seqs, int32_t seq_len, int32_t dec_len, mimose_sample* out) {
  if (!c || !out) return MIMOSE_E_INVALID;
  mimose_batch bt{nullptr, nullptr, nullptr, nullptr, n_seqs, seq_len, 1, nullptr, nullptr, dec_len, 0};
  if (mimose_status s = check_batch(c, &bt)) return s;
  const int L = n_units(c);
  Sample smp;
  smp.a.assign(L, 0); smp.y.assign(L, 0); smp.t_ms.assign(L, 0.f);
  int64_t peak;
  bool breach;
  const bool enf = c->ar.enforce;
  c->ar.enforce = false;
  dry_step(c, n_seqs, seq_len, ~0ull, true, &peak, &breach, &smp, c->cfg.arch == 2 ? dec_len : 0);
  c->ar.enforce = enf;
  std::memset(out, 0, sizeof(*out));
  out->x = (int64_t)n_seqs * seq_len; out->C = c->ar.C;
  out->xt = c->cfg.arch == 2 ? (int64_t)n_seqs * dec_len : 0;
  out->E = smp.E; out->Hd = smp.Hd; out->Th = smp.Th; out->Tb = smp.Tb; out->Te = smp.Te;
  for (int l = 0; l < L; ++l) { out->a[l] = smp.a[l]; out->y[l] = smp.y[l]; }
  return MIMOSE_OK;
}
mimose_status mimose_dry_collect(mimose_ctx* c, int32_t n_seqs, int32_t seq_len, mimose_sample* out) {
  return mimose_dry_collect2(c, n_seqs, seq_len, c && c->cfg.arch == 2 ? seq_len : 0, out);
}

static Series to_series(const mimose_series* s) {
  Series r;
  r.C = s->C; r.E = s->E; r.Hd = s->Hd; r.Th = s->Th; r.Tb = s->Tb; r.Te = s->Te;
  r.a.assign(s->a, s->a + s->n_layers);
  r.y.assign(s->y, s->y + s->n_layers);
  return r;
}

int64_t mimose_predicted_peak(const mimose_series* s, uint64_t mask) { return predicted_peak(to_series(s), mask); }

mimose_status mimose_plan_series(const mimose_series* s, int64_t budget, int64_t reserve, int32_t bn, int32_t bd,
                                 uint64_t* mask, int64_t* peak) {
  if (!s || !mask || !peak || s->n_layers < 1 || s->n_layers > 64 || bd <= 0) return MIMOSE_E_INVALID;
  const PlanResult r = bn == 0 ? plan_exact(to_series(s), budget, reserve) : plan_greedy(to_series(s), budget, reserve, bn, bd);
  *mask = r.drop_mask;
  *peak = r.peak;
  return r.feasible ? MIMOSE_OK : MIMOSE_E_INFEASIBLE;
}

mimose_status mimose_plan_series_cost(const mimose_series* s, const int64_t* cost, int64_t budget, int64_t reserve,
                                      uint64_t* mask, int64_t* peak) {
  if (!s || !cost || !mask || !peak || s->n_layers < 1 || s->n_layers > 64) return MIMOSE_E_INVALID;
  const PlanResult r =
      plan_exact_cost(to_series(s), std::vector<int64_t>(cost, cost + s->n_layers), budget, reserve);
  *mask = r.drop_mask;
  *peak = r.peak;
  return r.feasible ? MIMOSE_OK : MIMOSE_E_INFEASIBLE;
}

mimose_status mimose_fit_predict(const int64_t* xs, const int64_t* ys, int32_t n, int32_t degree,
                                 const int64_t* xe, int32_t ne, int64_t* out) {
  if (!xs || !ys || n < 1 || !xe || !out || degree < 0 || degree > 2) return MIMOSE_E_INVALID;
  Poly p;
  p.fit(std::vector<int64_t>(xs, xs + n), std::vector<int64_t>(ys, ys + n), degree);
  for (int i = 0; i < ne; ++i) out[i] = p.predict(xe[i]);
  return MIMOSE_OK;
}

}  // extern "C"
