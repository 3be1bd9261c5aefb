// Attention of the post-LN encoder layer (Fig. 8: Q K^T ->
// scale -> softmax -> x V), flash-style: the S x S score/probability tensors
// are never stored (so the per-layer activation bytes are linear in S; the
// estimator's quadratic term then fits ~0 — DESIGN "Memory model").  Only the
// row log-sum-exp is kept for backward.  Dropout on the probabilities uses the
// Philox site (KIND_ATTN_PROBS, layer), element ((b*h + head)*S + q)*S + k.
//
// This is the first, SIMT version (fp32 FMA, K/V tiles staged in shared
// memory, one query row per thread, exact two-pass softmax).  Backward is
// deterministic: pass A (key-outer) produces dK, dV; pass B (query-outer)
// produces dQ; no atomics.
#include "kernels.h"

#include <cmath>

namespace mimose {

static inline int cdiv(int64_t a, int64_t b) { return (int)((a + b - 1) / b); }

// tcgen05 versions (kernels_attn_tc.cu): bf16, head dim 64, S <= 128
bool attn_fwd_tc(const void* qkv, const int32_t* lengths, void* O, float* lse, int B, int S, int H, int h,
                 Drop drop, cudaStream_t st, bool causal);
bool attn_bwd_tc(const void* qkv, const void* O, const void* dO, const float* lse, const int32_t* lengths,
                 void* dqkv, int B, int S, int H, int h, Drop drop, cudaStream_t st, bool causal);

// tcgen05 versions for 128 < S <= 1024 (kernels_attn_tcl.cu)
bool attn_fwd_tcl(const void* qkv, const int32_t* lengths, void* O, float* lse, int B, int S, int H, int h,
                  Drop drop, cudaStream_t st, bool causal);
bool attn_bwd_tcl(const void* qkv, const void* O, const void* dO, const float* lse, const int32_t* lengths,
                  float* Dbuf, void* dqkv, int B, int S, int H, int h, Drop drop, cudaStream_t st, bool causal);

static bool g_attn_tc = true;
void set_attn_tc(bool on) { g_attn_tc = on; }
bool attn_tc_enabled() { return g_attn_tc; }

constexpr int AT = 64;  // forward: rows per CTA / keys per tile
constexpr int BT = 32;  // backward tile (4 fp32 tiles must fit the 48 KB static smem)

template <typename E, int D>
__global__ void __launch_bounds__(AT) k_attn_fwd(const E* __restrict__ qkv, const int32_t* __restrict__ lengths,
                                                 E* __restrict__ O, float* __restrict__ lse, int S, int H,
                                                 int h, float scale, Drop drop, int causal) {
  pdl_enter();
  __shared__ float Ks[AT][D + 1];
  __shared__ float Vs[AT][D + 1];
  const int bh = blockIdx.y, b = bh / h, hd = bh % h;
  const int q = blockIdx.x * AT + threadIdx.x;
  const int len = lengths[b];
  const int64_t ld = 3 * (int64_t)H;
  const bool active = q < S;
  const int kl = causal ? min(len, q + 1) : len;      // keys visible to this query
  float qv[D];
  const E* qrow = qkv + ((int64_t)b * S + (active ? q : 0)) * ld + hd * D;
#pragma unroll
  for (int c = 0; c < D; ++c) qv[c] = active ? ldf(qrow + c) * scale : 0.f;
  // pass 1: row max and normaliser
  float m = -INFINITY, l = 0.f;
  for (int k0 = 0; k0 < len; k0 += AT) {
    __syncthreads();
    for (int i = threadIdx.x; i < AT * D; i += AT) {
      const int r = i / D, c = i % D;
      const int kk = k0 + r;
      Ks[r][c] = kk < len ? ldf(qkv + ((int64_t)b * S + kk) * ld + H + hd * D + c) : 0.f;
    }
    __syncthreads();
    const int kend = min(AT, kl - k0);
    for (int j = 0; j < kend; ++j) {
      float s = 0.f;
#pragma unroll
      for (int c = 0; c < D; ++c) s += qv[c] * Ks[j][c];
      if (s > m) { l = l * expf(m - s) + 1.f; m = s; } else { l += expf(s - m); }
    }
  }
  const float L = m + logf(l);
  // pass 2: O = sum_k drop(exp(s - L)) v_k
  float o[D];
#pragma unroll
  for (int c = 0; c < D; ++c) o[c] = 0.f;
  const uint64_t ebase = (((uint64_t)b * h + hd) * S + (uint64_t)(active ? q : 0)) * S;
  for (int k0 = 0; k0 < len; k0 += AT) {
    __syncthreads();
    for (int i = threadIdx.x; i < AT * D; i += AT) {
      const int r = i / D, c = i % D;
      const int kk = k0 + r;
      const E* base = qkv + ((int64_t)b * S + kk) * ld + hd * D + c;
      Ks[r][c] = kk < len ? ldf(base + H) : 0.f;
      Vs[r][c] = kk < len ? ldf(base + 2 * H) : 0.f;
    }
    __syncthreads();
    const int kend = min(AT, kl - k0);
    for (int j = 0; j < kend; ++j) {
      float s = 0.f;
#pragma unroll
      for (int c = 0; c < D; ++c) s += qv[c] * Ks[j][c];
      const float p = expf(s - L) * drop_factor(drop, ebase + k0 + j);
#pragma unroll
      for (int c = 0; c < D; ++c) o[c] += p * Vs[j][c];
    }
  }
  if (!active) return;
  E* orow = O + ((int64_t)b * S + q) * H + hd * D;
#pragma unroll
  for (int c = 0; c < D; ++c) stf(orow + c, o[c]);
  lse[((int64_t)b * h + hd) * S + q] = L;
}

void attn_fwd(DType dt, const void* qkv, const int32_t* lengths, void* O, float* lse, int B, int S, int H,
              int h, Drop drop, cudaStream_t st, bool causal) {
  note_launch(1);
  if (dt == DT_BF16 && attn_tc_enabled() &&
      (attn_fwd_tc(qkv, lengths, O, lse, B, S, H, h, drop, st, causal) ||
       attn_fwd_tcl(qkv, lengths, O, lse, B, S, H, h, drop, st, causal)))
    return;
  const int D = H / h;
  const float scale = 1.0f / sqrtf((float)D);
  dim3 grid(cdiv(S, AT), B * h);
  auto go = [&](auto* tag, auto dconst) {
    using E = std::remove_pointer_t<decltype(tag)>;
    constexpr int DD = decltype(dconst)::value;
    launch_k(k_attn_fwd<E, DD>, grid, AT, 0, st, (const E*)qkv, lengths, (E*)O, lse, S, H, h, scale, drop, causal ? 1 : 0);
  };
  if (dt == DT_F32) {
    if (D == 32) go((float*)nullptr, std::integral_constant<int, 32>{});
    else go((float*)nullptr, std::integral_constant<int, 64>{});
  } else {
    if (D == 32) go((__nv_bfloat16*)nullptr, std::integral_constant<int, 32>{});
    else go((__nv_bfloat16*)nullptr, std::integral_constant<int, 64>{});
  }
}

// D[b,h,q] = sum_c dO[q,c] O[q,c] (per head)
template <typename E>
__global__ void k_attn_dot(const E* __restrict__ O, const E* __restrict__ dO, float* __restrict__ Dbuf,
                           int B, int S, int H, int h) {
  pdl_enter();
  const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (w >= B * h * S) return;
  const int q = w % S, bh = w / S, b = bh / h, hd = bh % h;
  const int D = H / h;
  const int64_t off = ((int64_t)b * S + q) * H + hd * D;
  float acc = 0.f;
  for (int c = lane; c < D; c += 32) acc += ldf(O + off + c) * ldf(dO + off + c);
  acc = warp_sum(acc);
  if (lane == 0) Dbuf[w] = acc;
}

// pass A: thread per key j; loop over valid queries; dK, dV in registers.
template <typename E, int D>
__global__ void __launch_bounds__(BT) k_attn_bwd_kv(const E* __restrict__ qkv, const E* __restrict__ dO,
                                                    const float* __restrict__ lse, const float* __restrict__ Dbuf,
                                                    const int32_t* __restrict__ lengths, E* __restrict__ dqkv,
                                                    int S, int H, int h, float scale, Drop drop, int causal) {
  pdl_enter();
  __shared__ float Qs[BT][D + 1];
  __shared__ float dOs[BT][D + 1];
  __shared__ float Kt[D][BT + 1];
  __shared__ float Vt[D][BT + 1];
  __shared__ float Ls[BT], Ds[BT];
  const int bh = blockIdx.y, b = bh / h, hd = bh % h;
  const int j0 = blockIdx.x * BT;
  const int j = j0 + threadIdx.x;
  const int len = lengths[b];
  const int64_t ld = 3 * (int64_t)H;
  for (int i = threadIdx.x; i < BT * D; i += BT) {
    const int r = i / D, c = i % D;
    const int kk = j0 + r;
    const E* base = qkv + ((int64_t)b * S + min(kk, S - 1)) * ld + hd * D + c;
    Kt[c][r] = kk < len ? ldf(base + H) : 0.f;
    Vt[c][r] = kk < len ? ldf(base + 2 * H) : 0.f;
  }
  float dk[D], dv[D];
#pragma unroll
  for (int c = 0; c < D; ++c) { dk[c] = 0.f; dv[c] = 0.f; }
  const bool keyvalid = j < len;
  for (int q0 = 0; q0 < len; q0 += BT) {     // padded query rows carry exactly zero gradient
    __syncthreads();
    for (int i = threadIdx.x; i < BT * D; i += BT) {
      const int r = i / D, c = i % D;
      const int qq = q0 + r;
      const int64_t off = ((int64_t)b * S + min(qq, S - 1)) * H + hd * D + c;
      Qs[r][c] = qq < len ? ldf(qkv + ((int64_t)b * S + min(qq, S - 1)) * ld + hd * D + c) * scale : 0.f;
      dOs[r][c] = qq < len ? ldf(dO + off) : 0.f;
    }
    if (threadIdx.x < BT) {
      const int qq = q0 + threadIdx.x;
      Ls[threadIdx.x] = qq < len ? lse[((int64_t)b * h + hd) * S + qq] : 0.f;
      Ds[threadIdx.x] = qq < len ? Dbuf[((int64_t)b * h + hd) * S + qq] : 0.f;
    }
    __syncthreads();
    if (!keyvalid) continue;
    const int qend = min(BT, len - q0);
    for (int i = 0; i < qend; ++i) {
      if (causal && q0 + i < j) continue;           // key j invisible to earlier queries
      float s = 0.f, dp = 0.f;
#pragma unroll
      for (int c = 0; c < D; ++c) { s += Qs[i][c] * Kt[c][threadIdx.x]; dp += dOs[i][c] * Vt[c][threadIdx.x]; }
      const float p = expf(s - Ls[i]);           // same s = (q*scale).k as the forward
      const uint64_t e = (((uint64_t)b * h + hd) * S + (uint64_t)(q0 + i)) * S + j;
      const float f = drop_factor(drop, e);
      const float pd = p * f;
      const float ds = p * (dp * f - Ds[i]);     // dK = sum ds * (q*scale)
#pragma unroll
      for (int c = 0; c < D; ++c) { dv[c] += pd * dOs[i][c]; dk[c] += ds * Qs[i][c]; }
    }
  }
  if (j >= S) return;
  E* row = dqkv + ((int64_t)b * S + j) * ld + hd * D;
#pragma unroll
  for (int c = 0; c < D; ++c) { stf(row + H + c, dk[c]); stf(row + 2 * H + c, dv[c]); }
}

// pass B: thread per query i; loop over valid keys; dQ in registers.
template <typename E, int D>
__global__ void __launch_bounds__(BT) k_attn_bwd_q(const E* __restrict__ qkv, const E* __restrict__ dO,
                                                   const float* __restrict__ lse, const float* __restrict__ Dbuf,
                                                   const int32_t* __restrict__ lengths, E* __restrict__ dqkv,
                                                   int S, int H, int h, float scale, Drop drop, int causal) {
  pdl_enter();
  __shared__ float Qt[D][BT + 1];
  __shared__ float dOt[D][BT + 1];
  __shared__ float Ks[BT][D + 1];
  __shared__ float Vs[BT][D + 1];
  const int bh = blockIdx.y, b = bh / h, hd = bh % h;
  const int i0 = blockIdx.x * BT;
  const int i = i0 + threadIdx.x;
  const int len = lengths[b];
  const int64_t ld = 3 * (int64_t)H;
  for (int t = threadIdx.x; t < BT * D; t += BT) {
    const int r = t / D, c = t % D;
    const int qq = i0 + r;
    const int qc = min(qq, S - 1);
    Qt[c][r] = qq < len ? ldf(qkv + ((int64_t)b * S + qc) * ld + hd * D + c) * scale : 0.f;
    dOt[c][r] = qq < len ? ldf(dO + ((int64_t)b * S + qc) * H + hd * D + c) : 0.f;
  }
  const bool valid = i < len;
  const float Li = valid ? lse[((int64_t)b * h + hd) * S + i] : 0.f;
  const float Di = valid ? Dbuf[((int64_t)b * h + hd) * S + i] : 0.f;
  float dq[D];
#pragma unroll
  for (int c = 0; c < D; ++c) dq[c] = 0.f;
  for (int k0 = 0; k0 < len; k0 += BT) {
    __syncthreads();
    for (int t = threadIdx.x; t < BT * D; t += BT) {
      const int r = t / D, c = t % D;
      const int kk = k0 + r;
      const E* base = qkv + ((int64_t)b * S + min(kk, S - 1)) * ld + hd * D + c;
      Ks[r][c] = kk < len ? ldf(base + H) : 0.f;
      Vs[r][c] = kk < len ? ldf(base + 2 * H) : 0.f;
    }
    __syncthreads();
    if (!valid) continue;
    const int kend = min(BT, (causal ? min(len, i + 1) : len) - k0);
    for (int jj = 0; jj < kend; ++jj) {
      float s = 0.f, dp = 0.f;
#pragma unroll
      for (int c = 0; c < D; ++c) { s += Qt[c][threadIdx.x] * Ks[jj][c]; dp += dOt[c][threadIdx.x] * Vs[jj][c]; }
      const float p = expf(s - Li);
      const uint64_t e = (((uint64_t)b * h + hd) * S + (uint64_t)i) * S + k0 + jj;
      const float f = drop_factor(drop, e);
      const float ds = p * (dp * f - Di) * scale;
#pragma unroll
      for (int c = 0; c < D; ++c) dq[c] += ds * Ks[jj][c];
    }
  }
  if (i >= S) return;
  E* row = dqkv + ((int64_t)b * S + i) * ld + hd * D;
#pragma unroll
  for (int c = 0; c < D; ++c) stf(row + c, valid ? dq[c] : 0.f);
}

void attn_bwd(DType dt, const void* qkv, const void* O, const void* dO, const float* lse,
              const int32_t* lengths, float* Dbuf, void* dqkv, int B, int S, int H, int h, Drop drop,
              cudaStream_t st, bool causal) {
  if (dt == DT_BF16 && attn_tc_enabled() &&
      attn_bwd_tc(qkv, O, dO, lse, lengths, dqkv, B, S, H, h, drop, st, causal)) {
    note_launch(1);
    return;
  }
  if (dt == DT_BF16 && attn_tc_enabled() &&
      attn_bwd_tcl(qkv, O, dO, lse, lengths, Dbuf, dqkv, B, S, H, h, drop, st, causal)) {
    note_launch(2);
    return;
  }
  const int D = H / h;
  const float scale = 1.0f / sqrtf((float)D);
  dim3 grid(cdiv(S, BT), B * h);
  note_launch(3);
  auto go = [&](auto* tag, auto dconst) {
    using E = std::remove_pointer_t<decltype(tag)>;
    constexpr int DD = decltype(dconst)::value;
    launch_k(k_attn_dot<E>, cdiv((int64_t)B * h * S, 8), 256, 0, st, (const E*)O, (const E*)dO, Dbuf, B, S, H, h);
    launch_k(k_attn_bwd_kv<E, DD>, grid, BT, 0, st, (const E*)qkv, (const E*)dO, lse, Dbuf, lengths, (E*)dqkv, S, H, h,
                                             scale, drop, causal ? 1 : 0);
    launch_k(k_attn_bwd_q<E, DD>, grid, BT, 0, st, (const E*)qkv, (const E*)dO, lse, Dbuf, lengths, (E*)dqkv, S, H, h,
                                            scale, drop, causal ? 1 : 0);
  };
  if (dt == DT_F32) {
    if (D == 32) go((float*)nullptr, std::integral_constant<int, 32>{});
    else go((float*)nullptr, std::integral_constant<int, 64>{});
  } else {
    if (D == 32) go((__nv_bfloat16*)nullptr, std::integral_constant<int, 32>{});
    else go((__nv_bfloat16*)nullptr, std::integral_constant<int, 64>{});
  }
}

}  // namespace mimose
