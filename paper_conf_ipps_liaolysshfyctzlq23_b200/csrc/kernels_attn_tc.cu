// Attention on the 5th-gen tensor cores (tcgen05 / TMEM / TMA), head dim 64,
// whole sequence in one 128-row tile (S <= 128: the BERT-base workload range).
// PAPER.md P:160 / Fig. 8: S = Q K^T -> scale -> softmax -> x V.
//
// One CTA (4 warps) per (sequence b, head h); thread t owns TMEM lane t, i.e.
// query row t (S, dP, O, dQ) or key row t (dV, dK).
//
// forward:  TMA Q,K,V tiles -> S = Q K^T (TMEM) -> row softmax + Philox dropout
//           in registers -> P~ (bf16, 128B-swizzled smem) -> O = P~ V (TMEM)
//           -> O (bf16) and LSE (fp32) to global.
// backward: TMA Q,K,V,dO -> S = Q K^T, dP~ = dO V^T (TMEM) -> P = exp(S - LSE),
//           dS = P (dP~ f - D), D = rowsum(dO * O) -> P~, dS tiles (smem) ->
//           dV = P~^T dO, dK = dS^T Q, dQ = dS K (the same smem tile read as an
//           MN-major or a K-major operand) -> dQKV (bf16).  No atomics.
// Dropout element e = ((b*h + head)*S + q)*S + k, site (KIND_ATTN_PROBS, layer),
// identical to the SIMT kernels and the oracle.
#include <cuda.h>

#include <mutex>

#include "kernels.h"
#include "tc_common.cuh"

namespace mimose {

constexpr int AQ = 128;                  // rows of the tile (queries / keys)
constexpr int AD = 64;                   // head dim
constexpr int TILE = AQ * AD * 2;        // 16 KB: one [128 x 64] bf16 SW128 tile
constexpr int PT = AQ * AQ * 2;          // 32 KB: one [128 x 128] bf16 tile (2 atoms)

struct AttnArgs {
  int S, H, h, B;              // S: query rows per sequence
  int Sk;                      // key rows per sequence (== S for self-attention)
  int qcol, kcol, vcol;        // column bases of Q (in tq), K and V (in tk): 0, H, 2H for a [T, 3H] qkv
  int ldo, ocq, ock, ocv;      // backward: dQ row stride, column bases of dQ / dK / dV
  int ldk;                     // backward: dK / dV row stride (0: ldo)
  const int32_t* klens;        // key lengths (key padding mask); lengths = query lengths
  __nv_bfloat16* dq;           // backward: dQ rows (b*S + t); dqkv for self-attention
  __nv_bfloat16* dkv;          // backward: dK / dV rows (b*Sk + t)
  int causal;                  // GPT-2: key k visible to query q iff k <= q
  float scale;
  Drop drop;
  const int32_t* lengths;
  const __nv_bfloat16* O;      // fwd output / bwd input
  __nv_bfloat16* Oout;
  float* lse;
  const float* lse_in;
  const __nv_bfloat16* dO;
};

// Write 32 consecutive bf16 values (keys [32c, 32c+32)) of row r into a
// [128 x 128] K-major SW128 tile made of two 64-wide atoms.
MDEV void st_tile_row32(uint8_t* tile, int r, int c, const float* v) {
  const int atom = c >> 1, cb = (c & 1) * 4;
  uint8_t* base = tile + atom * (AQ * 128);
#pragma unroll
  for (int j = 0; j < 4; ++j) *(uint4*)(base + sw128(r, cb + j)) = pack8(v + 8 * j);
}

// Same, for the 16 keys [32c + 16hh, 32c + 16hh + 16).
MDEV void st_tile_row16(uint8_t* tile, int r, int c, int hh, const float* v) {
  const int atom = c >> 1, cb = (c & 1) * 4 + 2 * hh;
  uint8_t* base = tile + atom * (AQ * 128);
#pragma unroll
  for (int j = 0; j < 2; ++j) *(uint4*)(base + sw128(r, cb + j)) = pack8(v + 8 * j);
}

MDEV float4 drop4_or(const Drop& d, uint64_t e) {
  if (!d.enabled) return make_float4(1.f, 1.f, 1.f, 1.f);
  if ((e & 3) == 0) return drop_factor4(d, e >> 2);
  return make_float4(drop_factor(d, e), drop_factor(d, e + 1), drop_factor(d, e + 2), drop_factor(d, e + 3));
}

// 8 warps: warp w reads TMEM lane quarter w % 4 (rows 32(w%4)..+31) and
// handles key half w / 4 of every row: 16-key units [0, umid) or [umid, n16),
// umid = ceil(n16 / 2) (the halves differ by at most one unit).
// The two halves of a row combine their max / sum / dot partials through
// shared memory in a fixed order (half 0 + half 1), so results are
// deterministic.
constexpr int ATT = 256;
MDEV float ex2f(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// kmax = roundup(S, 32): the key range every MMA and every softmax pass covers.
// Softmax: pass 1 takes the row max, pass 2 writes the unnormalised
// P~ = exp(s - max) * dropout (bf16) and the row sum l; O = (P~ V) / l in the
// epilogue, LSE = max + log l (what the backward recomputes P from).
__global__ void __launch_bounds__(ATT, 3) k_attn_fwd_tc(const __grid_constant__ CUtensorMap tq,
                                                     const __grid_constant__ CUtensorMap tk, const AttnArgs a) {
  pdl_enter();
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* sQ = sm;
  uint8_t* sK = sm + TILE;
  uint8_t* sV = sm + 2 * TILE;
  uint8_t* sP = sm;                       // reuses Q and K (dead after S = Q K^T)
  uint64_t* bar = (uint64_t*)(sm + 3 * TILE);   // [0] tma, [1] mma S, [2] mma O
  uint32_t* tslot = (uint32_t*)(bar + 4);
  float* red = (float*)(sm + 3 * TILE + 64);     // [2][128] per-half row partials
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int hf = warp >> 2, t = 32 * (warp & 3) + lane;
  const int bh = blockIdx.x, b = bh / a.h, hd = bh % a.h;
  const int S = a.S, Sk = a.Sk, len = a.klens[b];
  // key half hf covers 16-key units [u0, u1): halves differ by at most one unit
  const int kmax = (Sk + 31) & ~31, n16 = kmax >> 4, umid = (n16 + 1) >> 1;
  const int u0 = hf ? umid : 0, u1 = hf ? n16 : umid;
  if (threadIdx.x == 0) {
    for (int i = 0; i < 3; ++i) mbar_init(&bar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tslot)), "r"(128));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;
  const int row0 = b * S, krow0 = b * Sk;
  if (threadIdx.x == 0) {
    mbar_expect_tx(&bar[0], 3 * TILE);
    tma_load_2d(&tq, &bar[0], sQ, a.qcol + hd * AD, row0);
    tma_load_2d(&tk, &bar[0], sK, a.kcol + hd * AD, krow0);
    tma_load_2d(&tk, &bar[0], sV, a.vcol + hd * AD, krow0);
    mbar_wait(&bar[0], 0);
    tc_fence_after();
    const uint32_t id = idesc_bf16(AQ, kmax, 0, 0);
    const uint32_t q0 = smem_u32(sQ), k0 = smem_u32(sK);
#pragma unroll
    for (int kk = 0; kk < AD / 16; ++kk)
      mma_bf16(tmem, make_desc(q0 + 32 * kk, 16, 1024), make_desc(k0 + 32 * kk, 16, 1024), id, kk > 0);
    mma_commit(&bar[1]);
  }
  mbar_wait(&bar[1], 0);
  __syncwarp();
  tc_fence_after();
  // ---- softmax of row t over keys [0, kl), kl = len (or min(len, t+1) causal) ----
  const uint32_t trow = tmem + ((uint32_t)(32 * (warp & 3)) << 16);
  const int kl = a.causal ? min(len, t + 1) : len;
  float mx = -INFINITY;
  for (int u = u0; u < u1; ++u) {
    float v[16];
    tmem_ld16(trow + 16 * u, v);                // every lane loads (.sync.aligned)
    if (16 * u < kl) {
#pragma unroll
      for (int i = 0; i < 16; ++i)
        if (16 * u + i < kl) mx = fmaxf(mx, v[i]);
    }
  }
  red[hf * 128 + t] = mx;
  __syncthreads();
  const float sl2 = a.scale * 1.4426950408889634f;               // scale * log2(e)
  const float mrow = fmaxf(red[t], red[128 + t]) * sl2;          // row max of s * scale * log2(e)
  const uint64_t ebase = (((uint64_t)b * a.h + hd) * S + (uint64_t)t) * Sk;
  // The S MMA has completed (bar[1]), so Q and K are dead: each thread writes its
  // P~ row straight into their space.
  float l = 0.f;
  for (int u = u0; u < u1; ++u) {
    {
      const int c = u >> 1, hh = u & 1;
      float v[16];
      tmem_ld16(trow + 16 * u, v);
      const int kb = 16 * u;
      if (kb < kl && t < S) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int k = kb + 4 * j;
          const float4 f = (k < kl) ? drop4_or(a.drop, ebase + k) : make_float4(0.f, 0.f, 0.f, 0.f);
          const float ff[4] = {f.x, f.y, f.z, f.w};
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const float p = (k + i < kl) ? ex2f(fmaf(v[4 * j + i], sl2, -mrow)) : 0.f;
            l += p;
            v[4 * j + i] = p * ff[i];
          }
        }
      } else {
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] = 0.f;
      }
      st_tile_row16(sP, t, c, hh, v);
    }
  }
  __syncthreads();                              // red[] (max) reads done before reuse
  red[hf * 128 + t] = l;
  fence_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const float lsum = red[t] + red[128 + t];
  if (threadIdx.x == 0) {
    const uint32_t id = idesc_bf16(AQ, AD, 0, 1);
    const uint32_t p0 = smem_u32(sP), v0 = smem_u32(sV);
    for (int kk = 0; kk < kmax / 16; ++kk) {
      const uint64_t da = make_desc(p0 + (kk >> 2) * (AQ * 128) + 32 * (kk & 3), 16, 1024);
      const uint64_t db = make_desc(v0 + 2048 * kk, 16384, 1024);
      mma_bf16(tmem, da, db, id, kk > 0);                   // O over S's dead columns
    }
    mma_commit(&bar[2]);
  }
  mbar_wait(&bar[2], 0);
  __syncwarp();
  tc_fence_after();
  {  // tcgen05.ld is .sync.aligned: every lane loads, only rows t < S store; half hf stores dims 32hf..
    __nv_bfloat16* orow = a.Oout + ((int64_t)row0 + t) * a.H + hd * AD;
    const float inv = lsum > 0.f ? 1.0f / lsum : 0.f;
    float v[32];
    tmem_ld32(trow + 32 * hf, v);
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] *= inv;
    if (t < S) st_bf16x32(orow + 32 * hf, v);
    if (t < S && hf == 0) a.lse[((int64_t)b * a.h + hd) * S + t] = (mrow + __log2f(lsum)) * 0.69314718055994531f;
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(128));
  }
}

template <bool DC>   // DC: D = sum_k P~ dP~ (cross-attention); else rowsum(dO * O)
__global__ void __launch_bounds__(ATT, 2) k_attn_bwd_tc(const __grid_constant__ CUtensorMap tq,
                                                     const __grid_constant__ CUtensorMap tk,
                                                     const __grid_constant__ CUtensorMap tdo, const AttnArgs a) {
  pdl_enter();
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* sQ = sm;
  uint8_t* sK = sm + TILE;
  uint8_t* sdO = sm + 2 * TILE;
  uint8_t* sV = sm + 3 * TILE;
  uint8_t* sP = sV;                        // P~ (32 KB) reuses V (dead after dP) + 16 KB
  uint8_t* sdS = sm + 5 * TILE;
  uint64_t* bar = (uint64_t*)(sdS + PT);  // [0] tma, [1] mma S/dP, [2] mma grads
  uint32_t* tslot = (uint32_t*)(bar + 4);
  float* red = (float*)sdS;               // [2][128] per-half partial of D (dS is written only after D is read)
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int hf = warp >> 2, t = 32 * (warp & 3) + lane;
  const int bh = blockIdx.x, b = bh / a.h, hd = bh % a.h;
  const int S = a.S, Sk = a.Sk, len = a.lengths[b], klen = a.klens[b];
  const int kmax = (Sk + 31) & ~31, n16 = kmax >> 4, umid = (n16 + 1) >> 1;
  const int qmax = (S + 31) & ~31;                 // contraction range of dV, dK (query rows)
  const int u0 = hf ? umid : 0, u1 = hf ? n16 : umid;   // this half's 16-key units (<= 4)
  if (threadIdx.x == 0) {
    for (int i = 0; i < 3; ++i) mbar_init(&bar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tslot)), "r"(256));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;
  const int row0 = b * S, krow0 = b * Sk;
  if (threadIdx.x == 0) {
    mbar_expect_tx(&bar[0], 4 * TILE);
    tma_load_2d(&tq, &bar[0], sQ, a.qcol + hd * AD, row0);
    tma_load_2d(&tk, &bar[0], sK, a.kcol + hd * AD, krow0);
    tma_load_2d(&tk, &bar[0], sV, a.vcol + hd * AD, krow0);
    tma_load_2d(&tdo, &bar[0], sdO, hd * AD, row0);
    mbar_wait(&bar[0], 0);
    tc_fence_after();
    const uint32_t id = idesc_bf16(AQ, kmax, 0, 0);
    const uint32_t q0 = smem_u32(sQ), k0 = smem_u32(sK), v0 = smem_u32(sV), o0 = smem_u32(sdO);
#pragma unroll
    for (int kk = 0; kk < AD / 16; ++kk)
      mma_bf16(tmem, make_desc(q0 + 32 * kk, 16, 1024), make_desc(k0 + 32 * kk, 16, 1024), id, kk > 0);
#pragma unroll
    for (int kk = 0; kk < AD / 16; ++kk)
      mma_bf16(tmem + 128, make_desc(o0 + 32 * kk, 16, 1024), make_desc(v0 + 32 * kk, 16, 1024), id, kk > 0);
    mma_commit(&bar[1]);
  }
  // D_t = sum_k P~_tk dP~_tk over this row's keys, in fp32 from the same P~ and
  // dP~ = dO V^T that dS uses (exactly rowsum(dO * O) in exact arithmetic, but
  // consistent with dP~ under bf16 storage of O, so dS sums to ~0 per row:
  // near-uniform attention rows -- e.g. cross-attention -- keep their relative
  // accuracy).  Pass 1 over the TMEM row: P~, the dropout keep bits (kept in two
  // registers for pass 2), the D partial of this key half; D = half 0 + half 1.
  float Lt = 0.f, Dh = 0.f;
  if (t < len) Lt = a.lse_in[((int64_t)b * a.h + hd) * S + t];
  if (!DC && t < len) {
    // self-attention: D = rowsum(dO * O), half hf sums dims [32hf, 32hf+32); the
    // global reads overlap the MMAs
    const __nv_bfloat16* orow = a.O + ((int64_t)row0 + t) * a.H + hd * AD + 32 * hf;
    const __nv_bfloat16* drow = a.dO + ((int64_t)row0 + t) * a.H + hd * AD + 32 * hf;
    float ov[32], dv[32];
    ld_bf16x32(orow, ov);
    ld_bf16x32(drow, dv);
#pragma unroll
    for (int i = 0; i < 32; ++i) Dh += ov[i] * dv[i];
  }
  mbar_wait(&bar[1], 0);
  __syncwarp();
  tc_fence_after();
  const uint32_t trow = tmem + ((uint32_t)(32 * (warp & 3)) << 16);
  const uint64_t ebase = (((uint64_t)b * a.h + hd) * S + (uint64_t)t) * Sk;
  const int kl = a.causal ? min(klen, t + 1) : klen;
  const float sl2 = a.scale * 1.4426950408889634f, Ll2 = Lt * 1.4426950408889634f;
  const float keepf = a.drop.enabled ? a.drop.scale : 1.0f;
  uint32_t kb0 = 0u, kb1 = 0u;             // keep bits of units u0, u0 + 1 (kb0) and u0 + 2, u0 + 3 (kb1)
  for (int u = u0; u < u1 && DC; ++u) {
    const int hh = (u - u0) & 1;
    const bool lo = u - u0 < 2;
    float sv[16], dp[16];
    tmem_ld16(trow + 16 * u, sv);
    tmem_ld16(trow + 128 + 16 * u, dp);
    const int kb = 16 * u;
    if (t < len && kb < kl) {
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int k = kb + 4 * j;
        const float4 f = (k < kl) ? drop4_or(a.drop, ebase + k) : make_float4(0.f, 0.f, 0.f, 0.f);
        const float ff[4] = {f.x, f.y, f.z, f.w};
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int kk = k + i;
          const float p = (kk < kl) ? ex2f(fmaf(sv[4 * j + i], sl2, -Ll2)) : 0.f;
          Dh = fmaf(p * ff[i], dp[4 * j + i], Dh);
          if (ff[i] != 0.f) {
            if (lo) kb0 |= 1u << (16 * hh + 4 * j + i);
            else kb1 |= 1u << (16 * hh + 4 * j + i);
          }
        }
      }
    }
  }
  red[hf * 128 + t] = Dh;
  __syncthreads();                        // red[] complete; every thread is past the MMAs (V dead)
  const float Dt = red[t] + red[128 + t];
  __syncthreads();                        // every D read before dS overwrites red[]
  for (int u = u0; u < u1; ++u) {
    const int c = u >> 1, hh = u & 1;            // smem tile chunk of the unit
    const int bh = (u - u0) & 1;                 // bit half of the unit's keep word
    const bool lo = u - u0 < 2;
    float sv[16], dp[16];
    tmem_ld16(trow + 16 * u, sv);
    tmem_ld16(trow + 128 + 16 * u, dp);
    const int kb = 16 * u;
    const bool live = t < len && kb < kl;        // padded / foreign query rows contribute 0
    if (live) {
      float fself[16];
      if (!DC) {                                 // self-attention: the mask from Philox here
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int k = kb + 4 * j;
          const float4 f = (k < kl) ? drop4_or(a.drop, ebase + k) : make_float4(0.f, 0.f, 0.f, 0.f);
          fself[4 * j] = f.x; fself[4 * j + 1] = f.y; fself[4 * j + 2] = f.z; fself[4 * j + 3] = f.w;
        }
      }
#pragma unroll
      for (int q = 0; q < 16; ++q) {
        const int kk = kb + q;
        const float p = (kk < kl) ? ex2f(fmaf(sv[q], sl2, -Ll2)) : 0.f;
        const float fq = !DC ? fself[q] : ((((lo ? kb0 : kb1) >> (16 * bh + q)) & 1u) ? keepf : 0.f);
        sv[q] = p * fq;                                            // P~
        dp[q] = p * (dp[q] * fq - Dt) * a.scale;                   // dS (scale folded)
      }
    } else {
#pragma unroll
      for (int i = 0; i < 16; ++i) { sv[i] = 0.f; dp[i] = 0.f; }
    }
    st_tile_row16(sP, t, c, hh, sv);
    st_tile_row16(sdS, t, c, hh, dp);
  }
  fence_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (threadIdx.x == 0) {
    const uint32_t id_t = idesc_bf16(AQ, AD, 1, 1);   // A MN-major (keys), B MN-major (d)
    const uint32_t id_q = idesc_bf16(AQ, AD, 0, 1);   // A K-major (queries), B MN-major (d)
    const uint32_t p0 = smem_u32(sP), s0 = smem_u32(sdS);
    const uint32_t q0 = smem_u32(sQ), k0 = smem_u32(sK), o0 = smem_u32(sdO);
    for (int kk = 0; kk < max(kmax, qmax) / 16; ++kk) {   // contraction over queries (dV, dK) / keys (dQ)
      if (kk < qmax / 16) {
        const uint64_t at_p = make_desc(p0 + 2048 * kk, 16384, 1024);
        const uint64_t at_s = make_desc(s0 + 2048 * kk, 16384, 1024);
        const uint64_t bq_do = make_desc(o0 + 2048 * kk, 16384, 1024);
        const uint64_t bq_q = make_desc(q0 + 2048 * kk, 16384, 1024);
        mma_bf16(tmem + 0, at_p, bq_do, id_t, kk > 0);        // dV = P~^T dO
        mma_bf16(tmem + 64, at_s, bq_q, id_t, kk > 0);        // dK = dS^T Q
      }
      if (kk < kmax / 16) {
        const uint64_t ak_s = make_desc(s0 + (kk >> 2) * (AQ * 128) + 32 * (kk & 3), 16, 1024);
        const uint64_t bk_k = make_desc(k0 + 2048 * kk, 16384, 1024);
        mma_bf16(tmem + 128, ak_s, bk_k, id_q, kk > 0);       // dQ = dS K
      }
    }
    mma_commit(&bar[2]);
  }
  mbar_wait(&bar[2], 0);
  __syncwarp();
  tc_fence_after();
  {  // every lane loads (.sync.aligned); query rows t < S store dQ, key rows t < Sk store dK, dV;
     // half hf stores dims [32hf, 32hf+32)
    __nv_bfloat16* qrow = a.dq + ((int64_t)row0 + t) * a.ldo + a.ocq + hd * AD + 32 * hf;
    __nv_bfloat16* krow = a.dkv + ((int64_t)krow0 + t) * (a.ldk ? a.ldk : a.ldo) + hd * AD + 32 * hf;
    float v[32];
    tmem_ld32(trow + 128 + 32 * hf, v);
    if (t < S) st_bf16x32(qrow, v);                          // dQ
    tmem_ld32(trow + 64 + 32 * hf, v);
    if (t < Sk) st_bf16x32(krow + a.ock, v);                 // dK
    tmem_ld32(trow + 32 * hf, v);
    if (t < Sk) st_bf16x32(krow + a.ocv, v);                 // dV
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(256));
  }
}

// ------------------------------------------------------------------ host --
bool tc_map_bf16(CUtensorMap* out, const void* ptr, uint64_t inner, uint64_t outer, uint64_t stride_elems,
                 uint32_t box_inner, uint32_t box_outer);   // kernels_gemm_tc.cu

constexpr int FWD_SMEM = 3 * TILE + 64 + 1024 + 128;      // P~ reuses Q/K; + barriers, row partials
constexpr int BWD_SMEM = 5 * TILE + PT + 128;             // P~ reuses V; D partials live in dS (2 CTAs / SM)

bool attn_tc_ok(int S, int H, int h) { return S <= AQ && H / h == AD && H % 64 == 0; }

bool attn_fwd_tc(const void* qkv, const int32_t* lengths, void* O, float* lse, int B, int S, int H, int h,
                 Drop drop, cudaStream_t st, bool causal) {
  if (!attn_tc_ok(S, H, h)) return false;
  CUtensorMap tq;
  if (!tc_map_bf16(&tq, qkv, 3ull * H, (uint64_t)B * S, 3ull * H, 64, AQ)) return false;
  static std::once_flag once;
  std::call_once(once, [] { cudaFuncSetAttribute(k_attn_fwd_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, FWD_SMEM); });
  AttnArgs a{};
  a.S = S; a.Sk = S; a.H = H; a.h = h; a.B = B;
  a.qcol = 0; a.kcol = H; a.vcol = 2 * H;
  a.scale = 1.0f / sqrtf((float)AD);
  a.drop = drop; a.lengths = lengths; a.klens = lengths; a.Oout = (__nv_bfloat16*)O; a.lse = lse; a.causal = causal;
  launch_k(k_attn_fwd_tc, B * h, ATT, FWD_SMEM, st, tq, tq, a);
  return true;
}

bool attn_bwd_tc(const void* qkv, const void* O, const void* dO, const float* lse, const int32_t* lengths,
                 void* dqkv, int B, int S, int H, int h, Drop drop, cudaStream_t st, bool causal) {
  if (!attn_tc_ok(S, H, h)) return false;
  CUtensorMap tq, tdo;
  if (!tc_map_bf16(&tq, qkv, 3ull * H, (uint64_t)B * S, 3ull * H, 64, AQ)) return false;
  if (!tc_map_bf16(&tdo, dO, (uint64_t)H, (uint64_t)B * S, (uint64_t)H, 64, AQ)) return false;
  static std::once_flag once;
  std::call_once(once, [] {
    cudaFuncSetAttribute(k_attn_bwd_tc<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, BWD_SMEM);
  });
  AttnArgs a{};
  a.S = S; a.Sk = S; a.H = H; a.h = h; a.B = B;
  a.qcol = 0; a.kcol = H; a.vcol = 2 * H;
  a.ldo = 3 * H; a.ocq = 0; a.ock = H; a.ocv = 2 * H;
  a.scale = 1.0f / sqrtf((float)AD);
  a.drop = drop; a.lengths = lengths; a.klens = lengths; a.O = (const __nv_bfloat16*)O; a.dO = (const __nv_bfloat16*)dO;
  a.lse_in = lse; a.dq = (__nv_bfloat16*)dqkv; a.dkv = (__nv_bfloat16*)dqkv; a.causal = causal;
  launch_k(k_attn_bwd_tc<false>, B * h, ATT, BWD_SMEM, st, tq, tq, tdo, a);
  return true;
}

// Cross-attention (encoder-decoder): queries q [B*Sq, H], keys and
// values kv [B*Sk, 2H] (k | v), key padding by klens, no causal mask; both
// lengths <= 128.  Dropout element ((b*h + head)*Sq + q)*Sk + k.
bool attn_cross_ok(int Sq, int Sk, int H, int h) { return Sq <= AQ && Sk <= AQ && H / h == AD && H % 64 == 0; }

bool attn_cross_fwd_tc(const void* q, const void* kv, const int32_t* qlens, const int32_t* klens, void* O, float* lse,
                       int B, int Sq, int Sk, int H, int h, Drop drop, cudaStream_t st) {
  if (!attn_cross_ok(Sq, Sk, H, h))        // a length above 128: the tiled kernels
    return attn_cross_fwd_tcl(q, kv, qlens, klens, O, lse, B, Sq, Sk, H, h, drop, st);
  CUtensorMap tq, tk;
  if (!tc_map_bf16(&tq, q, (uint64_t)H, (uint64_t)B * Sq, (uint64_t)H, 64, AQ)) return false;
  if (!tc_map_bf16(&tk, kv, 2ull * H, (uint64_t)B * Sk, 2ull * H, 64, AQ)) return false;
  static std::once_flag once;
  std::call_once(once, [] { cudaFuncSetAttribute(k_attn_fwd_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, FWD_SMEM); });
  AttnArgs a{};
  a.S = Sq; a.Sk = Sk; a.H = H; a.h = h; a.B = B;
  a.qcol = 0; a.kcol = 0; a.vcol = H;
  a.scale = 1.0f / sqrtf((float)AD);
  a.drop = drop; a.lengths = qlens; a.klens = klens; a.Oout = (__nv_bfloat16*)O; a.lse = lse; a.causal = 0;
  launch_k(k_attn_fwd_tc, B * h, ATT, FWD_SMEM, st, tq, tk, a);
  return true;
}

bool attn_cross_bwd_tc(const void* q, const void* kv, const void* O, const void* dO, const float* lse,
                       const int32_t* qlens, const int32_t* klens, float* Dbuf, void* dq, void* dkv, int B, int Sq,
                       int Sk, int H, int h, Drop drop, cudaStream_t st) {
  if (!attn_cross_ok(Sq, Sk, H, h))
    return attn_cross_bwd_tcl(q, kv, O, dO, lse, qlens, klens, Dbuf, dq, dkv, B, Sq, Sk, H, h, drop, st);
  CUtensorMap tq, tk, tdo;
  if (!tc_map_bf16(&tq, q, (uint64_t)H, (uint64_t)B * Sq, (uint64_t)H, 64, AQ)) return false;
  if (!tc_map_bf16(&tk, kv, 2ull * H, (uint64_t)B * Sk, 2ull * H, 64, AQ)) return false;
  if (!tc_map_bf16(&tdo, dO, (uint64_t)H, (uint64_t)B * Sq, (uint64_t)H, 64, AQ)) return false;
  static std::once_flag once;
  std::call_once(once, [] {
    cudaFuncSetAttribute(k_attn_bwd_tc<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, BWD_SMEM);
  });
  AttnArgs a{};
  a.S = Sq; a.Sk = Sk; a.H = H; a.h = h; a.B = B;
  a.qcol = 0; a.kcol = 0; a.vcol = H;
  a.scale = 1.0f / sqrtf((float)AD);
  a.drop = drop; a.lengths = qlens; a.klens = klens; a.O = (const __nv_bfloat16*)O; a.dO = (const __nv_bfloat16*)dO;
  a.lse_in = lse; a.causal = 0;
  // dQ [B*Sq, H] and dKV [B*Sk, 2H] have different row strides: two output
  // pointers, one stride each (ldo for dQ rows, 2H for dK / dV rows)
  a.dq = (__nv_bfloat16*)dq; a.dkv = (__nv_bfloat16*)dkv;
  a.ldo = H; a.ocq = 0; a.ock = 0; a.ocv = H;
  a.ldk = 2 * H;
  launch_k(k_attn_bwd_tc<true>, B * h, ATT, BWD_SMEM, st, tq, tk, tdo, a);
  return true;
}

}  // namespace mimose
