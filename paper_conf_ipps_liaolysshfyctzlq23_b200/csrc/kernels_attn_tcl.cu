// Attention for long sequences (128 < S <= 1024) on the 5th-gen tensor cores,
// head dim 64: the S <= 128 kernels of kernels_attn_tc.cu tiled over 128-key
// blocks.  PAPER.md P:160 / Fig. 8: S = Q K^T -> scale -> softmax -> x V; the
// S x S tensors are never stored (flash-style, DESIGN "Memory model").
//
// One CTA (8 warps) per (128-row tile, sequence b, head h).  Warp w reads TMEM
// lane quarter w % 4 (tile rows 32(w%4)..+31) and owns the 64-column half w / 4
// of each 128-column score tile.  Per-half partials (row max / sum, D) combine
// through shared memory in a fixed order, so every result is deterministic.
//
// forward  (query tile): pass 1 streams K tiles, S_j = Q K_j^T (TMEM), and
//          takes the exact row max / sum; pass 2 recomputes S_j, writes the
//          normalised P~_j = exp(S_j - LSE) * dropout (bf16, swizzled smem) and
//          accumulates O += P~_j V_j in TMEM.  O (bf16) and LSE (fp32) out.
// backward (no atomics): dQ kernel per query tile: D = rowsum(dO * O) (also
//          stored for the dK/dV kernel), per key tile S_j, dP_j = dO V_j^T ->
//          dS_j -> dQ += dS_j K_j.  dK/dV kernel per key tile: per query tile
//          S_i = Q_i K^T, dP_i = dO_i V^T -> P~_i, dS_i -> dV += P~_i^T dO_i,
//          dK += dS_i^T Q_i (the smem tiles read as MN-major operands).
// Dropout element e = ((b*h + head)*S + q)*S + k, site (KIND_ATTN_PROBS,
// layer): the same Philox stream as the SIMT and S <= 128 kernels.
#include <cuda.h>

#include <mutex>

#include "kernels.h"
#include "tc_common.cuh"

namespace mimose {

namespace {

constexpr int LQ = 128;                  // rows of a tile (queries or keys)
constexpr int LD = 64;                   // head dim
constexpr int LT = LQ * LD * 2;          // 16 KB: [128 x 64] bf16 SW128 tile
constexpr int LPT = LQ * LQ * 2;         // 32 KB: [128 x 128] bf16 tile (2 atoms)
constexpr int LTH = 256;                 // 8 warps

struct LArgs {
  int S, H, h, B;              // S: query rows per sequence
  int Sk;                      // key rows per sequence (== S for self-attention)
  int qcol, kcol, vcol;        // column bases of Q (tq) and K, V (tk)
  const int32_t* klens;        // key lengths; lengths = query lengths
  __nv_bfloat16* dq;           // dQ rows b*S + q (row stride ldq, column base ocq)
  __nv_bfloat16* dkv;          // dK / dV rows b*Sk + k (row stride ldk, column bases ock / ocv)
  int ldq, ocq, ldk, ock, ocv;
  int causal;
  float scale;
  Drop drop;
  const int32_t* lengths;
  const __nv_bfloat16* O;
  __nv_bfloat16* Oout;
  float* lse;
  const float* lse_in;
  float* Dbuf;
  const __nv_bfloat16* dO;
};

MDEV float ex2a(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
MDEV float4 drop4l(const Drop& d, uint64_t e) {   // e % 4 == 0
  if (!d.enabled) return make_float4(1.f, 1.f, 1.f, 1.f);
  return drop_factor4(d, e >> 2);
}
// 16 keys [16c, 16c + 16) (c = 0..7) of row r of a [128 x 128] K-major SW128 tile (two 64-key atoms).
MDEV void st_row16(uint8_t* tile, int r, int c, const float* v) {
  uint8_t* base = tile + (c >> 2) * (LQ * 128);
  const int cb = (c & 3) * 2;
#pragma unroll
  for (int j = 0; j < 2; ++j) *(uint4*)(base + sw128(r, cb + j)) = pack8(v + 8 * j);
}
MDEV void bar_sync_all() {
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
}
MDEV void tmem_alloc(uint32_t* slot, uint32_t cols) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(slot)), "r"(cols));
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
}
MDEV void tmem_free(uint32_t tmem, uint32_t cols) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(cols));
}
// C[128 x 128] (TMEM) = A[128 x 64] B[128 x 64]^T, both K-major [rows x 64] tiles.
MDEV void mma_nt64(uint32_t d, uint32_t a, uint32_t b) {
  const uint32_t id = idesc_bf16(LQ, LQ, 0, 0);
#pragma unroll
  for (int kk = 0; kk < LD / 16; ++kk)
    mma_bf16(d, make_desc(a + 32 * kk, 16, 1024), make_desc(b + 32 * kk, 16, 1024), id, kk > 0);
}
// C[128 x 64] (+)= P[128 x 128] V[128 x 64]: P K-major (rows x keys), V rows = keys (MN-major B).
MDEV void mma_pv(uint32_t d, uint32_t p, uint32_t v, bool acc) {
  const uint32_t id = idesc_bf16(LQ, LD, 0, 1);
  for (int kk = 0; kk < LQ / 16; ++kk)
    mma_bf16(d, make_desc(p + (kk >> 2) * (LQ * 128) + 32 * (kk & 3), 16, 1024), make_desc(v + 2048 * kk, 16384, 1024),
             id, (acc || kk > 0) ? 1u : 0u);
}
// C[128 x 64] (+)= P^T[128 x 128] X[128 x 64]: P stored rows = contraction (MN-major A), X MN-major B.
MDEV void mma_ptx(uint32_t d, uint32_t p, uint32_t x, bool acc) {
  const uint32_t id = idesc_bf16(LQ, LD, 1, 1);
  for (int kk = 0; kk < LQ / 16; ++kk)
    mma_bf16(d, make_desc(p + 2048 * kk, 16384, 1024), make_desc(x + 2048 * kk, 16384, 1024), id,
             (acc || kk > 0) ? 1u : 0u);
}

// ---------------------------------------------------------------- forward --
constexpr int LF_SMEM = 3 * LT + LPT + 1024 + 4096;   // Q, K, V, P~ + barriers / row partials + align slack

__global__ void __launch_bounds__(LTH, 2) k_attn_fwd_tcl(const __grid_constant__ CUtensorMap tq,
                                                       const __grid_constant__ CUtensorMap tk, const LArgs a) {
  pdl_enter();
  extern __shared__ uint8_t smraw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)smraw + 1023) & ~(uintptr_t)1023);
  uint8_t* sQ = sm;
  uint8_t* sK = sm + LT;
  uint8_t* sV = sm + 2 * LT;
  uint8_t* sP = sm + 3 * LT;
  // [0] Q, [1] K buffer sK, [2] MMA S, [3] MMA O, [4] K buffer sV (pass 1), [5] V (pass 2)
  uint64_t* bar = (uint64_t*)(sP + LPT);
  uint32_t* tslot = (uint32_t*)(bar + 6);
  float* red = (float*)(bar + 8);               // [2][128] x 2
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int hf = warp >> 2, t = 32 * (warp & 3) + lane;
  const int q0 = blockIdx.x * LQ, bh = blockIdx.y, b = bh / a.h, hd = bh % a.h;
  const int S = a.S, Sk = a.Sk, len = a.klens[b];
  const int q = q0 + t;
  const int kl = a.causal ? min(len, q + 1) : len;          // keys visible to row q
  const int kl_tile = a.causal ? min(len, q0 + LQ) : len;
  const int nkt = (kl_tile + LQ - 1) / LQ;
  if (threadIdx.x == 0) {
    for (int i = 0; i < 6; ++i) mbar_init(&bar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) tmem_alloc(tslot, 256);
  bar_sync_all();
  const uint32_t tmem = *tslot;                 // S: cols 0..127, O: cols 128..191
  const uint32_t trow = tmem + ((uint32_t)(32 * (warp & 3)) << 16);
  const int row0 = b * S, krow0 = b * Sk;
  const float sl2 = a.scale * 1.4426950408889634f;
  // TMA prefetch (thread 0 only; its phase bits): pass 1 double-buffers K in sK / sV
  // (V is not needed yet); pass 2 reloads K as soon as S = Q K_j is done and V as
  // soon as O += P~ V_j is done, so each tile's loads overlap the previous tile.
  uint32_t ph_k0 = 0, ph_k1 = 0, ph_v = 0;
  if (threadIdx.x == 0 && nkt > 0) {
    mbar_expect_tx(&bar[0], LT);
    tma_load_2d(&tq, &bar[0], sQ, a.qcol + hd * LD, row0 + q0);
    mbar_expect_tx(&bar[1], LT);
    tma_load_2d(&tk, &bar[1], sK, a.kcol + hd * LD, krow0);
  }
  int ph_s = 0, ph_o = 0;
  // ---- pass 1: exact row max (the sum is taken in pass 2 from the same exponentials) ----
  float m = -INFINITY;
  for (int j = 0; j < nkt; ++j) {
    if (threadIdx.x == 0) {
      const int bf = j & 1;
      if (j + 1 < nkt) {                        // buffer !bf held K_{j-1}: its MMA is done
        mbar_expect_tx(&bar[bf ? 1 : 4], LT);
        tma_load_2d(&tk, &bar[bf ? 1 : 4], bf ? sK : sV, a.kcol + hd * LD, krow0 + (j + 1) * LQ);
      }
      if (j == 0) mbar_wait(&bar[0], 0);
      if (bf) { mbar_wait(&bar[4], ph_k1); ph_k1 ^= 1; }
      else { mbar_wait(&bar[1], ph_k0); ph_k0 ^= 1; }
      tc_fence_after();
      mma_nt64(tmem, smem_u32(sQ), smem_u32(bf ? sV : sK));
      mma_commit(&bar[2]);
    }
    mbar_wait(&bar[2], ph_s);
    ph_s ^= 1;
    __syncwarp();
    tc_fence_after();
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      float v[16];
      tmem_ld16(trow + 64 * hf + 16 * c, v);
      const int kb = j * LQ + 64 * hf + 16 * c;
      if (kb < kl) {
#pragma unroll
        for (int i = 0; i < 16; ++i)
          if (kb + i < kl) m = fmaxf(m, v[i]);
      }
    }
    bar_sync_all();                             // S read before the next MMA overwrites it
  }
  red[hf * 128 + t] = m;
  __syncthreads();
  const float M = fmaxf(red[t], red[128 + t]) * sl2;   // log2-domain row max of s * scale
  const uint64_t ebase = (((uint64_t)b * a.h + hd) * S + (uint64_t)q) * Sk;
  float l = 0.f;                                // this half's sum of exp(s - max), fp32, before dropout
  // ---- pass 2: P~ = exp(S - max) * dropout (unnormalised), O += P~ V; O / l in the epilogue ----
  if (threadIdx.x == 0 && nkt > 0) {            // every pass-1 MMA is done (bar[2] waited)
    mbar_expect_tx(&bar[1], LT);
    tma_load_2d(&tk, &bar[1], sK, a.kcol + hd * LD, krow0);
    mbar_expect_tx(&bar[5], LT);
    tma_load_2d(&tk, &bar[5], sV, a.vcol + hd * LD, krow0);
  }
  for (int j = 0; j < nkt; ++j) {
    if (threadIdx.x == 0) {
      mbar_wait(&bar[1], ph_k0);
      ph_k0 ^= 1;
      tc_fence_after();
      mma_nt64(tmem, smem_u32(sQ), smem_u32(sK));
      mma_commit(&bar[2]);
    }
    mbar_wait(&bar[2], ph_s);
    ph_s ^= 1;
    __syncwarp();
    tc_fence_after();
    if (threadIdx.x == 0 && j + 1 < nkt) {      // sK is free once S = Q K_j is in TMEM
      mbar_expect_tx(&bar[1], LT);
      tma_load_2d(&tk, &bar[1], sK, a.kcol + hd * LD, krow0 + (j + 1) * LQ);
    }
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      float v[16];
      tmem_ld16(trow + 64 * hf + 16 * c, v);
      const int kb = j * LQ + 64 * hf + 16 * c;
      if (kb < kl && q < S) {
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          const int k = kb + 4 * g;
          const float4 f = k < kl ? drop4l(a.drop, ebase + k) : make_float4(0.f, 0.f, 0.f, 0.f);
          const float ff[4] = {f.x, f.y, f.z, f.w};
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const float p = (k + i < kl) ? ex2a(fmaf(v[4 * g + i], sl2, -M)) : 0.f;
            l += p;
            v[4 * g + i] = p * ff[i];
          }
        }
      } else {
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] = 0.f;
      }
      st_row16(sP, t, 4 * hf + c, v);
    }
    fence_async_smem();
    bar_sync_all();
    if (threadIdx.x == 0) {
      mbar_wait(&bar[5], ph_v);
      ph_v ^= 1;
      tc_fence_after();
      mma_pv(tmem + 128, smem_u32(sP), smem_u32(sV), j > 0);
      mma_commit(&bar[3]);
    }
    mbar_wait(&bar[3], ph_o);                   // P~, V and S free for the next tile
    ph_o ^= 1;
    __syncwarp();
    tc_fence_after();
    if (threadIdx.x == 0 && j + 1 < nkt) {
      mbar_expect_tx(&bar[5], LT);
      tma_load_2d(&tk, &bar[5], sV, a.vcol + hd * LD, krow0 + (j + 1) * LQ);
    }
  }
  red[256 + hf * 128 + t] = l;                 // row sum: half 0 + half 1, fixed order
  __syncthreads();
  const float lt = red[256 + t] + red[384 + t];
  const float L2 = M + __log2f(lt);             // log2-domain LSE of s * scale (what the backward reads)
  {  // epilogue: half hf stores dims [32hf, 32hf + 32) of row q, O = (P~ V) / l
    float v[32];
    tmem_ld32(trow + 128 + 32 * hf, v);
    const float inv = (nkt > 0 && lt > 0.f) ? 1.0f / lt : 0.f;
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] *= inv;
    if (q < S) {
      st_bf16x32(a.Oout + ((int64_t)row0 + q) * a.H + hd * LD + 32 * hf, v);
      if (hf == 0) a.lse[((int64_t)b * a.h + hd) * S + q] = L2 * 0.69314718055994531f;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    tmem_free(tmem, 256);
  }
}

// ------------------------------------------------------------ backward dQ --
constexpr int LQ_SMEM = 6 * LT + LPT + 1024 + 2048;   // Q, dO, K[2], V[2], dS

// DC (cross-attention): D = sum_k P~ dP~ over every key tile, in fp32 from the
// same P~ and dP~ = dO V^T that dS uses (consistent under bf16 storage of O;
// kernels_attn_tc.cu), by a first pass over the key tiles; else rowsum(dO * O).
template <bool DC>
__global__ void __launch_bounds__(LTH, 1) k_attn_bwd_dq_tcl(const __grid_constant__ CUtensorMap tq,
                                                            const __grid_constant__ CUtensorMap tk,
                                                            const __grid_constant__ CUtensorMap tdo, const LArgs a) {
  pdl_enter();
  extern __shared__ uint8_t smraw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)smraw + 1023) & ~(uintptr_t)1023);
  uint8_t* sQ = sm;
  uint8_t* sdO = sm + LT;
  // K_j / V_j in buffer j & 1 (K at 2LT + 2LT*buf, V right after): tile j+1 loads
  // while tile j is processed
  auto sKb = [&](int bf) { return sm + 2 * LT + 2 * LT * bf; };
  auto sVb = [&](int bf) { return sm + 3 * LT + 2 * LT * bf; };
  uint8_t* sdS = sm + 6 * LT;
  uint64_t* bar = (uint64_t*)(sdS + LPT);       // [0] Q/dO, [1] K/V buf 0, [2] MMA S/dP, [3] MMA dQ, [4] K/V buf 1
  uint32_t* tslot = (uint32_t*)(bar + 6);
  float* red = (float*)(bar + 8);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int hf = warp >> 2, t = 32 * (warp & 3) + lane;
  const int q0 = blockIdx.x * LQ, bh = blockIdx.y, b = bh / a.h, hd = bh % a.h;
  const int S = a.S, Sk = a.Sk, len = a.lengths[b], klen = a.klens[b];
  const int q = q0 + t;
  const bool live = q < len;                    // padded query rows carry zero gradient (A26)
  const int kl = a.causal ? min(klen, q + 1) : klen;
  const int kl_tile = a.causal ? min(klen, q0 + LQ) : klen;
  const int nkt = q0 < len ? (kl_tile + LQ - 1) / LQ : 0;
  if (threadIdx.x == 0) {
    for (int i = 0; i < 5; ++i) mbar_init(&bar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) tmem_alloc(tslot, 512);
  bar_sync_all();
  const uint32_t tmem = *tslot;                 // S 0..127, dP 128..255, dQ 256..319
  const uint32_t trow = tmem + ((uint32_t)(32 * (warp & 3)) << 16);
  const int row0 = b * S, krow0 = b * Sk;
  auto load_kv = [&](int j, int bf) {           // thread 0
    mbar_expect_tx(&bar[bf ? 4 : 1], 2 * LT);
    tma_load_2d(&tk, &bar[bf ? 4 : 1], sKb(bf), a.kcol + hd * LD, krow0 + j * LQ);
    tma_load_2d(&tk, &bar[bf ? 4 : 1], sVb(bf), a.vcol + hd * LD, krow0 + j * LQ);
  };
  if (threadIdx.x == 0 && nkt > 0) {
    mbar_expect_tx(&bar[0], 2 * LT);
    tma_load_2d(&tq, &bar[0], sQ, a.qcol + hd * LD, row0 + q0);
    tma_load_2d(&tdo, &bar[0], sdO, hd * LD, row0 + q0);
    load_kv(0, 0);
  }
  float Dh = 0.f, Lt = 0.f;
  if (live) Lt = a.lse_in[((int64_t)b * a.h + hd) * S + q];
  if (!DC && live) {   // D_q = rowsum(dO * O): half hf sums dims [32hf, 32hf + 32)
    float ov[32], dv[32];
    ld_bf16x32(a.O + ((int64_t)row0 + q) * a.H + hd * LD + 32 * hf, ov);
    ld_bf16x32(a.dO + ((int64_t)row0 + q) * a.H + hd * LD + 32 * hf, dv);
#pragma unroll
    for (int i = 0; i < 32; ++i) Dh += ov[i] * dv[i];
  }
  const float sl2 = a.scale * 1.4426950408889634f, Ll2 = Lt * 1.4426950408889634f;
  const uint64_t ebase = (((uint64_t)b * a.h + hd) * S + (uint64_t)q) * Sk;
  uint32_t ph_kv0 = 0, ph_kv1 = 0;
  int ph_s = 0, ph_o = 0;
  float Dt = 0.f;
  // pass 0 (DC only): D over every key tile; pass 1: dS and dQ += dS K
  for (int pass = DC ? 0 : 1; pass < 2; ++pass) {
    if (pass == 1) {
      red[hf * 128 + t] = Dh;
      __syncthreads();
      Dt = red[t] + red[128 + t];
      if (hf == 0 && q < S) a.Dbuf[((int64_t)b * a.h + hd) * S + q] = Dt;
      __syncthreads();                          // every D read before red[] is reused
      if (DC && threadIdx.x == 0 && nkt > 0) load_kv(0, 0);   // pass 0's MMAs are done (bar[2] waited)
    }
    for (int j = 0; j < nkt; ++j) {
      const int bf = j & 1;
      uint8_t* sK = sKb(bf);
      uint8_t* sV = sVb(bf);
      if (threadIdx.x == 0) {
        if (j + 1 < nkt) load_kv(j + 1, bf ^ 1);   // buffer !bf held tile j-1: its MMAs are done
        if (j == 0 && pass == (DC ? 0 : 1)) mbar_wait(&bar[0], 0);
        if (bf) { mbar_wait(&bar[4], ph_kv1); ph_kv1 ^= 1; }
        else { mbar_wait(&bar[1], ph_kv0); ph_kv0 ^= 1; }
        tc_fence_after();
        mma_nt64(tmem, smem_u32(sQ), smem_u32(sK));          // S = Q K^T
        mma_nt64(tmem + 128, smem_u32(sdO), smem_u32(sV));   // dP~ = dO V^T
        mma_commit(&bar[2]);
      }
      mbar_wait(&bar[2], ph_s);
      ph_s ^= 1;
      __syncwarp();
      tc_fence_after();
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        float sv[16], dp[16];
        tmem_ld16(trow + 64 * hf + 16 * c, sv);
        tmem_ld16(trow + 128 + 64 * hf + 16 * c, dp);
        const int kb = j * LQ + 64 * hf + 16 * c;
        if (live && kb < kl) {
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            const int k = kb + 4 * g;
            const float4 f = k < kl ? drop4l(a.drop, ebase + k) : make_float4(0.f, 0.f, 0.f, 0.f);
            const float ff[4] = {f.x, f.y, f.z, f.w};
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const float p = (k + i < kl) ? ex2a(fmaf(sv[4 * g + i], sl2, -Ll2)) : 0.f;
              if (pass == 0) Dh = fmaf(p * ff[i], dp[4 * g + i], Dh);
              dp[4 * g + i] = p * (dp[4 * g + i] * ff[i] - Dt) * a.scale;   // dS (scale folded)
            }
          }
        } else {
#pragma unroll
          for (int i = 0; i < 16; ++i) dp[i] = 0.f;
        }
        if (pass == 1) st_row16(sdS, t, 4 * hf + c, dp);
      }
      if (pass == 0) {
        bar_sync_all();                          // S / dP read before the next tile's MMAs
        continue;
      }
      fence_async_smem();
      bar_sync_all();
      if (threadIdx.x == 0) {
        mma_pv(tmem + 256, smem_u32(sdS), smem_u32(sK), j > 0);   // dQ += dS K
        mma_commit(&bar[3]);
      }
      mbar_wait(&bar[3], ph_o);
      ph_o ^= 1;
      __syncwarp();
      tc_fence_after();
    }
  }
  {
    float v[32];
    tmem_ld32(trow + 256 + 32 * hf, v);
    if (nkt == 0 || !live) {
#pragma unroll
      for (int i = 0; i < 32; ++i) v[i] = 0.f;
    }
    if (q < S) st_bf16x32(a.dq + ((int64_t)row0 + q) * a.ldq + a.ocq + hd * LD + 32 * hf, v);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    tmem_free(tmem, 512);
  }
}

// --------------------------------------------------------- backward dK, dV --
constexpr int LKV_SMEM = 6 * LT + 2 * LPT + 1024 + 2048;   // K, V, Q[2], dO[2], P~, dS

__global__ void __launch_bounds__(LTH, 1) k_attn_bwd_dkv_tcl(const __grid_constant__ CUtensorMap tq,
                                                             const __grid_constant__ CUtensorMap tk,
                                                             const __grid_constant__ CUtensorMap tdo, const LArgs a) {
  pdl_enter();
  extern __shared__ uint8_t smraw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)smraw + 1023) & ~(uintptr_t)1023);
  uint8_t* sK = sm;
  uint8_t* sV = sm + LT;
  // Q_i / dO_i in buffer (i - i0) & 1: tile i+1 loads while tile i is processed
  auto sQb = [&](int bf) { return sm + 2 * LT + 2 * LT * bf; };
  auto sdOb = [&](int bf) { return sm + 3 * LT + 2 * LT * bf; };
  uint8_t* sP = sm + 6 * LT;
  uint8_t* sdS = sP + LPT;
  uint64_t* bar = (uint64_t*)(sdS + LPT);       // [0] K/V, [1] Q/dO buf 0, [2] MMA S/dP, [3] MMA dV/dK, [4] Q/dO buf 1
  uint32_t* tslot = (uint32_t*)(bar + 6);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int hf = warp >> 2, t = 32 * (warp & 3) + lane;
  const int k0 = blockIdx.x * LQ, bh = blockIdx.y, b = bh / a.h, hd = bh % a.h;
  const int S = a.S, Sk = a.Sk, len = a.lengths[b], klen = a.klens[b];
  // query tiles that see keys [k0, k0 + 128): causal -> q >= k0; only q < len carry gradient
  const int i0 = a.causal ? k0 / LQ : 0;
  const int i1 = k0 < klen ? (len + LQ - 1) / LQ : 0;
  if (threadIdx.x == 0) {
    for (int i = 0; i < 5; ++i) mbar_init(&bar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) tmem_alloc(tslot, 512);
  bar_sync_all();
  const uint32_t tmem = *tslot;                 // S 0..127, dP 128..255, dV 256..319, dK 320..383
  const uint32_t trow = tmem + ((uint32_t)(32 * (warp & 3)) << 16);
  const int row0 = b * S, krow0 = b * Sk;
  if (threadIdx.x == 0 && i1 > i0) {
    mbar_expect_tx(&bar[0], 2 * LT);
    tma_load_2d(&tk, &bar[0], sK, a.kcol + hd * LD, krow0 + k0);
    tma_load_2d(&tk, &bar[0], sV, a.vcol + hd * LD, krow0 + k0);
    mbar_expect_tx(&bar[1], 2 * LT);
    tma_load_2d(&tq, &bar[1], sQb(0), a.qcol + hd * LD, row0 + i0 * LQ);
    tma_load_2d(&tdo, &bar[1], sdOb(0), hd * LD, row0 + i0 * LQ);
  }
  const float sl2 = a.scale * 1.4426950408889634f;
  uint32_t ph_q0 = 0, ph_q1 = 0;
  int ph_s = 0, ph_o = 0;
  for (int i = i0; i < i1; ++i) {
    const int bf = (i - i0) & 1;
    uint8_t* sQ = sQb(bf);
    uint8_t* sdO = sdOb(bf);
    if (threadIdx.x == 0) {
      if (i + 1 < i1) {                         // buffer !bf held tile i-1: its MMAs are done
        mbar_expect_tx(&bar[bf ? 1 : 4], 2 * LT);
        tma_load_2d(&tq, &bar[bf ? 1 : 4], sQb(bf ^ 1), a.qcol + hd * LD, row0 + (i + 1) * LQ);
        tma_load_2d(&tdo, &bar[bf ? 1 : 4], sdOb(bf ^ 1), hd * LD, row0 + (i + 1) * LQ);
      }
      if (i == i0) mbar_wait(&bar[0], 0);
      if (bf) { mbar_wait(&bar[4], ph_q1); ph_q1 ^= 1; }
      else { mbar_wait(&bar[1], ph_q0); ph_q0 ^= 1; }
      tc_fence_after();
      mma_nt64(tmem, smem_u32(sQ), smem_u32(sK));          // S_i = Q_i K^T (rows = queries)
      mma_nt64(tmem + 128, smem_u32(sdO), smem_u32(sV));   // dP~_i = dO_i V^T
      mma_commit(&bar[2]);
    }
    const int q = i * LQ + t;
    const bool live = q < len;
    const int kl = a.causal ? min(klen, q + 1) : klen;
    float Lt = 0.f, Dt = 0.f;
    if (live) {
      Lt = a.lse_in[((int64_t)b * a.h + hd) * S + q];
      Dt = a.Dbuf[((int64_t)b * a.h + hd) * S + q];
    }
    const float Ll2 = Lt * 1.4426950408889634f;
    const uint64_t ebase = (((uint64_t)b * a.h + hd) * S + (uint64_t)q) * Sk;
    mbar_wait(&bar[2], ph_s);
    ph_s ^= 1;
    __syncwarp();
    tc_fence_after();
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      float sv[16], dp[16];
      tmem_ld16(trow + 64 * hf + 16 * c, sv);
      tmem_ld16(trow + 128 + 64 * hf + 16 * c, dp);
      const int kb = k0 + 64 * hf + 16 * c;
      if (live && kb < kl) {
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          const int k = kb + 4 * g;
          const float4 f = k < kl ? drop4l(a.drop, ebase + k) : make_float4(0.f, 0.f, 0.f, 0.f);
          const float ff[4] = {f.x, f.y, f.z, f.w};
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const float p = (k + e < kl) ? ex2a(fmaf(sv[4 * g + e], sl2, -Ll2)) : 0.f;
            sv[4 * g + e] = p * ff[e];                                    // P~
            dp[4 * g + e] = p * (dp[4 * g + e] * ff[e] - Dt) * a.scale;   // dS
          }
        }
      } else {
#pragma unroll
        for (int e = 0; e < 16; ++e) { sv[e] = 0.f; dp[e] = 0.f; }
      }
      st_row16(sP, t, 4 * hf + c, sv);
      st_row16(sdS, t, 4 * hf + c, dp);
    }
    fence_async_smem();
    bar_sync_all();
    if (threadIdx.x == 0) {
      mma_ptx(tmem + 256, smem_u32(sP), smem_u32(sdO), i > i0);   // dV += P~^T dO
      mma_ptx(tmem + 320, smem_u32(sdS), smem_u32(sQ), i > i0);   // dK += dS^T Q
      mma_commit(&bar[3]);
    }
    mbar_wait(&bar[3], ph_o);
    ph_o ^= 1;
    __syncwarp();
    tc_fence_after();
  }
  {  // TMEM lanes of dV / dK = key rows k0 + t
    const int k = k0 + t;
    __nv_bfloat16* row = a.dkv + ((int64_t)krow0 + k) * a.ldk + hd * LD + 32 * hf;
    float v[32];
    tmem_ld32(trow + 320 + 32 * hf, v);
    if (i1 <= i0) {
#pragma unroll
      for (int e = 0; e < 32; ++e) v[e] = 0.f;
    }
    if (k < Sk) st_bf16x32(row + a.ock, v);              // dK
    tmem_ld32(trow + 256 + 32 * hf, v);
    if (i1 <= i0) {
#pragma unroll
      for (int e = 0; e < 32; ++e) v[e] = 0.f;
    }
    if (k < Sk) st_bf16x32(row + a.ocv, v);              // dV
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    tmem_free(tmem, 512);
  }
}

}  // namespace

// ------------------------------------------------------------------ host --
bool tc_map_bf16(CUtensorMap* out, const void* ptr, uint64_t inner, uint64_t outer, uint64_t stride_elems,
                 uint32_t box_inner, uint32_t box_outer);   // kernels_gemm_tc.cu

bool attn_tcl_ok(int S, int H, int h) { return S > LQ && S <= 1024 && H / h == LD && H % 64 == 0; }

namespace {
LArgs self_args(int B, int S, int H, int h, Drop drop, const int32_t* lengths, bool causal) {
  LArgs a{};
  a.S = S; a.Sk = S; a.H = H; a.h = h; a.B = B;
  a.qcol = 0; a.kcol = H; a.vcol = 2 * H;
  a.scale = 1.0f / sqrtf((float)LD);
  a.drop = drop; a.lengths = lengths; a.klens = lengths; a.causal = causal;
  a.ldq = 3 * H; a.ocq = 0; a.ldk = 3 * H; a.ock = H; a.ocv = 2 * H;
  return a;
}
void set_attrs() {
  static std::once_flag once;
  std::call_once(once, [] {
    cudaFuncSetAttribute(k_attn_fwd_tcl, cudaFuncAttributeMaxDynamicSharedMemorySize, LF_SMEM);
    cudaFuncSetAttribute(k_attn_bwd_dq_tcl<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, LQ_SMEM);
    cudaFuncSetAttribute(k_attn_bwd_dq_tcl<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, LQ_SMEM);
    cudaFuncSetAttribute(k_attn_bwd_dkv_tcl, cudaFuncAttributeMaxDynamicSharedMemorySize, LKV_SMEM);
  });
}
}  // namespace

bool attn_fwd_tcl(const void* qkv, const int32_t* lengths, void* O, float* lse, int B, int S, int H, int h,
                  Drop drop, cudaStream_t st, bool causal) {
  if (!attn_tcl_ok(S, H, h)) return false;
  CUtensorMap tq;
  if (!tc_map_bf16(&tq, qkv, 3ull * H, (uint64_t)B * S, 3ull * H, 64, LQ)) return false;
  set_attrs();
  LArgs a = self_args(B, S, H, h, drop, lengths, causal);
  a.Oout = (__nv_bfloat16*)O; a.lse = lse;
  launch_k(k_attn_fwd_tcl, dim3((S + LQ - 1) / LQ, B * h), LTH, LF_SMEM, st, tq, tq, a);
  return true;
}

bool attn_bwd_tcl(const void* qkv, const void* O, const void* dO, const float* lse, const int32_t* lengths,
                  float* Dbuf, void* dqkv, int B, int S, int H, int h, Drop drop, cudaStream_t st, bool causal) {
  if (!attn_tcl_ok(S, H, h)) return false;
  CUtensorMap tq, tdo;
  if (!tc_map_bf16(&tq, qkv, 3ull * H, (uint64_t)B * S, 3ull * H, 64, LQ)) return false;
  if (!tc_map_bf16(&tdo, dO, (uint64_t)H, (uint64_t)B * S, (uint64_t)H, 64, LQ)) return false;
  set_attrs();
  LArgs a = self_args(B, S, H, h, drop, lengths, causal);
  a.O = (const __nv_bfloat16*)O; a.dO = (const __nv_bfloat16*)dO;
  a.lse_in = lse; a.Dbuf = Dbuf; a.dq = (__nv_bfloat16*)dqkv; a.dkv = (__nv_bfloat16*)dqkv;
  const dim3 grid((S + LQ - 1) / LQ, B * h);
  launch_k(k_attn_bwd_dq_tcl<false>, grid, LTH, LQ_SMEM, st, tq, tq, tdo, a);   // also writes D for the dK/dV pass
  launch_k(k_attn_bwd_dkv_tcl, grid, LTH, LKV_SMEM, st, tq, tq, tdo, a);
  return true;
}

// Cross-attention (encoder-decoder) on the tiled kernels: queries q [B*Sq, H],
// keys / values kv [B*Sk, 2H]; Sq, Sk <= 1024.  The backward's D is the
// consistent sum_k P~ dP~ (dQ kernel pass 0), kept in Dbuf [B, h, Sq].
bool attn_cross_tcl_ok(int Sq, int Sk, int H, int h) {
  return Sq <= 1024 && Sk <= 1024 && H / h == LD && H % 64 == 0;
}

bool attn_cross_fwd_tcl(const void* q, const void* kv, const int32_t* qlens, const int32_t* klens, void* O, float* lse,
                        int B, int Sq, int Sk, int H, int h, Drop drop, cudaStream_t st) {
  if (!attn_cross_tcl_ok(Sq, Sk, H, h)) return false;
  CUtensorMap tq, tk;
  if (!tc_map_bf16(&tq, q, (uint64_t)H, (uint64_t)B * Sq, (uint64_t)H, 64, LQ)) return false;
  if (!tc_map_bf16(&tk, kv, 2ull * H, (uint64_t)B * Sk, 2ull * H, 64, LQ)) return false;
  set_attrs();
  LArgs a = self_args(B, Sq, H, h, drop, qlens, false);
  a.Sk = Sk; a.klens = klens; a.qcol = 0; a.kcol = 0; a.vcol = H;
  a.Oout = (__nv_bfloat16*)O; a.lse = lse;
  launch_k(k_attn_fwd_tcl, dim3((Sq + LQ - 1) / LQ, B * h), LTH, LF_SMEM, st, tq, tk, a);
  return true;
}

bool attn_cross_bwd_tcl(const void* q, const void* kv, const void* O, const void* dO, const float* lse,
                        const int32_t* qlens, const int32_t* klens, float* Dbuf, void* dq, void* dkv, int B, int Sq,
                        int Sk, int H, int h, Drop drop, cudaStream_t st) {
  if (!attn_cross_tcl_ok(Sq, Sk, H, h)) return false;
  CUtensorMap tq, tk, tdo;
  if (!tc_map_bf16(&tq, q, (uint64_t)H, (uint64_t)B * Sq, (uint64_t)H, 64, LQ)) return false;
  if (!tc_map_bf16(&tk, kv, 2ull * H, (uint64_t)B * Sk, 2ull * H, 64, LQ)) return false;
  if (!tc_map_bf16(&tdo, dO, (uint64_t)H, (uint64_t)B * Sq, (uint64_t)H, 64, LQ)) return false;
  set_attrs();
  LArgs a = self_args(B, Sq, H, h, drop, qlens, false);
  a.Sk = Sk; a.klens = klens; a.qcol = 0; a.kcol = 0; a.vcol = H;
  a.O = (const __nv_bfloat16*)O; a.dO = (const __nv_bfloat16*)dO; a.lse_in = lse; a.Dbuf = Dbuf;
  a.dq = (__nv_bfloat16*)dq; a.ldq = H; a.ocq = 0;
  a.dkv = (__nv_bfloat16*)dkv; a.ldk = 2 * H; a.ock = 0; a.ocv = H;
  launch_k(k_attn_bwd_dq_tcl<true>, dim3((Sq + LQ - 1) / LQ, B * h), LTH, LQ_SMEM, st, tq, tk, tdo, a);
  launch_k(k_attn_bwd_dkv_tcl, dim3((Sk + LQ - 1) / LQ, B * h), LTH, LKV_SMEM, st, tq, tk, tdo, a);
  return true;
}

}  // namespace mimose
