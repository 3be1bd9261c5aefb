// tcgen05 / TMEM / TMA GEMM for bf16 mode on sm_100a.
//
//   C[m, n] = sum_k A(m, k) B(n, k)  (+ the fused epilogues of gemm_epi.cuh)
//
// One CTA computes a 128 x BN tile with fp32 accumulators in TMEM:
//   warp 0      TMA producer: 128B-swizzled A/B k-blocks (64 wide) into a
//               STAGES-deep smem ring, mbarrier complete_tx
//   warp 1      TMEM allocation + the single-thread tcgen05.mma issuer
//               (kind::f16, M=128, N=BN, K=16 per instruction); tcgen05.commit
//               frees smem stages and finally signals the epilogue
//   warps 2..5  epilogue: tcgen05.ld 32x32b.x32 (warp w reads TMEM lanes
//               32*(w%4)..), fused bias / GELU / dropout+residual / GELU' /
//               residual-add / split-K fp32, vectorised global stores
// Operands may be K-major (forward: X, W; dgrad: dY) or MN-major (dgrad: W;
// wgrad: dY^T, X^T) — the UMMA descriptors encode both, so no transposes are
// materialised.  Split-K over blockIdx.z writes fp32 partials that a fixed-order
// kernel reduces (deterministic wgrad).
#include <cuda.h>

#include <cstdio>
#include <atomic>
#include <mutex>
#include <unordered_map>

#include "gemm_epi.cuh"
#include "kernels.h"
#include "tc_common.cuh"

namespace mimose {

constexpr int TBM = 128, TBK = 64;
struct TcArgs {
  GemmArgs g;
  int a_mn, b_mn;           // 1: operand is MN-major (MN contiguous)
  int kb_per_split;         // k-blocks per blockIdx.z
  int kb_total;
};

// ---- coalesced tile stores through a per-warp staging buffer -------------
// The warp holds a 32 x 32 fragment (lane = row).  It is written to a 32 x 128 B
// smem buffer with the 16-B chunk index XOR-swizzled by row, then read back so
// that each store instruction writes whole row segments: fp32 -> 4 rows x 128 B,
// bf16 -> 8 rows x 64 B (full 32-B sectors, no partial-sector writes).
MDEV void sts128(uint32_t a, uint4 w) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(w.x), "r"(w.y), "r"(w.z), "r"(w.w) : "memory");
}
MDEV uint4 lds128(uint32_t a) {
  uint4 w;
  asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(w.x), "=r"(w.y), "=r"(w.z), "=r"(w.w) : "r"(a) : "memory");
  return w;
}
MDEV void stage_store_f32(uint8_t* stg_p, const float (&v)[32], float* out, int64_t ld, int rows_valid, int lane) {
  const uint32_t stg = (uint32_t)__cvta_generic_to_shared(stg_p);
#pragma unroll
  for (int c = 0; c < 8; ++c)
    sts128(stg + lane * 128 + ((c ^ (lane & 7)) << 4),
           make_uint4(__float_as_uint(v[4 * c]), __float_as_uint(v[4 * c + 1]), __float_as_uint(v[4 * c + 2]),
                      __float_as_uint(v[4 * c + 3])));
  __syncwarp();
#pragma unroll
  for (int h = 0; h < 2; ++h) {   // shared loads in groups of 4, then the stores (no LDS -> STG round trips)
    uint4 w[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int R = (lane >> 3) + 4 * (4 * h + k), c = lane & 7;
      w[k] = lds128(stg + R * 128 + ((c ^ (R & 7)) << 4));
    }
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int R = (lane >> 3) + 4 * (4 * h + k), c = lane & 7;
      if (R < rows_valid) *(uint4*)(out + (int64_t)R * ld + 4 * c) = w[k];
    }
  }
  __syncwarp();
}
// bf16 fragments travel packed: pk[c] = columns 8c..8c+7 of row `lane` (pack8 order).
MDEV void stage_store_bf16(uint8_t* stg_p, const uint4 (&pk)[4], __nv_bfloat16* out, int64_t ld, int rows_valid,
                           int lane) {
  const uint32_t stg = (uint32_t)__cvta_generic_to_shared(stg_p);
#pragma unroll
  for (int c = 0; c < 4; ++c) sts128(stg + lane * 128 + ((c ^ (lane & 3)) << 4), pk[c]);
  __syncwarp();
  uint4 w[4];
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int R = (lane >> 2) + 8 * k, c = lane & 3;
    w[k] = lds128(stg + R * 128 + ((c ^ (R & 3)) << 4));
  }
  __syncwarp();
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int R = (lane >> 2) + 8 * k, c = lane & 3;
    if (R < rows_valid) *(uint4*)(out + (int64_t)R * ld + 8 * c) = w[k];
  }
}


// ---- TMA (bulk tensor) stores: the warp writes its 32 x 32 fragment into its
// staging buffer in the tensor map's swizzled layout and one lane issues
// cp.async.bulk.tensor (global <- shared); the TMA unit writes whole lines and
// clips rows >= M, and the warp does not wait for the write.  bf16 fragments
// (64-B rows, SWIZZLE_64B: 16-B chunk ^= (row / 2) % 4) alternate between the
// two 2 KB halves of the buffer; fp32 fragments (128-B rows, SWIZZLE_128B:
// chunk ^= row % 8) use all 4 KB.  Before a half is rewritten, the bulk group
// that last read it must have finished reading (wait_group.read).
struct EpiOut {
  uint8_t* stg;             // this warp's 4 KB staging buffer (1024-B aligned)
  const CUtensorMap* mc;    // map of C (TMA mode)
  const CUtensorMap* mc2;   // map of C2 (TMA mode, GELU epilogues)
  int half;                 // next bf16 half
};
template <int N>
MDEV void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
MDEV void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
MDEV void tma_store_2d(const CUtensorMap* map, uint32_t src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];"
               ::"l"(map), "r"(src), "r"(c0), "r"(c1) : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
MDEV void tma_out_bf16(EpiOut& o, const uint4 (&pk)[4], const CUtensorMap* map, int n, int m_base, int lane) {
  const uint32_t s = smem_u32(o.stg) + 2048u * (uint32_t)o.half;
  o.half ^= 1;
  if (lane == 0) bulk_wait_read<1>();    // the group before last used this half
  __syncwarp();
#pragma unroll
  for (int c = 0; c < 4; ++c) sts128(s + lane * 64 + ((c ^ ((lane >> 1) & 3)) << 4), pk[c]);
  fence_async_smem();
  __syncwarp();
  if (lane == 0) tma_store_2d(map, s, n, m_base);
}
MDEV void tma_out_f32(EpiOut& o, const float (&v)[32], const CUtensorMap* map, int n, int m_base, int lane) {
  const uint32_t s = smem_u32(o.stg);
  if (lane == 0) bulk_wait_read<0>();
  __syncwarp();
#pragma unroll
  for (int c = 0; c < 8; ++c)
    sts128(s + lane * 128 + ((c ^ (lane & 7)) << 4),
           make_uint4(__float_as_uint(v[4 * c]), __float_as_uint(v[4 * c + 1]), __float_as_uint(v[4 * c + 2]),
                      __float_as_uint(v[4 * c + 3])));
  fence_async_smem();
  __syncwarp();
  if (lane == 0) tma_store_2d(map, s, n, m_base);
}
// Output of one fragment: TMA (ST = 1) or LSU stores through the staging buffer (ST = 0).
template <int ST>
MDEV void out_bf16p(EpiOut& o, const uint4 (&pk)[4], __nv_bfloat16* base, int64_t ld, const CUtensorMap* map, int n,
                    int m_base, int rows_valid, int lane) {
  if constexpr (ST == 1) tma_out_bf16(o, pk, map, n, m_base, lane);
  else stage_store_bf16(o.stg, pk, base + (int64_t)m_base * ld + n, ld, rows_valid, lane);
}
template <int ST>
MDEV void out_bf16(EpiOut& o, const float (&v)[32], __nv_bfloat16* base, int64_t ld, const CUtensorMap* map, int n,
                   int m_base, int rows_valid, int lane) {
  uint4 pk[4];
#pragma unroll
  for (int c = 0; c < 4; ++c) pk[c] = pack8(v + 8 * c);
  out_bf16p<ST>(o, pk, base, ld, map, n, m_base, rows_valid, lane);
}
// GELU epilogues: u = acc + bias is stored as bf16 and the GELU reads the STORED
// u, so u is packed once (F2FP pairs) and unpacked with integer shifts instead of
// a per-element F2F round trip (which runs on the quarter-rate XU pipe beside the
// MUFU.TANH of the GELU).
template <int ST>
MDEV void out_u_gelu(EpiOut& o, float (&v)[32], __nv_bfloat16* u, __nv_bfloat16* gout, int64_t ld,
                     const CUtensorMap* mu, const CUtensorMap* mg, int n, int m_base, int rows_valid, int lane) {
  uint4 pk[4];
#pragma unroll
  for (int c = 0; c < 4; ++c) pk[c] = pack8(v + 8 * c);
  out_bf16p<ST>(o, pk, u, ld, mu, n, m_base, rows_valid, lane);
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    const uint32_t w[4] = {pk[c].x, pk[c].y, pk[c].z, pk[c].w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const float2 uu = make_float2(__uint_as_float(w[j] << 16), __uint_as_float(w[j] & 0xFFFF0000u));
      const float2 r = gelu_fast_x2(uu);
      v[8 * c + 2 * j] = r.x;
      v[8 * c + 2 * j + 1] = r.y;
    }
  }
  out_bf16<ST>(o, v, gout, ld, mg, n, m_base, rows_valid, lane);
}
template <int ST>
MDEV void out_f32(EpiOut& o, const float (&v)[32], float* base, int64_t ld, const CUtensorMap* map, int n, int m_base,
                  int rows_valid, int lane) {
  if constexpr (ST == 1) tma_out_f32(o, v, map, n, m_base, lane);
  else stage_store_f32(o.stg, v, base + (int64_t)m_base * ld + n, ld, rows_valid, lane);
}

// Epilogue inputs of one 32-column chunk, loaded one chunk ahead (software
// pipelining hides the L2 latency of bias / u / residual behind the previous
// chunk's math and stores).
struct EpiIn {
  uint4 b[4];   // bias (bf16 x 32)
  uint4 x[8];   // aux or residual: bf16 x 32 uses x[0..3], fp32 x 32 uses x[0..7]
};

// Dropout keep bits of the 32 consecutive elements e0..e0+31 (e0 % 4 == 0): bit i
// = word(e0 + i) < thresh, the same Philox words and rule as drop_factor4.  The
// persistent GEMM computes them before its accumulator is ready, so the Philox
// work of a tile overlaps that tile's MMAs instead of extending its epilogue.
MDEV uint32_t drop_bits32(const Drop& d, uint64_t e0) {
  if (!d.enabled) return 0xFFFFFFFFu;
  uint32_t bits = 0;
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    const uint4 w = drop_words(d, (e0 >> 2) + q);
    bits |= ((uint32_t)(w.x < d.thresh) | ((uint32_t)(w.y < d.thresh) << 1) | ((uint32_t)(w.z < d.thresh) << 2) |
             ((uint32_t)(w.w < d.thresh) << 3)) << (4 * q);
  }
  return bits;
}
MDEV float4 drop_from_bits(const Drop& d, uint32_t bits, int q) {
  const float s = d.enabled ? d.scale : 1.0f;
  return make_float4((bits >> (4 * q)) & 1 ? s : 0.f, (bits >> (4 * q + 1)) & 1 ? s : 0.f,
                     (bits >> (4 * q + 2)) & 1 ? s : 0.f, (bits >> (4 * q + 3)) & 1 ? s : 0.f);
}
// Row-tensor inputs of a chunk (residual / GELU' aux) are loaded COALESCED --
// consecutive lanes read consecutive 16-B pieces of one row (fp32: 8 lanes per
// 128-B row, 4 rows per instruction; bf16: 4 lanes per 64-B row, 8 rows) -- and
// transposed to the lane = row layout of the accumulator fragment through the
// warp's staging buffer (epi_in_transpose).  One row per lane per instruction
// would touch 32 lines per load (32 L1 wavefronts instead of 4-8).
template <int EPI>
constexpr int epi_in_kind() {   // 0 none, 1 bf16 rows, 2 fp32 rows
  return (EPI == EPI_BIAS_DROP_RES || EPI == EPI_GELU_BWD || EPI == EPI_GELUT_BWD) ? 1
       : (EPI == EPI_ACC_RES_F32 || EPI == EPI_BIAS_DROP_RESF32) ? 2 : 0;
}
template <int EPI>
MDEV void epi_load(const GemmArgs& g, int m_base, int n, int lane, EpiIn& in) {
  if constexpr (EPI == EPI_BIAS || EPI == EPI_BIAS_GELU || EPI == EPI_BIAS_DROP_RES || EPI == EPI_BIAS_GELUT ||
                EPI == EPI_BIAS_DROP_RESF32) {
    const uint4* p = (const uint4*)((const __nv_bfloat16*)g.bias + n);
#pragma unroll
    for (int i = 0; i < 4; ++i) in.b[i] = p[i];
  }
  if constexpr (epi_in_kind<EPI>() == 1) {
    const __nv_bfloat16* base = EPI == EPI_BIAS_DROP_RES ? (const __nv_bfloat16*)g.res : (const __nv_bfloat16*)g.aux;
    const int64_t ld = EPI == EPI_BIAS_DROP_RES ? g.ldr : g.ldx;
#pragma unroll
    for (int k = 0; k < 4; ++k) {   // rows >= M: defined (zero) inputs, results never stored
      const int R = 8 * k + (lane >> 2), c = lane & 3;
      in.x[k] = m_base + R < g.M ? *(const uint4*)(base + (int64_t)(m_base + R) * ld + n + 8 * c) : make_uint4(0u, 0u, 0u, 0u);
    }
  } else if constexpr (epi_in_kind<EPI>() == 2) {
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int R = 4 * k + (lane >> 3), c = lane & 7;
      in.x[k] = m_base + R < g.M ? *(const uint4*)((const float*)g.res + (int64_t)(m_base + R) * g.ldr + n + 4 * c)
                                 : make_uint4(0u, 0u, 0u, 0u);
    }
  }
}
// Coalesced pieces -> lane = row: bf16 x[c] = columns 8c..8c+7 of row `lane`,
// fp32 x[c] = columns 4c..4c+3 (bf16: 64-B rows, chunk ^= (row / 2) % 4; fp32:
// 128-B rows, chunk ^= row % 8 -- conflict-free both ways).  The buffer must be
// free: the previous TMA store has finished reading it (ST = 1), the LSU staging
// ends with __syncwarp (ST = 0).
template <int EPI, int ST>
MDEV void epi_in_transpose(EpiOut& o, EpiIn& in, int lane) {
  constexpr int kind = epi_in_kind<EPI>();
  if constexpr (kind != 0) {
    const uint32_t s = smem_u32(o.stg);
    if constexpr (ST == 1) {
      if (lane == 0) bulk_wait_read<0>();
    }
    __syncwarp();
    if constexpr (kind == 1) {
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const int R = 8 * k + (lane >> 2), c = lane & 3;
        sts128(s + R * 64 + ((c ^ ((R >> 1) & 3)) << 4), in.x[k]);
      }
      __syncwarp();
#pragma unroll
      for (int c = 0; c < 4; ++c) in.x[c] = lds128(s + lane * 64 + ((c ^ ((lane >> 1) & 3)) << 4));
    } else {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const int R = 4 * k + (lane >> 3), c = lane & 7;
        sts128(s + R * 128 + ((c ^ (R & 7)) << 4), in.x[k]);
      }
      __syncwarp();
#pragma unroll
      for (int c = 0; c < 8; ++c) in.x[c] = lds128(s + lane * 128 + ((c ^ (lane & 7)) << 4));
    }
    __syncwarp();   // every lane has its row before the buffer takes the output
  }
}

template <int EPI, int ST>
MDEV void epi_frag32_in(const GemmArgs& g, int m_base, int n, float (&v)[32], int z, EpiOut& o, int lane,
                        EpiIn& in, uint32_t keep) {
  epi_in_transpose<EPI, ST>(o, in, lane);
  using E = __nv_bfloat16;
  const int m = m_base + lane;
  const int rows_valid = g.M - m_base;
  const bool live = m < g.M;
  if constexpr (EPI == EPI_STORE) {
    out_bf16<ST>(o, v, (E*)g.C, g.ldc, o.mc, n, m_base, rows_valid, lane);
  } else if constexpr (EPI == EPI_BIAS || EPI == EPI_BIAS_GELU || EPI == EPI_BIAS_DROP_RES) {
    float b[32];
#pragma unroll
    for (int i = 0; i < 4; ++i) unpack8(in.b[i], b + 8 * i);
#pragma unroll
    for (int i = 0; i < 32; i += 2) {
      const float2 r = fadd2(make_float2(v[i], v[i + 1]), make_float2(b[i], b[i + 1]));
      v[i] = r.x;
      v[i + 1] = r.y;
    }
    if constexpr (EPI == EPI_BIAS) {
      out_bf16<ST>(o, v, (E*)g.C, g.ldc, o.mc, n, m_base, rows_valid, lane);
    } else if constexpr (EPI == EPI_BIAS_GELU) {
      out_u_gelu<ST>(o, v, (E*)g.C, (E*)g.C2, g.ldc, o.mc, o.mc2, n, m_base, rows_valid, lane);
    } else {
      float r[32];
#pragma unroll
      for (int i = 0; i < 4; ++i) unpack8(in.x[i], r + 8 * i);
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        // rows >= M: zero residual and keep bits, never stored
        const float4 f = drop_from_bits(g.drop, keep, q);
        v[4 * q + 0] = r[4 * q + 0] + v[4 * q + 0] * f.x;
        v[4 * q + 1] = r[4 * q + 1] + v[4 * q + 1] * f.y;
        v[4 * q + 2] = r[4 * q + 2] + v[4 * q + 2] * f.z;
        v[4 * q + 3] = r[4 * q + 3] + v[4 * q + 3] * f.w;
      }
      out_f32<ST>(o, v, (float*)g.C, g.ldc, o.mc, n, m_base, rows_valid, lane);
    }
  } else if constexpr (EPI == EPI_GELU_BWD) {
    float u[32];
#pragma unroll
    for (int i = 0; i < 4; ++i) unpack8(in.x[i], u + 8 * i);
#pragma unroll
    for (int i = 0; i < 32; i += 2) {   // rows >= M are never stored
      const float2 r = fmul2(make_float2(v[i], v[i + 1]), gelu_grad_fast_x2(make_float2(u[i], u[i + 1])));
      v[i] = r.x;
      v[i + 1] = r.y;
    }
    out_bf16<ST>(o, v, (E*)g.C, g.ldc, o.mc, n, m_base, rows_valid, lane);
  } else if constexpr (EPI == EPI_ACC_RES_F32) {
    if (live) {
      const float4* r = (const float4*)in.x;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const float4 a = r[q];
        v[4 * q] += a.x; v[4 * q + 1] += a.y; v[4 * q + 2] += a.z; v[4 * q + 3] += a.w;
      }
    }
    out_f32<ST>(o, v, (float*)g.C, g.ldc, o.mc, n, m_base, rows_valid, lane);
  } else if constexpr (EPI == EPI_BIAS_GELUT || EPI == EPI_BIAS_DROP_RESF32) {
    float b[32];
#pragma unroll
    for (int i = 0; i < 4; ++i) unpack8(in.b[i], b + 8 * i);
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] += b[i];
    if constexpr (EPI == EPI_BIAS_GELUT) {   // gelu_new == the tanh form
      out_u_gelu<ST>(o, v, (E*)g.C, (E*)g.C2, g.ldc, o.mc, o.mc2, n, m_base, rows_valid, lane);
    } else {
      const float* r = (const float*)in.x;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        // rows >= M: zero residual and keep bits, never stored
        const float4 f = drop_from_bits(g.drop, keep, q);
        v[4 * q + 0] = r[4 * q + 0] + v[4 * q + 0] * f.x;
        v[4 * q + 1] = r[4 * q + 1] + v[4 * q + 1] * f.y;
        v[4 * q + 2] = r[4 * q + 2] + v[4 * q + 2] * f.z;
        v[4 * q + 3] = r[4 * q + 3] + v[4 * q + 3] * f.w;
      }
      out_f32<ST>(o, v, (float*)g.C, g.ldc, o.mc, n, m_base, rows_valid, lane);
    }
  } else if constexpr (EPI == EPI_GELUT_BWD) {
    float u[32];
#pragma unroll
    for (int i = 0; i < 4; ++i) unpack8(in.x[i], u + 8 * i);
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] *= gelu_grad_fast(u[i]);
    out_bf16<ST>(o, v, (E*)g.C, g.ldc, o.mc, n, m_base, rows_valid, lane);
  } else if constexpr (EPI == EPI_ACC_F32) {
    if (live) {
      float* out = (float*)g.C + (int64_t)m * g.ldc + n;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        float4 a = ((float4*)out)[q];
        a.x += v[4 * q]; a.y += v[4 * q + 1]; a.z += v[4 * q + 2]; a.w += v[4 * q + 3];
        ((float4*)out)[q] = a;
      }
    }
  } else if constexpr (EPI == EPI_NONE) {
    float t = 0.f;
#pragma unroll
    for (int i = 0; i < 32; ++i) t += v[i];
    if (t == 1234.5f) ((float*)g.C)[0] = t;
  } else {
    out_f32<ST>(o, v, (float*)g.C + (int64_t)z * g.split_stride, g.ldc, o.mc, n, m_base, rows_valid, lane);   // TMA: split 1
  }
}

constexpr int TP_EPI_WARPS = 8;
constexpr int TP_THREADS = 64 + 32 * TP_EPI_WARPS;

template <int BN, int ST>
struct TpCfg {
  static constexpr int STAGES = BN >= 256 ? 4 : (BN >= 128 ? 6 : 8);
  static constexpr int A_BYTES = TBM * TBK * 2;
  static constexpr int B_BYTES = BN * TBK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STG_PER = 4096;   // per-warp store staging (1024-B aligned: TMA swizzle atoms)
  static constexpr int STG_BYTES = TP_EPI_WARPS * STG_PER;
  static constexpr int SMEM = STAGES * STAGE_BYTES + STG_BYTES + 1024 + 256;
};

struct TpArgs {
  TcArgs t;
  int m_blocks = 0, n_blocks = 0, n_tiles = 0;
};

// Work segment i of this CTA: tile r (m-block * n_blocks + n-block), split z
// and k-block range [kb0, kb1); tile-major round robin, unit = blockIdx.x + i * gridDim.x.
struct Seg { int r, z, kb0, kb1, p = 0; };
MDEV bool seg_of(const TpArgs& a, int i, Seg& s) {
  const TcArgs& ta = a.t;
  const int tile = blockIdx.x + i * gridDim.x;
  if (tile >= a.n_tiles) return false;
  const int per_split = a.m_blocks * a.n_blocks;
  s.z = tile / per_split;
  s.r = tile % per_split;
  s.kb0 = s.z * ta.kb_per_split;
  s.kb1 = min(ta.kb_total, s.kb0 + ta.kb_per_split);
  return true;
}
// Grouped launch of two independent problems (same epilogue, no split): tiles
// of problem 0 first, then problem 1, one round-robin order over both.
template <bool G2>
MDEV bool seg_of2(const TpArgs& a, const TpArgs& a2, int i, Seg& s) {
  if constexpr (!G2) {
    return seg_of(a, i, s);
  } else {
    const int tile = blockIdx.x + i * gridDim.x;
    if (tile >= a.n_tiles + a2.n_tiles) return false;
    s.p = tile >= a.n_tiles;
    s.r = s.p ? tile - a.n_tiles : tile;
    s.z = 0;
    s.kb0 = 0;
    s.kb1 = (s.p ? a2 : a).t.kb_total;
    return true;
  }
}
// Epilogue of one accumulator tile by one epilogue warp: rows m0 + 32 q + lane
// (q = TMEM lane quarter of the warp), column group grp of the BN columns.
// Keep bits and the first chunk's inputs are prepared before the accumulator
// is waited for (tfull_bar, parity), so they overlap the tile's MMAs.
template <int BN, int EPI, int ST>
MDEV void epi_tile(const GemmArgs& g, int m0, int n0, int z, bool no_k, uint32_t tacc, uint64_t* tfull_bar,
                   uint32_t parity, EpiOut& eo, int q, int grp, int lane) {
  const int m = m0 + 32 * q + lane;
  constexpr int ngrp = TP_EPI_WARPS / 4;
  const int c_beg = grp * (BN / 32) / ngrp, c_end = (grp + 1) * (BN / 32) / ngrp;
  {  // pull this tile's epilogue inputs into L2 while the MMAs run
    const int nb = n0 + 32 * c_beg;
    if (m < g.M && nb < g.N) {
      const char* pa = nullptr;
      int bytes = 0;
      const int ncol = 32 * (c_end - c_beg);
      if constexpr (EPI == EPI_GELU_BWD || EPI == EPI_GELUT_BWD) { pa = (const char*)((const __nv_bfloat16*)g.aux + (int64_t)m * g.ldx + nb); bytes = 2 * ncol; }
      if constexpr (EPI == EPI_BIAS_DROP_RESF32) { pa = (const char*)((const float*)g.res + (int64_t)m * g.ldr + nb); bytes = 4 * ncol; }
      if constexpr (EPI == EPI_BIAS_DROP_RES) { pa = (const char*)((const __nv_bfloat16*)g.res + (int64_t)m * g.ldr + nb); bytes = 2 * ncol; }
      if constexpr (EPI == EPI_ACC_RES_F32) { pa = (const char*)((const float*)g.res + (int64_t)m * g.ldr + nb); bytes = 4 * ncol; }
      for (int o = 0; o < bytes; o += 128) asm volatile("prefetch.global.L2 [%0];" ::"l"(pa + o));
    }
  }
  // dropout keep bits of this warp's chunks, computed while the MMAs run
  constexpr int NCH = BN / 32 / (TP_EPI_WARPS / 4);
  uint32_t kbits[NCH];
  constexpr bool DROP_EPI = EPI == EPI_BIAS_DROP_RES || EPI == EPI_BIAS_DROP_RESF32;
#pragma unroll
  for (int i = 0; i < NCH; ++i) {
    kbits[i] = 0u;
    if constexpr (DROP_EPI) {
      const int n = n0 + 32 * (c_beg + i);
      if (m < g.M && n + 32 <= g.N) kbits[i] = drop_bits32(g.drop, (uint64_t)m * g.ldc + n);
    }
  }
  EpiIn nxt;   // the first chunk's epilogue inputs are in flight while the MMAs finish
  if (n0 + 32 * c_beg + 32 <= g.N) epi_load<EPI>(g, m0 + 32 * q, n0 + 32 * c_beg, lane, nxt);
  mbar_wait(tfull_bar, parity);
  __syncwarp();
  tc_fence_after();
#pragma unroll 1
  for (int c = c_beg; c < c_end; ++c) {
    EpiIn cur = nxt;
    const uint32_t keep = kbits[0];
#pragma unroll
    for (int i = 0; i + 1 < NCH; ++i) kbits[i] = kbits[i + 1];   // register rotation, no local memory
    const int n = n0 + 32 * c;
    if (c + 1 < c_end && n + 64 <= g.N) epi_load<EPI>(g, m0 + 32 * q, n + 32, lane, nxt);
    float v[32];
    tmem_ld32(tacc + ((uint32_t)(32 * q) << 16) + 32 * c, v);
    if (no_k) {
#pragma unroll
      for (int i = 0; i < 32; ++i) v[i] = 0.f;
    }
    if (n + 32 <= g.N) {
      if (m0 + 32 * q < g.M) epi_frag32_in<EPI, ST>(g, m0 + 32 * q, n, v, z, eo, lane, cur, keep);
    } else if (m < g.M) {
#pragma unroll
      for (int i = 0; i < 32; ++i)
        if (n + i < g.N) epilogue<__nv_bfloat16, EPI>(g, m, n + i, v[i], z);
    }
  }
}

template <int BN, int EPI, bool G2, int ST>
__global__ void __launch_bounds__(TP_THREADS, 1)
    k_gemm_tcp(const __grid_constant__ CUtensorMap tma_a, const __grid_constant__ CUtensorMap tma_b, const TpArgs args,
               const __grid_constant__ CUtensorMap tma_a2, const __grid_constant__ CUtensorMap tma_b2,
               const TpArgs args2, const __grid_constant__ CUtensorMap tma_c,
               const __grid_constant__ CUtensorMap tma_c2) {
  pdl_trigger();
  using Cf = TpCfg<BN, ST>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* stg_base = smem + Cf::STAGES * Cf::STAGE_BYTES;
  uint64_t* full = (uint64_t*)(stg_base + Cf::STG_BYTES);
  uint64_t* empty = full + Cf::STAGES;
  uint64_t* tfull = empty + Cf::STAGES;    // [2]
  uint64_t* tempty = tfull + 2;            // [2]
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  const TcArgs& ta = args.t;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < Cf::STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    for (int a = 0; a < 2; ++a) { mbar_init(&tfull[a], 1); mbar_init(&tempty[a], TP_EPI_WARPS); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tma_a) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tma_b) : "memory");
    if (G2) {
      asm volatile("prefetch.tensormap [%0];" ::"l"(&tma_a2) : "memory");
      asm volatile("prefetch.tensormap [%0];" ::"l"(&tma_b2) : "memory");
    }
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(2 * BN));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();                                       // prologue above overlaps the previous kernel
  const int per_split = args.m_blocks * args.n_blocks;

  if (warp == 0) {
    if (lane == 0) {                                   // ---------------- TMA producer
      int it = 0;
      Seg sg;
      for (int si = 0; seg_of2<G2>(args, args2, si, sg); ++si) {
        const TpArgs& A = (G2 && sg.p) ? args2 : args;
        const TcArgs& ta = A.t;
        const CUtensorMap* map_a = (G2 && sg.p) ? &tma_a2 : &tma_a;
        const CUtensorMap* map_b = (G2 && sg.p) ? &tma_b2 : &tma_b;
        const int r = sg.r;
        const int m0 = (r / A.n_blocks) * TBM, n0 = (r % A.n_blocks) * BN;
        const int kb0 = sg.kb0, kb1 = sg.kb1;
        for (int kb = kb0; kb < kb1; ++kb, ++it) {
          const int s = it % Cf::STAGES;
          if (it >= Cf::STAGES) mbar_wait(&empty[s], ((it / Cf::STAGES) - 1) & 1);
          uint8_t* sa = smem + s * Cf::STAGE_BYTES;
          uint8_t* sb = sa + Cf::A_BYTES;
          const int k = kb * TBK;
          mbar_expect_tx(&full[s], Cf::STAGE_BYTES);
          if (ta.a_mn) {
            tma_load_2d(map_a, &full[s], sa, m0, k);
            tma_load_2d(map_a, &full[s], sa + 8192, m0 + 64, k);
          } else {
            tma_load_2d(map_a, &full[s], sa, k, m0);
          }
          if (ta.b_mn) {
#pragma unroll
            for (int j = 0; j < BN / 64; ++j) tma_load_2d(map_b, &full[s], sb + 8192 * j, n0 + 64 * j, k);
          } else {
#pragma unroll
            for (int j = 0; j < (BN + 255) / 256; ++j)      // box rows <= 256
              tma_load_2d(map_b, &full[s], sb + j * 256 * 128, k, n0 + 256 * j);
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {                                   // ---------------- MMA issuer
      int it = 0, local = 0;
      Seg sg;
      for (; seg_of2<G2>(args, args2, local, sg); ++local) {
        const TcArgs& ta = ((G2 && sg.p) ? args2 : args).t;
        const uint32_t idesc = idesc_bf16(TBM, BN, ta.a_mn, ta.b_mn);
        const int kb0 = sg.kb0, kb1 = sg.kb1;
        const int acc = local & 1;
        if (local >= 2) mbar_wait(&tempty[acc], ((local >> 1) - 1) & 1);
        tc_fence_after();
        const uint32_t d = tmem + acc * BN;
        for (int kb = kb0; kb < kb1; ++kb, ++it) {
          const int s = it % Cf::STAGES;
          mbar_wait(&full[s], (it / Cf::STAGES) & 1);
          tc_fence_after();
          const uint32_t sa = smem_u32(smem + s * Cf::STAGE_BYTES);
          const uint32_t sb = sa + Cf::A_BYTES;
#pragma unroll
          for (int kk = 0; kk < TBK / 16; ++kk) {
            const uint64_t da = ta.a_mn ? make_desc(sa + kk * 2048, 8192, 1024) : make_desc(sa + kk * 32, 16, 1024);
            const uint64_t db = ta.b_mn ? make_desc(sb + kk * 2048, 8192, 1024) : make_desc(sb + kk * 32, 16, 1024);
            mma_bf16(d, da, db, idesc, (kb > kb0 || kk > 0) ? 1u : 0u);
          }
          mma_commit(&empty[s]);
        }
        mma_commit(&tfull[acc]);
      }
    }
  } else {                                             // ---------------- epilogue warps
    const int e = warp - 2;
    EpiOut eo{stg_base + e * Cf::STG_PER, &tma_c, &tma_c2, 0};
    const int q = warp & 3;                            // TMEM lane quarter of this warp
    const int grp = e >> 2;                            // column group of this warp
    int local = 0;
    Seg sg;
    for (; seg_of2<G2>(args, args2, local, sg); ++local) {
      const TpArgs& A = (G2 && sg.p) ? args2 : args;
      const GemmArgs& g = A.t.g;
      if constexpr (G2) eo.mc = sg.p ? &tma_c2 : &tma_c;
      const int z = sg.z, r = sg.r;
      const int m0 = (r / A.n_blocks) * TBM, n0 = (r % A.n_blocks) * BN;
      const int kb0 = sg.kb0, kb1 = sg.kb1;
      const int acc = local & 1;
      epi_tile<BN, EPI, ST>(g, m0, n0, z, kb1 <= kb0, tmem + acc * BN, &tfull[acc], (local >> 1) & 1, eo, q, grp,
                            lane);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&tempty[acc])) : "memory");
    }
    if constexpr (ST == 1) {
      if (lane == 0) bulk_wait_all();   // the bulk stores have completed before the CTA exits
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(2 * BN));
  }
}


// ---------------------------------------------------------------------------
// CTA-pair kernel (cta_group::2): a cluster of two CTAs (one TPC) computes
// 256 x BN tiles.  CTA r TMA-loads rows [128 r, 128 r + 128) of A and rows
// [BN/2 r, BN/2 (r + 1)) of the B tile into its own smem, the transaction bytes
// of both landing on the leader's full barrier; the leader's single thread
// issues tcgen05.mma.cta_group::2 (M = 256, N = BN), which reads both CTAs'
// smem and accumulates rows 128 r.. of the tile in CTA r's TMEM.  Commits are
// multicast to both CTAs (stage release, accumulator ready); both CTAs'
// epilogue warps release an accumulator on the leader's tmem-empty barrier.
// Per SM the B bytes per MMA and the smem operand reads are halved relative to
// the single-CTA kernel, and a stage is 32 KB (6 stages in flight).  Each CTA
// runs the same epilogue (epi_tile) on its 128 rows.
// ---------------------------------------------------------------------------
constexpr uint32_t PEER_MASK = 0xFEFFFFFFu;   // shared::cta address -> the leader CTA's copy

template <int BN>
struct T2Cfg {
  static constexpr int A_BYTES = TBM * TBK * 2;
  static constexpr int B_BYTES = (BN / 2) * TBK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES = (192 * 1024) / STAGE_BYTES;
  static constexpr int STG_PER = 4096;
  static constexpr int STG_BYTES = TP_EPI_WARPS * STG_PER;
  static constexpr int SMEM = STAGES * STAGE_BYTES + STG_BYTES + 1024 + 256;
};

MDEV uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
MDEV void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
MDEV void tma_load_2d_2sm(const CUtensorMap* map, uint64_t* bar, void* dst, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
      ::"r"(smem_u32(dst)), "l"(map), "r"(smem_u32(bar) & PEER_MASK), "r"(c0), "r"(c1) : "memory");
}
MDEV void mma_bf16_2sm(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}"
      ::"r"(tmem_d), "l"(da), "l"(db), "r"(idesc), "r"(acc));
}
MDEV void mma_commit_2sm_mc(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
               ::"r"(smem_u32(bar)), "h"((uint16_t)3) : "memory");
}
MDEV void mbar_arrive_rank(uint64_t* bar, uint32_t rank) {
  asm volatile("{\n\t.reg .b32 ra;\n\tmapa.shared::cluster.u32 ra, %0, %1;\n\t"
               "mbarrier.arrive.release.cluster.shared::cluster.b64 _, [ra];\n\t}"
               ::"r"(smem_u32(bar)), "r"(rank) : "memory");
}

template <int BN, int EPI, int ST>
__global__ void __launch_bounds__(TP_THREADS, 1)
    k_gemm_tc2(const __grid_constant__ CUtensorMap tma_a, const __grid_constant__ CUtensorMap tma_b, const TpArgs args,
               const __grid_constant__ CUtensorMap tma_c, const __grid_constant__ CUtensorMap tma_c2) {
  pdl_trigger();
  using Cf = T2Cfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* stg_base = smem + Cf::STAGES * Cf::STAGE_BYTES;
  uint64_t* full = (uint64_t*)(stg_base + Cf::STG_BYTES);
  uint64_t* empty = full + Cf::STAGES;
  uint64_t* tfull = empty + Cf::STAGES;    // [2]
  uint64_t* tempty = tfull + 2;            // [2] (the leader's are used)
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  const TcArgs& ta = args.t;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_rank();
  const bool leader = rank == 0;
  const int cid = blockIdx.x >> 1, ncl = gridDim.x >> 1;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < Cf::STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    for (int a = 0; a < 2; ++a) { mbar_init(&tfull[a], 1); mbar_init(&tempty[a], 2 * TP_EPI_WARPS); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tma_a) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tma_b) : "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(2 * BN));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();

  if (warp == 0) {
    if (lane == 0) {                                   // ---------------- TMA producer (both CTAs)
      int it = 0;
      for (int tile = cid; tile < args.n_tiles; tile += ncl) {
        const int m0 = (tile / args.n_blocks) * 256 + 128 * (int)rank;
        const int nb = (tile % args.n_blocks) * BN + (BN / 2) * (int)rank;
        for (int kb = 0; kb < ta.kb_total; ++kb, ++it) {
          const int s = it % Cf::STAGES;
          if (it >= Cf::STAGES) mbar_wait(&empty[s], ((it / Cf::STAGES) - 1) & 1);
          uint8_t* sa = smem + s * Cf::STAGE_BYTES;
          uint8_t* sb = sa + Cf::A_BYTES;
          const int k = kb * TBK;
          if (leader) mbar_expect_tx(&full[s], 2 * Cf::STAGE_BYTES);
          if (ta.a_mn) {
            tma_load_2d_2sm(&tma_a, &full[s], sa, m0, k);
            tma_load_2d_2sm(&tma_a, &full[s], sa + 8192, m0 + 64, k);
          } else {
            tma_load_2d_2sm(&tma_a, &full[s], sa, k, m0);
          }
          if (ta.b_mn) {
#pragma unroll
            for (int j = 0; j < BN / 128; ++j) tma_load_2d_2sm(&tma_b, &full[s], sb + 8192 * j, nb + 64 * j, k);
          } else {
            tma_load_2d_2sm(&tma_b, &full[s], sb, k, nb);
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && leader) {                         // ---------------- MMA issuer (leader)
      const uint32_t idesc = idesc_bf16(256, BN, ta.a_mn, ta.b_mn);
      int it = 0, local = 0;
      for (int tile = cid; tile < args.n_tiles; tile += ncl, ++local) {
        const int acc = local & 1;
        if (local >= 2) mbar_wait(&tempty[acc], ((local >> 1) - 1) & 1);
        tc_fence_after();
        const uint32_t d = tmem + acc * BN;
        for (int kb = 0; kb < ta.kb_total; ++kb, ++it) {
          const int s = it % Cf::STAGES;
          mbar_wait(&full[s], (it / Cf::STAGES) & 1);
          tc_fence_after();
          const uint32_t sa = smem_u32(smem + s * Cf::STAGE_BYTES);
          const uint32_t sb = sa + Cf::A_BYTES;
#pragma unroll
          for (int kk = 0; kk < TBK / 16; ++kk) {
            const uint64_t da = ta.a_mn ? make_desc(sa + kk * 2048, 8192, 1024) : make_desc(sa + kk * 32, 16, 1024);
            const uint64_t db = ta.b_mn ? make_desc(sb + kk * 2048, 8192, 1024) : make_desc(sb + kk * 32, 16, 1024);
            mma_bf16_2sm(d, da, db, idesc, (kb > 0 || kk > 0) ? 1u : 0u);
          }
          mma_commit_2sm_mc(&empty[s]);
        }
        mma_commit_2sm_mc(&tfull[acc]);
      }
    }
  } else {                                             // ---------------- epilogue warps (both CTAs)
    const int e = warp - 2;
    EpiOut eo{stg_base + e * Cf::STG_PER, &tma_c, &tma_c2, 0};
    const int q = warp & 3, grp = e >> 2;
    const GemmArgs& g = ta.g;
    int local = 0;
    for (int tile = cid; tile < args.n_tiles; tile += ncl, ++local) {
      const int m0 = (tile / args.n_blocks) * 256 + 128 * (int)rank;
      const int n0 = (tile % args.n_blocks) * BN;
      const int acc = local & 1;
      epi_tile<BN, EPI, ST>(g, m0, n0, 0, ta.kb_total <= 0, tmem + acc * BN, &tfull[acc], (local >> 1) & 1, eo, q,
                            grp, lane);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive_rank(&tempty[acc], 0);
    }
    if constexpr (ST == 1) {
      if (lane == 0) bulk_wait_all();
    }
  }
  tc_fence_before();
  cluster_sync_all();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(2 * BN));
  }
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeFn encode_fn() {
  static EncodeFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (EncodeFn)p;
  });
  return fn;
}

struct MapKey {
  const void* ptr;
  uint64_t inner, outer, stride;
  uint32_t box_inner, box_outer;
  int f32, swz;
  bool operator==(const MapKey& o) const {
    return ptr == o.ptr && inner == o.inner && outer == o.outer && stride == o.stride &&
           box_inner == o.box_inner && box_outer == o.box_outer && f32 == o.f32 && swz == o.swz;
  }
};
struct MapKeyHash {
  size_t operator()(const MapKey& k) const {
    size_t h = std::hash<const void*>()(k.ptr);
    for (uint64_t v : {k.inner, k.outer, k.stride, (uint64_t)k.box_inner << 32 | k.box_outer,
                       (uint64_t)k.f32 << 8 | (uint64_t)k.swz})
      h ^= std::hash<uint64_t>()(v) + 0x9e3779b97f4a7c15ull + (h << 6) + (h >> 2);
    return h;
  }
};

// 2D bf16 (or fp32) tensor [outer][inner] (inner contiguous), row stride in
// elements; swizzle 128B (operand tiles, fp32 store tiles) or 64B (bf16 store tiles).
static bool make_map(CUtensorMap* out, const void* ptr, uint64_t inner, uint64_t outer, uint64_t stride_elems,
                     uint32_t box_inner, uint32_t box_outer, int f32 = 0, int swz = 128) {
  static std::unordered_map<MapKey, CUtensorMap, MapKeyHash> cache;
  static std::mutex mu;
  MapKey key{ptr, inner, outer, stride_elems, box_inner, box_outer, f32, swz};
  std::lock_guard<std::mutex> lk(mu);
  auto it = cache.find(key);
  if (it != cache.end()) { *out = it->second; return true; }
  EncodeFn fn = encode_fn();
  if (!fn) return false;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {stride_elems * (f32 ? 4 : 2)};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = fn(out, f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2,
                  const_cast<void*>(ptr), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  swz == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return false;
  if (cache.size() > 8192) cache.clear();
  cache.emplace(key, *out);
  return true;
}

bool tc_map_bf16(CUtensorMap* out, const void* ptr, uint64_t inner, uint64_t outer, uint64_t stride_elems,
                 uint32_t box_inner, uint32_t box_outer) {
  return make_map(out, ptr, inner, outer, stride_elems, box_inner, box_outer);
}

static int num_sms();

template <int BN, int EPI, int ST>
static void launch_tcp(const CUtensorMap& ma, const CUtensorMap& mb, const TpArgs& a, const CUtensorMap& mc,
                       const CUtensorMap& mc2, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_gemm_tcp<BN, EPI, false, ST>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         TpCfg<BN, ST>::SMEM);
    attr = true;
  }
  launch_k(k_gemm_tcp<BN, EPI, false, ST>, std::min(num_sms(), a.n_tiles), TP_THREADS, TpCfg<BN, ST>::SMEM, st, ma,
           mb, a, ma, mb, a, mc, mc2);
}

// Two independent EPI_F32 problems in one persistent launch (grouped wgrad);
// mc / mc2: the two problems' C maps (TMA stores).
template <int BN, int ST>
static void launch_tcp_g2(const CUtensorMap& ma, const CUtensorMap& mb, const TpArgs& a, const CUtensorMap& ma2,
                          const CUtensorMap& mb2, const TpArgs& a2, const CUtensorMap& mc, const CUtensorMap& mc2,
                          cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_gemm_tcp<BN, EPI_F32, true, ST>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         TpCfg<BN, ST>::SMEM);
    attr = true;
  }
  launch_k(k_gemm_tcp<BN, EPI_F32, true, ST>, std::min(num_sms(), a.n_tiles + a2.n_tiles), TP_THREADS,
           TpCfg<BN, ST>::SMEM, st, ma, mb, a, ma2, mb2, a2, mc, mc2);
}

// ST = 1 (TMA stores) for every epilogue that overwrites its output; the
// read-modify-write EPI_ACC_F32 and the benchmark EPI_NONE keep LSU stores.
template <int BN, int ST>
static void dispatch_tcp(Epi epi, const CUtensorMap& ma, const CUtensorMap& mb, const TpArgs& a,
                         const CUtensorMap& mc, const CUtensorMap& mc2, cudaStream_t st) {
  switch (epi) {
    case EPI_STORE: launch_tcp<BN, EPI_STORE, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_BIAS: launch_tcp<BN, EPI_BIAS, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_BIAS_GELU: launch_tcp<BN, EPI_BIAS_GELU, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_BIAS_DROP_RES: launch_tcp<BN, EPI_BIAS_DROP_RES, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_GELU_BWD: launch_tcp<BN, EPI_GELU_BWD, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_ACC_RES_F32: launch_tcp<BN, EPI_ACC_RES_F32, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_NONE: launch_tcp<BN, EPI_NONE, 0>(ma, mb, a, mc, mc2, st); break;
    case EPI_BIAS_GELUT: launch_tcp<BN, EPI_BIAS_GELUT, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_GELUT_BWD: launch_tcp<BN, EPI_GELUT_BWD, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_BIAS_DROP_RESF32: launch_tcp<BN, EPI_BIAS_DROP_RESF32, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_ACC_F32: launch_tcp<BN, EPI_ACC_F32, 0>(ma, mb, a, mc, mc2, st); break;
    default: launch_tcp<BN, EPI_F32, ST>(ma, mb, a, mc, mc2, st); break;
  }
}

template <int BN, int EPI, int ST>
static void launch_tc2(const CUtensorMap& ma, const CUtensorMap& mb, const TpArgs& a, const CUtensorMap& mc,
                       const CUtensorMap& mc2, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_gemm_tc2<BN, EPI, ST>, cudaFuncAttributeMaxDynamicSharedMemorySize, T2Cfg<BN>::SMEM);
    attr = true;
  }
  launch_kc(k_gemm_tc2<BN, EPI, ST>, 2 * std::min(num_sms() / 2, a.n_tiles), TP_THREADS, T2Cfg<BN>::SMEM, st, 2, ma,
            mb, a, mc, mc2);
}

template <int BN, int ST>
static void dispatch_tc2(Epi epi, const CUtensorMap& ma, const CUtensorMap& mb, const TpArgs& a,
                         const CUtensorMap& mc, const CUtensorMap& mc2, cudaStream_t st) {
  switch (epi) {
    case EPI_STORE: launch_tc2<BN, EPI_STORE, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_BIAS: launch_tc2<BN, EPI_BIAS, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_BIAS_GELU: launch_tc2<BN, EPI_BIAS_GELU, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_BIAS_DROP_RES: launch_tc2<BN, EPI_BIAS_DROP_RES, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_GELU_BWD: launch_tc2<BN, EPI_GELU_BWD, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_ACC_RES_F32: launch_tc2<BN, EPI_ACC_RES_F32, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_NONE: launch_tc2<BN, EPI_NONE, 0>(ma, mb, a, mc, mc2, st); break;
    case EPI_BIAS_GELUT: launch_tc2<BN, EPI_BIAS_GELUT, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_GELUT_BWD: launch_tc2<BN, EPI_GELUT_BWD, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_BIAS_DROP_RESF32: launch_tc2<BN, EPI_BIAS_DROP_RESF32, ST>(ma, mb, a, mc, mc2, st); break;
    case EPI_ACC_F32: launch_tc2<BN, EPI_ACC_F32, 0>(ma, mb, a, mc, mc2, st); break;
    default: launch_tc2<BN, EPI_F32, ST>(ma, mb, a, mc, mc2, st); break;
  }
}

static int num_sms() {
  static int nsm = 0;
  if (!nsm) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (nsm <= 0) nsm = 148;
  }
  return nsm;
}

static int g_gemm_mode = 1;   // 1: default; 12 / 13: force 128 x 256 / 128 x 128 tiles and no grouped launches; 15: LSU-store epilogues instead of TMA stores; 17: CTA-pair kernel (test hooks)
void set_gemm_mode(int m) { g_gemm_mode = m; }

bool tc_available() { return encode_fn() != nullptr; }

// Output maps of the TMA-store epilogue: 32 x 32 boxes of C / C2 (bf16 with
// 64-B rows and SWIZZLE_64B, fp32 with 128-B rows and SWIZZLE_128B).
static bool epi_out_f32(Epi e) {
  return e == EPI_BIAS_DROP_RES || e == EPI_ACC_RES_F32 || e == EPI_F32 || e == EPI_BIAS_DROP_RESF32;
}
static bool out_map(CUtensorMap* m, const void* ptr, int M, int N, int64_t ld, bool f32) {
  if (!ptr || ((uintptr_t)ptr & 15) || (ld * (f32 ? 4 : 2)) % 16) return false;
  return make_map(m, ptr, (uint64_t)N, (uint64_t)M, (uint64_t)ld, 32, 32, f32 ? 1 : 0, f32 ? 128 : 64);
}
static bool tma_store_ok(Epi epi, const GemmArgs& g, CUtensorMap* mc, CUtensorMap* mc2) {
  if (g_gemm_mode == 15 || g.split != 1 || epi == EPI_ACC_F32 || epi == EPI_NONE) return false;
  const bool f32 = epi_out_f32(epi);
  if (!out_map(mc, g.C, g.M, g.N, g.ldc, f32)) return false;
  if (epi == EPI_BIAS_GELU || epi == EPI_BIAS_GELUT) return out_map(mc2, g.C2, g.M, g.N, g.ldc, false);
  *mc2 = *mc;
  return true;
}

bool gemm_tc(Epi epi, const GemmArgs& g, cudaStream_t st) {
  TcArgs a;
  a.g = g;
  // operand majors from the strides; the contiguous stride must be 1 and the
  // row stride 16-B aligned (multiple of 8 bf16)
  if (g.a_sk == 1 && g.a_sm % 8 == 0) a.a_mn = 0;
  else if (g.a_sm == 1 && g.a_sk % 8 == 0) a.a_mn = 1;
  else return false;
  if (g.b_sk == 1 && g.b_sn % 8 == 0) a.b_mn = 0;
  else if (g.b_sn == 1 && g.b_sk % 8 == 0) a.b_mn = 1;
  else return false;
  if (((uintptr_t)g.A | (uintptr_t)g.B) & 15) return false;
  // vectorised epilogue needs 16-B aligned rows of every epilogue tensor
  if (g.ldc % 8 || (g.res && g.ldr % 8) || (g.aux && g.ldx % 8)) return false;
  a.kb_total = (g.K + TBK - 1) / TBK;
  a.kb_per_split = (a.kb_total + g.split - 1) / g.split;
  const int m_blocks = (g.M + TBM - 1) / TBM;
  // BN = 256 when N is a multiple of 256 and the 128x256 tiles fill at least half
  // of the SMs; BN = 128 otherwise (measured per shape, tools/one_gemm.py).
  // 128-wide tiles run at ~0.58 of the 256-wide mainloop rate (half the work at
  // ~1.15x the time): 256-wide wins as soon as its tiles occupy half the SMs
  // (measured: T = 3584 x 768 x 3072 dropout-residual 29.1 us at 256 vs 39.5 at
  // 128; T = 2560: 27.6 vs 23.8).  Stream-K, CTA pairs, BN = 64, the
  // one-tile-per-CTA kernel and an in-kernel fused split-K were built in round
  // 1, measured slower on the step shapes and removed.
  // CTA pairs (256 x 256 tiles over two SMs) where the single-CTA kernel has
  // >= 600 tiles of 128 x 256 (about four waves) and the epilogue carries no
  // Philox dropout: measured 5-9% faster there (T = 8192 x 3072 / 4096 x 1024,
  // GPT-2's 50264 x 1024 x 2048 dW_e; BERT-large 622 -> 633 samples/s), equal
  // or slower with fewer tiles or the dropout epilogues (mode 17 vs 12 in
  // tools/bench_gemm.py; profiles/r2/gemm_tile_sweep.txt).
  const bool drop_epi = epi == EPI_BIAS_DROP_RES || epi == EPI_BIAS_DROP_RESF32;
  const bool pair = g.split == 1 && g.N % 256 == 0 &&
                    (g_gemm_mode == 17 || (g_gemm_mode == 1 && !drop_epi && g.bn != 128 &&
                                           (int64_t)m_blocks * (g.N / 256) >= 600));
  if (pair) {
    CUtensorMap ma2, mb2, mc, mc2;
    bool ok2 = a.a_mn ? make_map(&ma2, g.A, g.M, g.K, g.a_sk, 64, 64) : make_map(&ma2, g.A, g.K, g.M, g.a_sm, 64, TBM);
    if (ok2) ok2 = a.b_mn ? make_map(&mb2, g.B, g.N, g.K, g.b_sk, 64, 64) : make_map(&mb2, g.B, g.K, g.N, g.b_sn, 64, 128);
    if (ok2) {
      TpArgs p;
      p.t = a;
      p.m_blocks = (g.M + 255) / 256;
      p.n_blocks = g.N / 256;
      p.n_tiles = p.m_blocks * p.n_blocks;
      if (tma_store_ok(epi, g, &mc, &mc2)) dispatch_tc2<256, 1>(epi, ma2, mb2, p, mc, mc2, st);
      else dispatch_tc2<256, 0>(epi, ma2, mb2, p, ma2, ma2, st);
      return true;
    }
  }
  auto tiles = [&](int bn) { return m_blocks * ((g.N + bn - 1) / bn) * g.split; };
  int BN = (g.N % 256 == 0 && 2 * tiles(256) >= num_sms()) ? 256 : 128;
  if (g.bn == 256 && g.N % 256 == 0) BN = 256;
  if (g.bn == 128) BN = 128;
  if (g_gemm_mode == 12 && g.N % 256 == 0) BN = 256;
  if (g_gemm_mode == 13) BN = 128;
  CUtensorMap ma, mb;
  bool ok;
  if (a.a_mn) ok = make_map(&ma, g.A, g.M, g.K, g.a_sk, 64, 64);
  else ok = make_map(&ma, g.A, g.K, g.M, g.a_sm, 64, TBM);
  if (!ok) return false;
  if (a.b_mn) ok = make_map(&mb, g.B, g.N, g.K, g.b_sk, 64, 64);
  else ok = make_map(&mb, g.B, g.K, g.N, g.b_sn, 64, std::min(BN, 256));
  if (!ok) return false;
  TpArgs p;
  p.t = a;
  p.m_blocks = m_blocks;
  p.n_blocks = (g.N + BN - 1) / BN;
  p.n_tiles = p.m_blocks * p.n_blocks * g.split;
  CUtensorMap mc, mc2;
  if (tma_store_ok(epi, g, &mc, &mc2)) {
    if (BN == 256) dispatch_tcp<256, 1>(epi, ma, mb, p, mc, mc2, st);
    else dispatch_tcp<128, 1>(epi, ma, mb, p, mc, mc2, st);
  } else {
    if (BN == 256) dispatch_tcp<256, 0>(epi, ma, mb, p, ma, ma, st);
    else dispatch_tcp<128, 0>(epi, ma, mb, p, ma, ma, st);
  }
  return true;
}

// Grouped EPI_F32 GEMM: two independent problems (split 1, both operand majors
// as in gemm_tc) in one persistent launch -- tiles of g1 then g2 -- so two
// weight gradients with few output tiles each fill the SMs together (only when
// all tiles fit one wave; otherwise false and the caller launches them apart).  Each
// tile's K loop is the same as in a single launch, so results are bitwise
// equal to two separate launches with the same tile width.
bool gemm_tc_grouped(const GemmArgs& g1, const GemmArgs& g2, int bn, cudaStream_t st) {
  if ((g_gemm_mode != 1 && g_gemm_mode != 15) || g1.split != 1 || g2.split != 1) return false;
  if (bn != 128 && bn != 256) return false;
  TpArgs p[2];
  CUtensorMap ma[2], mb[2];
  const GemmArgs* gs[2] = {&g1, &g2};
  for (int i = 0; i < 2; ++i) {
    const GemmArgs& g = *gs[i];
    TcArgs a;
    a.g = g;
    if (g.a_sk == 1 && g.a_sm % 8 == 0) a.a_mn = 0;
    else if (g.a_sm == 1 && g.a_sk % 8 == 0) a.a_mn = 1;
    else return false;
    if (g.b_sk == 1 && g.b_sn % 8 == 0) a.b_mn = 0;
    else if (g.b_sn == 1 && g.b_sk % 8 == 0) a.b_mn = 1;
    else return false;
    if ((((uintptr_t)g.A | (uintptr_t)g.B) & 15) || g.ldc % 8 || g.N % bn) return false;
    a.kb_total = (g.K + TBK - 1) / TBK;
    a.kb_per_split = a.kb_total;
    bool ok = a.a_mn ? make_map(&ma[i], g.A, g.M, g.K, g.a_sk, 64, 64) : make_map(&ma[i], g.A, g.K, g.M, g.a_sm, 64, TBM);
    if (ok) ok = a.b_mn ? make_map(&mb[i], g.B, g.N, g.K, g.b_sk, 64, 64) : make_map(&mb[i], g.B, g.K, g.N, g.b_sn, 64, bn);
    if (!ok) return false;
    p[i].t = a;
    p[i].m_blocks = (g.M + TBM - 1) / TBM;
    p[i].n_blocks = g.N / bn;
    p[i].n_tiles = p[i].m_blocks * p[i].n_blocks;
  }
  if (p[0].n_tiles + p[1].n_tiles > num_sms()) return false;   // grouping pays only within one wave
  CUtensorMap mc[2];
  if (g_gemm_mode != 15 && out_map(&mc[0], g1.C, g1.M, g1.N, g1.ldc, true) &&
      out_map(&mc[1], g2.C, g2.M, g2.N, g2.ldc, true)) {
    if (bn == 256) launch_tcp_g2<256, 1>(ma[0], mb[0], p[0], ma[1], mb[1], p[1], mc[0], mc[1], st);
    else launch_tcp_g2<128, 1>(ma[0], mb[0], p[0], ma[1], mb[1], p[1], mc[0], mc[1], st);
  } else {
    if (bn == 256) launch_tcp_g2<256, 0>(ma[0], mb[0], p[0], ma[1], mb[1], p[1], ma[0], ma[0], st);
    else launch_tcp_g2<128, 0>(ma[0], mb[0], p[0], ma[1], mb[1], p[1], ma[0], ma[0], st);
  }
  return true;
}

}  // namespace mimose
