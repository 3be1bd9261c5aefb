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
#include <mutex>
#include <unordered_map>

#include "gemm_epi.cuh"
#include "kernels.h"
#include "tc_common.cuh"

namespace mimose {

constexpr int TBM = 128, TBK = 64;
constexpr int TC_THREADS = 192;

template <int BN>
struct TcCfg {
  // 3 stages (96 KB) so two CTAs share an SM: one CTA's epilogue overlaps the
  // other's TMA/MMA main loop, and 296 tiles are resident per wave
  static constexpr int STAGES = BN >= 256 ? 3 : 3;
  static constexpr int A_BYTES = TBM * TBK * 2;
  static constexpr int B_BYTES = BN * TBK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/;
};

struct TcArgs {
  GemmArgs g;
  int a_mn, b_mn;           // 1: operand is MN-major (MN contiguous)
  int kb_per_split;         // k-blocks per blockIdx.z
  int kb_total;
};

// Vectorised epilogue of 32 consecutive columns [n, n+32) of row m (all in range).
template <int EPI>
MDEV void epi_row32(const GemmArgs& g, int m, int n, float (&v)[32], int z = -1) {
  if (z < 0) z = blockIdx.z;
  using E = __nv_bfloat16;
  const int64_t o = (int64_t)m * g.ldc + n;
  if constexpr (EPI == EPI_STORE) {
    st_bf16x32((E*)g.C + o, v);
  } else if constexpr (EPI == EPI_BIAS || EPI == EPI_BIAS_GELU || EPI == EPI_BIAS_DROP_RES) {
    float b[32];
    ld_bf16x32((const E*)g.bias + n, b);
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] += b[i];
    if constexpr (EPI == EPI_BIAS) {
      st_bf16x32((E*)g.C + o, v);
    } else if constexpr (EPI == EPI_BIAS_GELU) {
      st_bf16x32((E*)g.C + o, v);
#pragma unroll
      for (int i = 0; i < 32; ++i) v[i] = gelu_f(__bfloat162float(__float2bfloat16_rn(v[i])));
      st_bf16x32((E*)g.C2 + o, v);
    } else {
      float r[32];
      ld_bf16x32((const E*)g.res + (int64_t)m * g.ldr + n, r);
      float* out = (float*)g.C + o;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const float4 f = drop_factor4(g.drop, (uint64_t)(o + 4 * q) >> 2);
        float4 w;
        w.x = r[4 * q + 0] + v[4 * q + 0] * f.x;
        w.y = r[4 * q + 1] + v[4 * q + 1] * f.y;
        w.z = r[4 * q + 2] + v[4 * q + 2] * f.z;
        w.w = r[4 * q + 3] + v[4 * q + 3] * f.w;
        ((float4*)out)[q] = w;
      }
    }
  } else if constexpr (EPI == EPI_GELU_BWD) {
    float u[32];
    ld_bf16x32((const E*)g.aux + (int64_t)m * g.ldx + n, u);
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] *= gelu_grad_f(u[i]);
    st_bf16x32((E*)g.C + o, v);
  } else if constexpr (EPI == EPI_ACC_RES_F32) {
    const float4* r = (const float4*)((const float*)g.res + (int64_t)m * g.ldr + n);
    float4* out = (float4*)((float*)g.C + o);
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const float4 a = r[q];
      out[q] = make_float4(v[4 * q] + a.x, v[4 * q + 1] + a.y, v[4 * q + 2] + a.z, v[4 * q + 3] + a.w);
    }
  } else {
    float4* out = (float4*)((float*)g.C + (int64_t)z * g.split_stride + o);
#pragma unroll
    for (int q = 0; q < 8; ++q) out[q] = make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
  }
}

template <int BN, int EPI>
__global__ void __launch_bounds__(TC_THREADS, 2)
    k_gemm_tc(const __grid_constant__ CUtensorMap tma_a, const __grid_constant__ CUtensorMap tma_b, const TcArgs args) {
  using Cf = TcCfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint64_t* full = (uint64_t*)(smem + Cf::STAGES * Cf::STAGE_BYTES);
  uint64_t* empty = full + Cf::STAGES;
  uint64_t* tfull = empty + Cf::STAGES;
  uint32_t* tmem_slot = (uint32_t*)(tfull + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * BN, m0 = blockIdx.y * TBM;
  const int kb0 = blockIdx.z * args.kb_per_split;
  const int kb1 = min(args.kb_total, kb0 + args.kb_per_split);
  const int nkb = kb1 - kb0;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < Cf::STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    mbar_init(tfull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tma_a) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tma_b) : "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(BN));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {                                   // ---------------- TMA producer
      for (int i = 0; i < nkb; ++i) {
        const int s = i % Cf::STAGES;
        if (i >= Cf::STAGES) mbar_wait(&empty[s], ((i / Cf::STAGES) - 1) & 1);
        uint8_t* sa = smem + s * Cf::STAGE_BYTES;
        uint8_t* sb = sa + Cf::A_BYTES;
        const int k = (kb0 + i) * TBK;
        mbar_expect_tx(&full[s], Cf::STAGE_BYTES);
        if (args.a_mn) {
          tma_load_2d(&tma_a, &full[s], sa, m0, k);
          tma_load_2d(&tma_a, &full[s], sa + 8192, m0 + 64, k);
        } else {
          tma_load_2d(&tma_a, &full[s], sa, k, m0);
        }
        if (args.b_mn) {
#pragma unroll
          for (int j = 0; j < BN / 64; ++j) tma_load_2d(&tma_b, &full[s], sb + 8192 * j, n0 + 64 * j, k);
        } else {
          tma_load_2d(&tma_b, &full[s], sb, k, n0);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {                                   // ---------------- MMA issuer
      const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)args.a_mn << 15) |
                             ((uint32_t)args.b_mn << 16) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(TBM >> 4) << 24);
      for (int i = 0; i < nkb; ++i) {
        const int s = i % Cf::STAGES;
        mbar_wait(&full[s], (i / Cf::STAGES) & 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t sa = smem_u32(smem + s * Cf::STAGE_BYTES);
        const uint32_t sb = sa + Cf::A_BYTES;
#pragma unroll
        for (int kk = 0; kk < TBK / 16; ++kk) {
          const uint64_t da = args.a_mn ? make_desc(sa + kk * 2048, 8192, 1024) : make_desc(sa + kk * 32, 16, 1024);
          const uint64_t db = args.b_mn ? make_desc(sb + kk * 2048, 8192, 1024) : make_desc(sb + kk * 32, 16, 1024);
          mma_bf16(tmem, da, db, idesc, (i > 0 || kk > 0) ? 1u : 0u);
        }
        mma_commit(&empty[s]);
      }
      mma_commit(tfull);
    }
  } else {                                             // ---------------- epilogue warps 2..5
    const int q = warp & 3;
    const int m = m0 + 32 * q + lane;
    mbar_wait(tfull, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const GemmArgs& g = args.g;
#pragma unroll 1
    for (int c = 0; c < BN / 32; ++c) {
      float v[32];
      tmem_ld32(tmem + ((uint32_t)(32 * q) << 16) + 32 * c, v);
      if (nkb <= 0) {                                  // empty split-K slice: exact zeros
#pragma unroll
        for (int i = 0; i < 32; ++i) v[i] = 0.f;
      }
      const int n = n0 + 32 * c;
      if (m < g.M) {
        if (n + 32 <= g.N) {
          epi_row32<EPI>(g, m, n, v);
        } else {
#pragma unroll
          for (int i = 0; i < 32; ++i)
            if (n + i < g.N) epilogue<__nv_bfloat16, EPI>(g, m, n + i, v[i]);
        }
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(BN));
  }
}


// ---------------------------------------------------------------------------
// Persistent variant: grid = #SMs; each CTA walks tiles t = blockIdx.x + i*gridDim.x
// (tile = (split, m-block, n-block), n fastest).  Two TMEM accumulators
// (2 x BN columns) let the epilogue of tile i overlap the MMAs of tile i+1; the
// smem ring continues across tiles.  8 epilogue warps: warp 2+e handles TMEM
// lane quarter e%4 and column half e/4.
// ---------------------------------------------------------------------------
constexpr int TP_EPI_WARPS = 8;
constexpr int TP_THREADS = 64 + 32 * TP_EPI_WARPS;

template <int BN>
struct TpCfg {
  static constexpr int STAGES = BN >= 256 ? 4 : 6;
  static constexpr int A_BYTES = TBM * TBK * 2;
  static constexpr int B_BYTES = BN * TBK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 512;
};

struct TpArgs {
  TcArgs t;
  int m_blocks, n_blocks, n_tiles;
};

template <int BN, int EPI>
__global__ void __launch_bounds__(TP_THREADS, 1)
    k_gemm_tcp(const __grid_constant__ CUtensorMap tma_a, const __grid_constant__ CUtensorMap tma_b, const TpArgs args) {
  using Cf = TpCfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint64_t* full = (uint64_t*)(smem + Cf::STAGES * Cf::STAGE_BYTES);
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
  const int per_split = args.m_blocks * args.n_blocks;

  if (warp == 0) {
    if (lane == 0) {                                   // ---------------- TMA producer
      int it = 0;
      for (int tile = blockIdx.x; tile < args.n_tiles; tile += gridDim.x) {
        const int z = tile / per_split, r = tile % per_split;
        const int m0 = (r / args.n_blocks) * TBM, n0 = (r % args.n_blocks) * BN;
        const int kb0 = z * ta.kb_per_split, kb1 = min(ta.kb_total, kb0 + ta.kb_per_split);
        for (int kb = kb0; kb < kb1; ++kb, ++it) {
          const int s = it % Cf::STAGES;
          if (it >= Cf::STAGES) mbar_wait(&empty[s], ((it / Cf::STAGES) - 1) & 1);
          uint8_t* sa = smem + s * Cf::STAGE_BYTES;
          uint8_t* sb = sa + Cf::A_BYTES;
          const int k = kb * TBK;
          mbar_expect_tx(&full[s], Cf::STAGE_BYTES);
          if (ta.a_mn) {
            tma_load_2d(&tma_a, &full[s], sa, m0, k);
            tma_load_2d(&tma_a, &full[s], sa + 8192, m0 + 64, k);
          } else {
            tma_load_2d(&tma_a, &full[s], sa, k, m0);
          }
          if (ta.b_mn) {
#pragma unroll
            for (int j = 0; j < BN / 64; ++j) tma_load_2d(&tma_b, &full[s], sb + 8192 * j, n0 + 64 * j, k);
          } else {
#pragma unroll
            for (int j = 0; j < (BN + 255) / 256; ++j)      // box rows <= 256
              tma_load_2d(&tma_b, &full[s], sb + j * 256 * 128, k, n0 + 256 * j);
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {                                   // ---------------- MMA issuer
      const uint32_t idesc = idesc_bf16(TBM, BN, ta.a_mn, ta.b_mn);
      int it = 0, local = 0;
      for (int tile = blockIdx.x; tile < args.n_tiles; tile += gridDim.x, ++local) {
        const int z = tile / per_split;
        const int kb0 = z * ta.kb_per_split, kb1 = min(ta.kb_total, kb0 + ta.kb_per_split);
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
    const int q = warp & 3;                            // TMEM lane quarter of this warp
    const int half = e >> 2;
    const GemmArgs& g = ta.g;
    int local = 0;
    for (int tile = blockIdx.x; tile < args.n_tiles; tile += gridDim.x, ++local) {
      const int z = tile / per_split, r = tile % per_split;
      const int m0 = (r / args.n_blocks) * TBM, n0 = (r % args.n_blocks) * BN;
      const int kb0 = z * ta.kb_per_split, kb1 = min(ta.kb_total, kb0 + ta.kb_per_split);
      const int acc = local & 1;
      const int m = m0 + 32 * q + lane;
      {  // pull this tile's epilogue inputs into L2 while the MMAs run
        const int nb = n0 + half * (BN / 2);
        if (m < g.M && nb < g.N) {
          const char* pa = nullptr;
          int bytes = 0;
          if constexpr (EPI == EPI_GELU_BWD) { pa = (const char*)((const __nv_bfloat16*)g.aux + (int64_t)m * g.ldx + nb); bytes = BN; }
          if constexpr (EPI == EPI_BIAS_DROP_RES) { pa = (const char*)((const __nv_bfloat16*)g.res + (int64_t)m * g.ldr + nb); bytes = BN; }
          if constexpr (EPI == EPI_ACC_RES_F32) { pa = (const char*)((const float*)g.res + (int64_t)m * g.ldr + nb); bytes = 2 * BN; }
          for (int o = 0; o < bytes; o += 128) asm volatile("prefetch.global.L2 [%0];" ::"l"(pa + o));
        }
      }
      mbar_wait(&tfull[acc], (local >> 1) & 1);
      __syncwarp();
      tc_fence_after();
#pragma unroll 1
      for (int c = half * (BN / 64); c < (half + 1) * (BN / 64); ++c) {
        float v[32];
        tmem_ld32(tmem + acc * BN + ((uint32_t)(32 * q) << 16) + 32 * c, v);
        if (kb1 <= kb0) {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = 0.f;
        }
        const int n = n0 + 32 * c;
        if (m < g.M) {
          if (n + 32 <= g.N) {
            epi_row32<EPI>(g, m, n, v, z);
          } else {
  #pragma unroll
          for (int i = 0; i < 32; ++i)
            if (n + i < g.N) epilogue<__nv_bfloat16, EPI>(g, m, n + i, v[i], z);
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&tempty[acc])) : "memory");
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(2 * BN));
  }
}

// ------------------------------------------------------------------ host --
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
  bool operator==(const MapKey& o) const {
    return ptr == o.ptr && inner == o.inner && outer == o.outer && stride == o.stride &&
           box_inner == o.box_inner && box_outer == o.box_outer;
  }
};
struct MapKeyHash {
  size_t operator()(const MapKey& k) const {
    size_t h = std::hash<const void*>()(k.ptr);
    for (uint64_t v : {k.inner, k.outer, k.stride, (uint64_t)k.box_inner << 32 | k.box_outer})
      h ^= std::hash<uint64_t>()(v) + 0x9e3779b97f4a7c15ull + (h << 6) + (h >> 2);
    return h;
  }
};

// 2D bf16 tensor [outer][inner] (inner contiguous), row stride in elements.
static bool make_map(CUtensorMap* out, const void* ptr, uint64_t inner, uint64_t outer, uint64_t stride_elems,
                     uint32_t box_inner, uint32_t box_outer) {
  static std::unordered_map<MapKey, CUtensorMap, MapKeyHash> cache;
  static std::mutex mu;
  MapKey key{ptr, inner, outer, stride_elems, box_inner, box_outer};
  std::lock_guard<std::mutex> lk(mu);
  auto it = cache.find(key);
  if (it != cache.end()) { *out = it->second; return true; }
  EncodeFn fn = encode_fn();
  if (!fn) return false;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {stride_elems * 2};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = fn(out, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(ptr), dims, strides, box, es,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return false;
  if (cache.size() > 8192) cache.clear();
  cache.emplace(key, *out);
  return true;
}

bool tc_map_bf16(CUtensorMap* out, const void* ptr, uint64_t inner, uint64_t outer, uint64_t stride_elems,
                 uint32_t box_inner, uint32_t box_outer) {
  return make_map(out, ptr, inner, outer, stride_elems, box_inner, box_outer);
}

template <int BN, int EPI>
static void launch_tc(const CUtensorMap& ma, const CUtensorMap& mb, const TcArgs& a, dim3 grid, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_gemm_tc<BN, EPI>, cudaFuncAttributeMaxDynamicSharedMemorySize, TcCfg<BN>::SMEM);
    attr = true;
  }
  k_gemm_tc<BN, EPI><<<grid, TC_THREADS, TcCfg<BN>::SMEM, st>>>(ma, mb, a);
}

template <int BN, int EPI>
static void launch_tcp(const CUtensorMap& ma, const CUtensorMap& mb, const TpArgs& a, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_gemm_tcp<BN, EPI>, cudaFuncAttributeMaxDynamicSharedMemorySize, TpCfg<BN>::SMEM);
    attr = true;
  }
  static int nsm = 0;
  if (!nsm) {
    int dev;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  }
  k_gemm_tcp<BN, EPI><<<std::min(nsm, a.n_tiles), TP_THREADS, TpCfg<BN>::SMEM, st>>>(ma, mb, a);
}

template <int BN>
static void dispatch_tcp(Epi epi, const CUtensorMap& ma, const CUtensorMap& mb, const TpArgs& a, cudaStream_t st) {
  switch (epi) {
    case EPI_STORE: launch_tcp<BN, EPI_STORE>(ma, mb, a, st); break;
    case EPI_BIAS: launch_tcp<BN, EPI_BIAS>(ma, mb, a, st); break;
    case EPI_BIAS_GELU: launch_tcp<BN, EPI_BIAS_GELU>(ma, mb, a, st); break;
    case EPI_BIAS_DROP_RES: launch_tcp<BN, EPI_BIAS_DROP_RES>(ma, mb, a, st); break;
    case EPI_GELU_BWD: launch_tcp<BN, EPI_GELU_BWD>(ma, mb, a, st); break;
    case EPI_ACC_RES_F32: launch_tcp<BN, EPI_ACC_RES_F32>(ma, mb, a, st); break;
    default: launch_tcp<BN, EPI_F32>(ma, mb, a, st); break;
  }
}

static int g_gemm_mode = 1;   // 0: one tile per CTA (k_gemm_tc); 1: persistent (k_gemm_tcp)
void set_gemm_mode(int m) { g_gemm_mode = m; }

bool tc_available() { return encode_fn() != nullptr; }

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
  // BN = 256 when N is a multiple of 256 and there are enough tiles to fill the SMs
  const int BN = (g_gemm_mode == 1 && g.N % 256 == 0 && m_blocks * (g.N / 256) * g.split >= 120) ? 256 : 128;
  CUtensorMap ma, mb;
  bool ok;
  if (a.a_mn) ok = make_map(&ma, g.A, g.M, g.K, g.a_sk, 64, 64);
  else ok = make_map(&ma, g.A, g.K, g.M, g.a_sm, 64, TBM);
  if (!ok) return false;
  if (a.b_mn) ok = make_map(&mb, g.B, g.N, g.K, g.b_sk, 64, 64);
  else ok = make_map(&mb, g.B, g.K, g.N, g.b_sn, 64, std::min(BN, 256));
  if (!ok) return false;
  if (g_gemm_mode == 1) {
    TpArgs p;
    p.t = a;
    p.m_blocks = m_blocks;
    p.n_blocks = (g.N + BN - 1) / BN;
    p.n_tiles = p.m_blocks * p.n_blocks * g.split;
    if (BN == 256) dispatch_tcp<256>(epi, ma, mb, p, st);
    else dispatch_tcp<128>(epi, ma, mb, p, st);
    return true;
  }
  constexpr int BN1 = 128;
  dim3 grid((g.N + BN1 - 1) / BN1, m_blocks, g.split);
  switch (epi) {
    case EPI_STORE: launch_tc<BN1, EPI_STORE>(ma, mb, a, grid, st); break;
    case EPI_BIAS: launch_tc<BN1, EPI_BIAS>(ma, mb, a, grid, st); break;
    case EPI_BIAS_GELU: launch_tc<BN1, EPI_BIAS_GELU>(ma, mb, a, grid, st); break;
    case EPI_BIAS_DROP_RES: launch_tc<BN1, EPI_BIAS_DROP_RES>(ma, mb, a, grid, st); break;
    case EPI_GELU_BWD: launch_tc<BN1, EPI_GELU_BWD>(ma, mb, a, grid, st); break;
    case EPI_ACC_RES_F32: launch_tc<BN1, EPI_ACC_RES_F32>(ma, mb, a, grid, st); break;
    default: launch_tc<BN1, EPI_F32>(ma, mb, a, grid, st); break;
  }
  return true;
}

}  // namespace mimose
