// Internal definitions shared by the host runtime and the sm_100a kernels.
// Nothing here is part of the public ABI (include/mimose.h).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <cstdlib>
#include <utility>

namespace mimose {

enum DType : int { DT_F32 = 0, DT_BF16 = 1 };

// Dropout site word (reading R-B): (rank << 16) | (layer << 4) | kind.
enum DropKind : uint32_t { KIND_ATTN_PROBS = 0, KIND_ATTN_OUT = 1, KIND_FFN_OUT = 2,
                           KIND_EMB = 3, KIND_HEAD = 4 };
constexpr uint32_t LAYER_NONE = 0xFFF;
inline uint32_t site_word(uint32_t kind, uint32_t layer, uint32_t rank) {
  return ((rank & 0xFFFFu) << 16) | ((layer & 0xFFFu) << 4) | (kind & 0xFu);
}

// Everything a dropout site needs on the device.
struct Drop {
  uint32_t seed_lo, seed_hi;
  uint32_t site, step;
  uint32_t thresh;   // keep iff r < thresh; thresh = floor((1-p) 2^32)
  float scale;       // 1/(1-p) rounded to fp32
  int enabled;       // p > 0
  // Philox round keys (k0 + r W0, k1 + r W1), r = 0..9, from (seed_lo, seed_hi) by
  // drop_set_keys: kernel-parameter constants, so the 10 rounds of every draw are
  // 2 IMAD.WIDE + 2 LOP3 each instead of re-deriving the key schedule per draw.
  uint32_t rk[20];
};
inline void drop_set_keys(Drop& d) {
  for (int r = 0; r < 10; ++r) {
    d.rk[2 * r] = d.seed_lo + (uint32_t)r * 0x9E3779B9u;
    d.rk[2 * r + 1] = d.seed_hi + (uint32_t)r * 0xBB67AE85u;
  }
}

// Programmatic dependent launch (PDL).  Every kernel of the library is launched
// with cudaLaunchAttributeProgrammaticStreamSerialization, so the next kernel in
// the stream is scheduled as soon as every CTA of the running one has started;
// it runs its prologue (barrier init, TMEM alloc, tensor-map prefetch) and then
// blocks in griddepcontrol.wait until the previous grid has completed and its
// memory is visible.  Every kernel calls pdl_enter() (or pdl_trigger() +
// pdl_wait() around a prologue that touches no global memory) before its first
// global access, so the stream order of all reads and writes is unchanged: the
// results are bitwise those of plain launches.  MIMOSE_PDL=0 disables it.
inline bool pdl_enabled() {
  static const int v = [] {
    const char* e = std::getenv("MIMOSE_PDL");
    return e ? std::atoi(e) : 1;
  }();
  return v != 0;
}
template <typename... KArgs, typename... Args>
inline cudaError_t launch_k(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                            Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, k, std::forward<Args>(args)...);
}

// Same, with a thread-block cluster of `cluster_x` CTAs along x.
template <typename... KArgs, typename... Args>
inline cudaError_t launch_kc(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, int cluster_x,
                             Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = cluster_x;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, k, std::forward<Args>(args)...);
}

constexpr int NPART = 296;   // fixed reduction-partial count (DESIGN "Memory model")

#if defined(__CUDACC__)
#define MDEV __device__ __forceinline__

MDEV void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
MDEV void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
MDEV void pdl_enter() {
  pdl_trigger();
  pdl_wait();
}

// Philox4x32-10, Salmon et al. SC'11 (same constants as Random123), with the
// key schedule k_r = k + r (0x9E3779B9, 0xBB67AE85) precomputed in Drop::rk.
MDEV uint4 philox4x32_10_rk(uint4 c, const uint32_t (&rk)[20]) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    uint32_t hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
    uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
    c = make_uint4(hi1 ^ c.y ^ rk[2 * r], lo1, hi0 ^ c.w ^ rk[2 * r + 1], lo0);
  }
  return c;
}

// Four random words for elements 4n..4n+3 of a site.
MDEV uint4 drop_words(const Drop& d, uint64_t n) {
  return philox4x32_10_rk(make_uint4((uint32_t)n, (uint32_t)(n >> 32), d.site, d.step), d.rk);
}
MDEV uint32_t word_of(uint4 w, int lane) {
  return lane == 0 ? w.x : lane == 1 ? w.y : lane == 2 ? w.z : w.w;
}
// Scaled keep factor (0 or 1/(1-p)) of element e.
MDEV float drop_factor(const Drop& d, uint64_t e) {
  if (!d.enabled) return 1.0f;
  uint4 w = drop_words(d, e >> 2);
  return word_of(w, (int)(e & 3)) < d.thresh ? d.scale : 0.0f;
}
// Factors for the 4 aligned elements 4n..4n+3.
MDEV float4 drop_factor4(const Drop& d, uint64_t n) {
  if (!d.enabled) return make_float4(1.f, 1.f, 1.f, 1.f);
  uint4 w = drop_words(d, n);
  return make_float4(w.x < d.thresh ? d.scale : 0.f, w.y < d.thresh ? d.scale : 0.f,
                     w.z < d.thresh ? d.scale : 0.f, w.w < d.thresh ? d.scale : 0.f);
}

MDEV float ldf(const float* p) { return *p; }
MDEV float ldf(const __nv_bfloat16* p) { return __bfloat162float(*p); }
MDEV void stf(float* p, float v) { *p = v; }
MDEV void stf(__nv_bfloat16* p, float v) { *p = __float2bfloat16_rn(v); }
// Round a value to the storage type and back (so stats are taken on stored values).
MDEV float rnd(float v, const float*) { return v; }
MDEV float rnd(float v, const __nv_bfloat16*) { return __bfloat162float(__float2bfloat16_rn(v)); }

MDEV int cdiv_dev(int a, int b) { return (a + b - 1) / b; }

MDEV float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
MDEV float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
#endif

}  // namespace mimose
