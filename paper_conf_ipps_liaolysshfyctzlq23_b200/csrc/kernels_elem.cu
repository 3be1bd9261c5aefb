// HBM-bound kernels of the Mimose step on sm_100a: embedding, LayerNorm
// forward/backward (fused with dropout and bias-gradient partials), column
// sums, deterministic keyed row sums (embedding gradient), task heads, AdamW.
//
// Determinism: no floating-point atomics anywhere;
// every reduction has a fixed assignment of rows to partials and a fixed
// summation order, so recompute and plan changes cannot change a
// single bit of the gradients.
#include "kernels.h"

#include <atomic>
#include <cmath>

namespace mimose {

static std::atomic<long long> g_launches{0};
void note_launch(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }
int64_t kernel_launch_count() { return g_launches.load(); }

template <typename F>
static void dispatch(DType dt, F f) {
  if (dt == DT_F32) f((float*)nullptr); else f((__nv_bfloat16*)nullptr);
}

static inline int cdiv(int64_t a, int64_t b) { return (int)((a + b - 1) / b); }

// ===================================================================== LN ===
// Vector helpers: 8 consecutive elements (16 B of bf16 / 32 B of fp32).
MDEV void ld8(const float* p, float* v) {
  const float4 a = ((const float4*)p)[0], b = ((const float4*)p)[1];
  v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}
MDEV void ld8(const __nv_bfloat16* p, float* v) {
  const uint4 u = *(const uint4*)p;
  const __nv_bfloat162* h = (const __nv_bfloat162*)&u;
#pragma unroll
  for (int i = 0; i < 4; ++i) { const float2 f = __bfloat1622float2(h[i]); v[2 * i] = f.x; v[2 * i + 1] = f.y; }
}
MDEV void st8(float* p, const float* v) {
  ((float4*)p)[0] = make_float4(v[0], v[1], v[2], v[3]);
  ((float4*)p)[1] = make_float4(v[4], v[5], v[6], v[7]);
}
MDEV void st8(__nv_bfloat16* p, const float* v) {
  uint4 u;
  __nv_bfloat162* h = (__nv_bfloat162*)&u;
#pragma unroll
  for (int i = 0; i < 4; ++i) h[i] = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);
  *(uint4*)p = u;
}
MDEV void drop8(const Drop& d, uint64_t e, float* f) {   // e multiple of 8
  const float4 a = drop_factor4(d, e >> 2), b = drop_factor4(d, (e >> 2) + 1);
  f[0] = a.x; f[1] = a.y; f[2] = a.z; f[3] = a.w; f[4] = b.x; f[5] = b.y; f[6] = b.z; f[7] = b.w;
}

// warp per row; lane owns 8-column chunks j = lane + 32 k (H % 8 == 0, H <= 1024)
template <typename E>
__global__ void __launch_bounds__(256) k_ln_fwd(const float* __restrict__ z, const E* __restrict__ g,
                                                const E* __restrict__ b, E* __restrict__ y,
                                                float2* __restrict__ st, int T, int H, float eps) {
  pdl_enter();
  const int row = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (row >= T) return;
  const int nch = H >> 3;
  const float* zr = z + (int64_t)row * H;
  float v[4][8];
  float s = 0.f;
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int j = lane + 32 * k;
    if (j < nch) {
      ld8(zr + 8 * j, v[k]);
#pragma unroll
      for (int i = 0; i < 8; ++i) s += v[k][i];
    }
  }
  const float mu = warp_sum(s) / (float)H;
  float q = 0.f;
#pragma unroll
  for (int k = 0; k < 4; ++k)
    if (lane + 32 * k < nch)
#pragma unroll
      for (int i = 0; i < 8; ++i) { const float d = v[k][i] - mu; q += d * d; }
  const float rstd = rsqrtf(warp_sum(q) / (float)H + eps);
  if (lane == 0) st[row] = make_float2(mu, rstd);
  if (y) {
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int j = lane + 32 * k;
      if (j < nch) {
        float gv[8], bv[8], o[8];
        ld8(g + 8 * j, gv);
        ld8(b + 8 * j, bv);
#pragma unroll
        for (int i = 0; i < 8; ++i) o[i] = (v[k][i] - mu) * rstd * gv[i] + bv[i];
        st8(y + (int64_t)row * H + 8 * j, o);
      }
    }
  }
}

void ln_fwd(DType dt, const float* z, const void* g, const void* b, void* y, float2* st, int T,
            int H, float eps, cudaStream_t s) {
  note_launch(1);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_ln_fwd<E>, cdiv(T, 8), 256, 0, s, z, (const E*)g, (const E*)b, (E*)y, st, T, H, eps);
  });
}

// NPART CTAs x 4 warps; warp w of CTA p owns rows r = p*4 + w + k*NPART*4 (fixed).
// Per-lane register partials of dgamma, dbeta, dbias over the warp's rows, then a
// fixed-order reduction over the 4 warps through shared memory.  KCH = 8-column
// chunks per lane (ceil(H / 256)); gamma is read from shared memory.  For
// H <= 768 the next row's loads are issued before the current row is processed.
// <= 255 registers x 128 threads: 2 CTAs / SM, so all NPART CTAs are resident at once.
constexpr int LNB_WARPS = 4;
template <typename E, int KCH>
__global__ void __launch_bounds__(32 * LNB_WARPS, 2) k_ln_bwd(const float* dy, Drop premask,
                                                              const float* __restrict__ z,
                                                              const float2* __restrict__ st, const E* __restrict__ g,
                                                              float* dz, E* __restrict__ dtout, Drop mask,
                                                              float* __restrict__ pg, float* __restrict__ pb,
                                                              float* __restrict__ pbias, int T, int H,
                                                              const float* res) {
  pdl_enter();
  extern __shared__ float sm[];            // [LNB_WARPS][3][H] partials, then gamma [H]
  float* sgam = sm + (size_t)LNB_WARPS * 3 * H;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nch = H >> 3;
  const float invH = 1.0f / (float)H;
  for (int c = threadIdx.x; c < H; c += blockDim.x) sgam[c] = ldf(g + c);
  __syncthreads();
  float ag[KCH][8], ab[KCH][8], at[KCH][8];
#pragma unroll
  for (int k = 0; k < KCH; ++k)
#pragma unroll
    for (int i = 0; i < 8; ++i) { ag[k][i] = 0.f; ab[k][i] = 0.f; at[k][i] = 0.f; }
  // software pipeline: the next row's dy, z and statistics are loaded before the
  // current row is processed (two rows of loads in flight per warp)
  constexpr int STRIDE = NPART * LNB_WARPS;
  float dyn[KCH][8], xn[KCH][8];
  float2 msn = make_float2(0.f, 0.f);
  auto load_row = [&](int rr) {
    msn = st[rr];
#pragma unroll
    for (int k = 0; k < KCH; ++k) {
      const int j = lane + 32 * k;
      if (j < nch) {
        ld8(dy + (int64_t)rr * H + 8 * j, dyn[k]);
        ld8(z + (int64_t)rr * H + 8 * j, xn[k]);
      }
    }
  };
  constexpr bool PF = KCH <= 3;        // H <= 768: registers allow the prefetch without spills
  if (PF && blockIdx.x * LNB_WARPS + warp < T) load_row(blockIdx.x * LNB_WARPS + warp);
  for (int row = blockIdx.x * LNB_WARPS + warp; row < T; row += STRIDE) {
    if (!PF) load_row(row);
    const float2 ms = msn;
    float dyv[KCH][8], xh[KCH][8];
#pragma unroll
    for (int k = 0; k < KCH; ++k)
#pragma unroll
      for (int i = 0; i < 8; ++i) { dyv[k][i] = dyn[k][i]; xh[k][i] = xn[k][i]; }
    if (PF && row + STRIDE < T) load_row(row + STRIDE);
    float s1 = 0.f, s2 = 0.f;
#pragma unroll
    for (int k = 0; k < KCH; ++k) {
      const int j = lane + 32 * k;
      if (j < nch) {
        if (premask.enabled) {
          float f[8];
          drop8(premask, (uint64_t)row * H + 8 * j, f);
#pragma unroll
          for (int i = 0; i < 8; ++i) dyv[k][i] *= f[i];
        }
        float gv[8];
        ld8(sgam + 8 * j, gv);
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          xh[k][i] = (xh[k][i] - ms.x) * ms.y;
          const float dxh = dyv[k][i] * gv[i];
          s1 += dxh;
          s2 += dxh * xh[k][i];
        }
      }
    }
    s1 = warp_sum(s1) * invH;
    s2 = warp_sum(s2) * invH;
#pragma unroll
    for (int k = 0; k < KCH; ++k) {
      const int j = lane + 32 * k;
      if (j < nch) {
        float o[8], gv[8];
        ld8(sgam + 8 * j, gv);
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          o[i] = ms.y * (dyv[k][i] * gv[i] - s1 - xh[k][i] * s2);
          ag[k][i] += dyv[k][i] * xh[k][i];
          ab[k][i] += dyv[k][i];
        }
        if (res) {                                    // pre-LN: residual gradient joins here
          float rv[8];
          ld8(res + (int64_t)row * H + 8 * j, rv);
#pragma unroll
          for (int i = 0; i < 8; ++i) o[i] += rv[i];
        }
        st8(dz + (int64_t)row * H + 8 * j, o);
        if (dtout) {
          float f[8];
          drop8(mask, (uint64_t)row * H + 8 * j, f);
#pragma unroll
          for (int i = 0; i < 8; ++i) o[i] = rnd(o[i] * f[i], dtout);   // the stored value
          st8(dtout + (int64_t)row * H + 8 * j, o);
#pragma unroll
          for (int i = 0; i < 8; ++i) at[k][i] += o[i];
        }
      }
    }
  }
  // fixed-order cross-warp reduction: smem [LNB_WARPS][3][H]
#pragma unroll
  for (int k = 0; k < KCH; ++k) {
    const int j = lane + 32 * k;
    if (j < nch) {
      float* base = sm + (size_t)warp * 3 * H + 8 * j;
      st8(base, ag[k]);
      st8(base + H, ab[k]);
      st8(base + 2 * H, at[k]);
    }
  }
  __syncthreads();
  for (int c = threadIdx.x; c < H; c += blockDim.x) {
    float sg = 0.f, sb = 0.f, sbias = 0.f;
    for (int w = 0; w < LNB_WARPS; ++w) {
      const float* base = sm + (size_t)w * 3 * H;
      sg += base[c]; sb += base[H + c]; sbias += base[2 * H + c];
    }
    pg[(size_t)blockIdx.x * H + c] = sg;
    pb[(size_t)blockIdx.x * H + c] = sb;
    if (pbias) pbias[(size_t)blockIdx.x * H + c] = sbias;
  }
}

template <typename E, int KCH>
static void launch_ln_bwd(const float* dy, Drop premask, const float* z, const float2* st, const void* g, float* dz,
                          void* dtout, Drop mask, float* pg, float* pb, float* pbias, int T, int H, cudaStream_t s,
                          const float* res) {
  const size_t smem = (size_t)(LNB_WARPS * 3 + 1) * H * sizeof(float);
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_ln_bwd<E, KCH>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (LNB_WARPS * 3 + 1) * 1024 * 4);
    attr = true;
  }
  launch_k(k_ln_bwd<E, KCH>, NPART, 32 * LNB_WARPS, smem, s, dy, premask, z, st, (const E*)g, dz, (E*)dtout, mask,
           pg, pb, pbias, T, H, res);
}

void ln_bwd(DType dt, const float* dy, Drop premask, const float* z, const float2* st, const void* g,
            float* dz, void* dtout, Drop mask, float* pg, float* pb, float* pbias, int T, int H,
            cudaStream_t s, const float* res) {
  note_launch(1);
  const int kch = (H / 8 + 31) / 32;
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    if (kch <= 1) launch_ln_bwd<E, 1>(dy, premask, z, st, g, dz, dtout, mask, pg, pb, pbias, T, H, s, res);
    else if (kch == 2) launch_ln_bwd<E, 2>(dy, premask, z, st, g, dz, dtout, mask, pg, pb, pbias, T, H, s, res);
    else if (kch == 3) launch_ln_bwd<E, 3>(dy, premask, z, st, g, dz, dtout, mask, pg, pb, pbias, T, H, s, res);
    else launch_ln_bwd<E, 4>(dy, premask, z, st, g, dz, dtout, mask, pg, pb, pbias, T, H, s, res);
  });
}

// out[c] = sum_{p < rows} part[p*ld + c] in a fixed order: warp w sums rows
// p = w, w+8, ... ascending; warp 0 then adds the 8 warp sums in order w = 0..7.
// blockIdx.y selects one of up to 3 (part, out) pairs.
struct RedJob { const float* part; float* out; };
struct RedJobs { RedJob j[3]; };
__global__ void __launch_bounds__(1024) k_reduce_rows(RedJobs jobs, int rows, int64_t ld, int n) {
  pdl_enter();
  __shared__ float sw[32][33];
  const RedJob jb = jobs.j[blockIdx.y];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int c = blockIdx.x * 32 + lane;
  float acc = 0.f;
  if (c < n && rows <= 320) {            // NPART rows: all <= 10 loads of a lane in flight at once
    float v[10];
#pragma unroll
    for (int i = 0; i < 10; ++i) v[i] = warp + 32 * i < rows ? jb.part[(int64_t)(warp + 32 * i) * ld + c] : 0.f;
#pragma unroll
    for (int i = 0; i < 10; ++i)
      if (warp + 32 * i < rows) acc += v[i];   // row order, as below
  } else if (c < n) {
    int p = warp;
    for (; p + 96 < rows; p += 128) {     // 4 independent loads in flight, added in row order
      const float v0 = jb.part[(int64_t)p * ld + c], v1 = jb.part[(int64_t)(p + 32) * ld + c];
      const float v2 = jb.part[(int64_t)(p + 64) * ld + c], v3 = jb.part[(int64_t)(p + 96) * ld + c];
      acc += v0; acc += v1; acc += v2; acc += v3;
    }
    for (; p < rows; p += 32) acc += jb.part[(int64_t)p * ld + c];
  }
  sw[warp][lane] = acc;
  __syncthreads();
  if (warp == 0 && c < n) {
    float t = 0.f;
#pragma unroll
    for (int w = 0; w < 32; ++w) t += sw[w][lane];
    jb.out[c] = t;
  }
}
void reduce_rows3(const float* p0, float* o0, const float* p1, float* o1, const float* p2, float* o2, int rows,
                  int64_t ld, int n, cudaStream_t s) {
  note_launch(1);
  RedJobs jobs{{{p0, o0}, {p1, o1}, {p2, o2}}};
  const int nj = p2 ? 3 : p1 ? 2 : 1;
  launch_k(k_reduce_rows, dim3(cdiv(n, 32), nj), 1024, 0, s, jobs, rows, ld, n);
}
void reduce_partials(const float* part, int64_t ld, int n, float* out, cudaStream_t s) {
  reduce_rows3(part, out, nullptr, nullptr, nullptr, nullptr, NPART, ld, n, s);
}

__global__ void k_splitk_reduce(const float* __restrict__ part, int splits, int64_t n, float* __restrict__ out) {
  pdl_enter();
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * 4; i < n; i += (int64_t)gridDim.x * blockDim.x * 4) {
    float4 s = ((const float4*)(part + i))[0];
    for (int k = 1; k < splits; ++k) {
      const float4 v = ((const float4*)(part + k * n + i))[0];
      s.x += v.x; s.y += v.y; s.z += v.z; s.w += v.w;
    }
    *(float4*)(out + i) = s;
  }
}
void splitk_reduce(const float* part, int splits, int64_t n, float* out, cudaStream_t s) {
  note_launch(1);
  launch_k(k_splitk_reduce, 592, 256, 0, s, part, splits, n, out);
}

// column sums of X [T, N] (E): CTA (cx, p) owns rows p, p+NPART, ... and columns
// [2048 cx, 2048 cx + 2048); a thread owns 8 consecutive columns.
template <typename E>
__global__ void __launch_bounds__(256) k_colsum(const E* __restrict__ X, int T, int N, float* __restrict__ part) {
  pdl_enter();
  const int c = blockIdx.x * 2048 + threadIdx.x * 8;
  if (c >= N) return;
  float acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
  int r = blockIdx.y;
  for (; r + 3 * NPART < T; r += 4 * NPART) {   // 4 rows of loads in flight, added in row order
    float v[4][8];
#pragma unroll
    for (int k = 0; k < 4; ++k) ld8(X + (int64_t)(r + k * NPART) * N + c, v[k]);
#pragma unroll
    for (int k = 0; k < 4; ++k)
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += v[k][i];
  }
  for (; r < T; r += NPART) {
    float v[8];
    ld8(X + (int64_t)r * N + c, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] += v[i];
  }
  st8(part + (int64_t)blockIdx.y * N + c, acc);
}
void colsum(DType dt, const void* X, int T, int N, float* part, cudaStream_t s) {
  note_launch(1);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_colsum<E>, dim3(cdiv(N, 2048), NPART), 256, 0, s, (const E*)X, T, N, part);
  });
}

// out(E) = in(f32) * mask, with column-sum partials of the stored values.
template <typename E>
__global__ void __launch_bounds__(256) k_drop_cast_colsum(const float* __restrict__ in, Drop mask, E* __restrict__ out,
                                                          int T, int N, float* __restrict__ part) {
  pdl_enter();
  const int c = blockIdx.x * 2048 + threadIdx.x * 8;
  if (c >= N) return;
  float acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
  for (int r = blockIdx.y; r < T; r += NPART) {
    float v[8], f[8];
    ld8(in + (int64_t)r * N + c, v);
    drop8(mask, (uint64_t)r * N + c, f);
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = rnd(v[i] * f[i], out);
    st8(out + (int64_t)r * N + c, v);
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] += v[i];
  }
  st8(part + (int64_t)blockIdx.y * N + c, acc);
}
void drop_cast_colsum(DType dt, const float* in, Drop mask, void* out, int T, int N, float* part, cudaStream_t s) {
  note_launch(1);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_drop_cast_colsum<E>, dim3(cdiv(N, 2048), NPART), 256, 0, s, in, mask, (E*)out, T, N, part);
  });
}

__global__ void k_drop_f32(const float* __restrict__ in, Drop mask, float* __restrict__ out, int64_t n) {
  pdl_enter();
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * 8; i < n; i += (int64_t)gridDim.x * blockDim.x * 8) {
    float v[8], f[8];
    ld8(in + i, v);
    drop8(mask, (uint64_t)i, f);
#pragma unroll
    for (int k = 0; k < 8; ++k) v[k] *= f[k];
    st8(out + i, v);
  }
}
void drop_f32(const float* in, Drop mask, float* out, int64_t n, cudaStream_t s) {
  note_launch(1);
  launch_k(k_drop_f32, 592, 256, 0, s, in, mask, out, n);
}

// ============================================================== embedding ===

template <typename E>
__global__ void __launch_bounds__(256) k_embed_fwd(const int32_t* __restrict__ ids, const int32_t* __restrict__ tt,
                                                   const E* __restrict__ Ww, const E* __restrict__ Wp,
                                                   const E* __restrict__ Wt, const E* __restrict__ g,
                                                   const E* __restrict__ b, float* __restrict__ z0,
                                                   float2* __restrict__ st0, E* __restrict__ x1, int T,
                                                   int S, int H, int pos_offset, float eps, Drop drop) {
  pdl_enter();
  const int t = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (t >= T) return;
  const int s = t % S;
  const E* w = Ww + (int64_t)ids[t] * H;
  const E* p = Wp + (int64_t)(pos_offset + s) * H;
  const E* ty = Wt + (int64_t)tt[t] * H;
  const int nv = H >> 5;
  float v[32];
  float sum = 0.f;
#pragma unroll
  for (int k = 0; k < 32; ++k)
    if (k < nv) {
      const int c = lane + 32 * k;
      v[k] = ldf(w + c) + ldf(p + c) + ldf(ty + c);
      z0[(int64_t)t * H + c] = v[k];
      sum += v[k];
    }
  const float mu = warp_sum(sum) / (float)H;
  float q = 0.f;
#pragma unroll
  for (int k = 0; k < 32; ++k)
    if (k < nv) { const float d = v[k] - mu; q += d * d; }
  const float rstd = rsqrtf(warp_sum(q) / (float)H + eps);
  if (lane == 0) st0[t] = make_float2(mu, rstd);
#pragma unroll
  for (int k = 0; k < 32; ++k)
    if (k < nv) {
      const int c = lane + 32 * k;
      const float o = ((v[k] - mu) * rstd * ldf(g + c) + ldf(b + c)) *
                      drop_factor(drop, (uint64_t)t * H + c);
      stf(x1 + (int64_t)t * H + c, o);
    }
}

void embed_fwd(DType dt, const int32_t* ids, const int32_t* tt, const void* Ww, const void* Wp,
               const void* Wt, const void* g, const void* b, float* z0, float2* st0, void* x1, int B,
               int S, int H, int pos_offset, float eps, Drop drop, cudaStream_t s) {
  const int T = B * S;
  note_launch(1);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_embed_fwd<E>, cdiv(T, 8), 256, 0, s, ids, tt, (const E*)Ww, (const E*)Wp, (const E*)Wt,
                                              (const E*)g, (const E*)b, z0, st0, (E*)x1, T, S, H,
                                              pos_offset, eps, drop);
  });
}

// partials [NPART][TV*H]; CTA p owns rows p, p+NPART, ...
__global__ void __launch_bounds__(256) k_type_part(const float* __restrict__ dz0, const int32_t* __restrict__ tt,
                                                   int T, int H, int TV, float* __restrict__ part) {
  pdl_enter();
  float acc[4][4];
#pragma unroll
  for (int k = 0; k < 4; ++k)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[k][j] = 0.f;
  for (int r = blockIdx.x; r < T; r += NPART) {
    const int key = tt[r];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int c = threadIdx.x + 256 * j;
      if (c < H) {
        const float v = dz0[(int64_t)r * H + c];
#pragma unroll
        for (int k = 0; k < 4; ++k) acc[k][j] += (k == key) ? v : 0.f;
      }
    }
  }
  for (int k = 0; k < TV; ++k)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int c = threadIdx.x + 256 * j;
      if (c < H) part[(int64_t)blockIdx.x * TV * H + (int64_t)k * H + c] = acc[k][j];
    }
}
void type_grad(const float* dz0, const int32_t* tt, int T, int H, int TV, float* part, float* dWt, cudaStream_t s) {
  note_launch(1);
  launch_k(k_type_part, NPART, 256, 0, s, dz0, tt, T, H, TV, part);
  reduce_partials(part, (int64_t)TV * H, TV * H, dWt, s);
}

template <typename E>
__global__ void k_embed_fwd_pre(const int32_t* __restrict__ ids, const E* __restrict__ Ww, const E* __restrict__ Wp,
                                float* __restrict__ x1, int T, int S, int H, int pos_offset, Drop drop) {
  pdl_enter();
  const int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * 8;
  if (i >= (int64_t)T * H) return;
  const int t = (int)(i / H), c = (int)(i % H);
  float w[8], p[8], f[8];
  ld8(Ww + (int64_t)ids[t] * H + c, w);
  ld8(Wp + (int64_t)(pos_offset + t % S) * H + c, p);
  drop8(drop, (uint64_t)i, f);
#pragma unroll
  for (int k = 0; k < 8; ++k) w[k] = (w[k] + p[k]) * f[k];
  st8(x1 + i, w);
}
void embed_fwd_pre(DType dt, const int32_t* ids, const void* Ww, const void* Wp, float* x1, int B, int S, int H,
                   int pos_offset, Drop drop, cudaStream_t s) {
  note_launch(1);
  const int T = B * S;
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_embed_fwd_pre<E>, cdiv((int64_t)T * H / 8, 256), 256, 0, s, ids, (const E*)Ww, (const E*)Wp, x1, T, S, H,
                                                                     pos_offset, drop);
  });
}

__global__ void k_pos_grad(const float* __restrict__ dz0, int B, int S, int H, int pos_offset,
                           float* __restrict__ dWp, int accumulate) {
  pdl_enter();
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= (int64_t)S * H) return;
  const int s = (int)(i / H), c = (int)(i % H);
  float acc = 0.f;
  for (int b = 0; b < B; ++b) acc += dz0[((int64_t)b * S + s) * H + c];
  float* o = dWp + (int64_t)(pos_offset + s) * H + c;
  *o = accumulate ? *o + acc : acc;
}
void pos_grad(const float* dz0, int B, int S, int H, int pos_offset, float* dWp, cudaStream_t s, bool accumulate) {
  note_launch(1);
  launch_k(k_pos_grad, cdiv((int64_t)S * H, 256), 256, 0, s, dz0, B, S, H, pos_offset, dWp, accumulate ? 1 : 0);
}

// ---- stable LSD radix sort of (key, token) pairs, 8-bit digits, 1024-key tiles ----
__global__ void __launch_bounds__(1024) k_rs_hist(const int32_t* __restrict__ keys, int T, int shift,
                                                  int ntiles, int32_t* __restrict__ hist) {
  pdl_enter();
  __shared__ int h[256];
  if (threadIdx.x < 256) h[threadIdx.x] = 0;
  __syncthreads();
  const int i = blockIdx.x * 1024 + threadIdx.x;
  if (i < T) atomicAdd(&h[(keys[i] >> shift) & 0xFF], 1);   // integer counts: order-free
  __syncthreads();
  if (threadIdx.x < 256) hist[threadIdx.x * ntiles + blockIdx.x] = h[threadIdx.x];
}

// exclusive scan of n <= 8192 ints, one CTA of 1024 threads, 8 per thread
__global__ void __launch_bounds__(1024) k_rs_scan(int32_t* __restrict__ a, int n) {
  pdl_enter();
  __shared__ int ws[32];
  int v[8], s = 0;
  const int base = threadIdx.x * 8;
#pragma unroll
  for (int j = 0; j < 8; ++j) { v[j] = base + j < n ? a[base + j] : 0; s += v[j]; }
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  int inc = s;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) { const int t = __shfl_up_sync(0xffffffffu, inc, o); if (lane >= o) inc += t; }
  if (lane == 31) ws[warp] = inc;
  __syncthreads();
  if (warp == 0) {
    int w = ws[lane], wi = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) { const int t = __shfl_up_sync(0xffffffffu, wi, o); if (lane >= o) wi += t; }
    ws[lane] = wi - w;
  }
  __syncthreads();
  int run = ws[warp] + inc - s;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    if (base + j < n) a[base + j] = run;
    run += v[j];
  }
}

__global__ void __launch_bounds__(1024) k_rs_scatter(const int32_t* __restrict__ kin, const int32_t* __restrict__ vin,
                                                     int T, int shift, int ntiles, const int32_t* __restrict__ off,
                                                     int32_t* __restrict__ kout, int32_t* __restrict__ vout) {
  pdl_enter();
  __shared__ int wc[32][257];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 32 * 257; i += 1024) (&wc[0][0])[i] = 0;
  __syncthreads();
  const int i = blockIdx.x * 1024 + threadIdx.x;
  const bool valid = i < T;
  const int key = valid ? kin[i] : 0;
  const int val = valid ? (vin ? vin[i] : i) : 0;
  const int d = valid ? (key >> shift) & 0xFF : 256 + lane;
  const unsigned peers = __match_any_sync(0xffffffffu, d);
  const int rank = __popc(peers & ((1u << lane) - 1u));
  if (valid && rank == 0) wc[warp][d] = __popc(peers);
  __syncthreads();
  if (threadIdx.x < 256) {
    int run = 0;
    for (int w = 0; w < 32; ++w) { const int c = wc[w][threadIdx.x]; wc[w][threadIdx.x] = run; run += c; }
  }
  __syncthreads();
  if (valid) {
    const int pos = off[d * ntiles + blockIdx.x] + wc[warp][d] + rank;
    kout[pos] = key;
    vout[pos] = val;
  }
}

// piece sums: warp per 32 sorted positions; a piece = a run of equal keys inside the chunk.
// The piece sum overwrites the X row of the piece's first token (read-before-write, same warp).
// Keys equal to `skip` (the pad id) are ignored.  The rows of 4 consecutive
// positions are loaded together (4 independent row loads in flight instead of
// one row per iteration) and then added in position order: the same sums.
__global__ void __launch_bounds__(256) k_piece_sum(const int32_t* __restrict__ keys, const int32_t* __restrict__ tok,
                                                   float* X, int T, int H, int skip) {
  pdl_enter();
  const int chunk = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  const int r0 = chunk * 32;
  if (r0 >= T) return;
  const int r1 = min(r0 + 32, T);
  const int nv = H >> 5;              // <= 32
  float acc[32];
#pragma unroll
  for (int j = 0; j < 32; ++j) acc[j] = 0.f;
  int start = r0;
  for (int rb = r0; rb < r1; rb += 4) {
    int kq[4];
    float v[4][32];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int r = rb + u;
      kq[u] = r < r1 ? keys[r] : skip;
      const float* xr = X + (int64_t)(r < r1 ? tok[r] : 0) * H;
#pragma unroll
      for (int j = 0; j < 32; ++j) v[u][j] = (kq[u] != skip && j < nv) ? xr[lane + 32 * j] : 0.f;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int r = rb + u;
      if (r >= r1) break;
      const int key = kq[u];
      if (key != skip) {
#pragma unroll
        for (int j = 0; j < 32; ++j) acc[j] += v[u][j];
      }
      if (r + 1 == r1 || keys[r + 1] != key) {
        if (key != skip) {
          float* dst = X + (int64_t)tok[start] * H;
#pragma unroll
          for (int j = 0; j < 32; ++j)
            if (j < nv) dst[lane + 32 * j] = acc[j];
        }
#pragma unroll
        for (int j = 0; j < 32; ++j) acc[j] = 0.f;
        start = r + 1;
      }
    }
  }
}

// segment sums: warp per sorted position that starts a run of equal keys.
__global__ void __launch_bounds__(256) k_segment_sum(const int32_t* __restrict__ keys, const int32_t* __restrict__ tok,
                                                     const float* __restrict__ X, int T, int H, float* __restrict__ out,
                                                     int skip, int accumulate) {
  pdl_enter();
  const int r = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (r >= T) return;
  const int key = keys[r];
  if (key == skip || (r > 0 && keys[r - 1] == key)) return;
  int end = T;                                        // warp-parallel search for the run end
  for (int base = r + 1; base < T; base += 32) {
    const int i = base + lane;
    const unsigned diff = __ballot_sync(0xffffffffu, i < T && keys[i] != key);
    if (diff) { end = base + __ffs(diff) - 1; break; }
  }
  const int nv = H >> 5;
  float acc[32];
  const float* x0 = X + (int64_t)tok[r] * H;
#pragma unroll
  for (int j = 0; j < 32; ++j) acc[j] = j < nv ? x0[lane + 32 * j] : 0.f;
  for (int q = (r / 32 + 1) * 32; q < end; q += 32) {
    const float* xq = X + (int64_t)tok[q] * H;
    float v[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) v[j] = j < nv ? xq[lane + 32 * j] : 0.f;
#pragma unroll
    for (int j = 0; j < 32; ++j) acc[j] += v[j];
  }
#pragma unroll
  for (int j = 0; j < 32; ++j)
    if (j < nv) {
      float* o = out + (int64_t)key * H + lane + 32 * j;
      *o = accumulate ? *o + acc[j] : acc[j];     // one writer per key: deterministic
    }
}

void keyed_rowsum(const int32_t* keys, int key_bits, float* X, int T, int H, float* out,
                  int32_t* work, int32_t* hist, int max_tiles, int skip, cudaStream_t s, bool accumulate) {
  const int ntiles = cdiv(T, 1024);
  int32_t *kA = work, *vA = work + T, *kB = work + 2 * T, *vB = work + 3 * T;
  const int passes = key_bits <= 8 ? 1 : 2;
  const int32_t* kin = keys;
  const int32_t* vin = nullptr;
  for (int p = 0; p < passes; ++p) {
    int32_t* ko = (p == 0) ? kB : kA;
    int32_t* vo = (p == 0) ? vB : vA;
    launch_k(k_rs_hist, ntiles, 1024, 0, s, kin, T, 8 * p, ntiles, hist);
    launch_k(k_rs_scan, 1, 1024, 0, s, hist, 256 * ntiles);
    launch_k(k_rs_scatter, ntiles, 1024, 0, s, kin, vin, T, 8 * p, ntiles, hist, ko, vo);
    kin = ko;
    vin = vo;
  }
  (void)max_tiles;
  note_launch(3 * passes + 2);
  launch_k(k_piece_sum, cdiv(cdiv(T, 32), 8), 256, 0, s, kin, vin, X, T, H, skip);
  launch_k(k_segment_sum, cdiv(T, 8), 256, 0, s, kin, vin, X, T, H, out, skip, accumulate ? 1 : 0);
}

// ================================================================== heads ===

template <typename E>
__global__ void k_pool_fwd(const E* __restrict__ y, int B, int S, int H, const E* __restrict__ Wp,
                           const E* __restrict__ bp, E* __restrict__ p) {
  pdl_enter();
  const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (w >= B * H) return;
  const int b = w / H, j = w % H;
  const E* yr = y + (int64_t)b * S * H;
  const E* wr = Wp + (int64_t)j * H;
  float acc = 0.f;
  for (int k = lane; k < H; k += 32) acc += ldf(yr + k) * ldf(wr + k);
  acc = warp_sum(acc);
  if (lane == 0) stf(p + (int64_t)b * H + j, tanhf(acc + ldf(bp + j)));
}

template <typename E>
__global__ void k_cls_fwd(const E* __restrict__ p, int B, int H, const E* __restrict__ Wc,
                          const E* __restrict__ bc, int n_out, float* __restrict__ logits, Drop drop) {
  pdl_enter();
  const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (w >= B * n_out) return;
  const int b = w / n_out, o = w % n_out;
  float acc = 0.f;
  for (int j = lane; j < H; j += 32)
    acc += ldf(p + (int64_t)b * H + j) * drop_factor(drop, (uint64_t)b * H + j) * ldf(Wc + (int64_t)o * H + j);
  acc = warp_sum(acc);
  if (lane == 0) logits[b * n_out + o] = acc + ldf(bc + o);
}

// rows x cols view of the logits for the CE: MC [B/C, C], seq-cls [B, n_out]
__device__ void ce_view(int head_kind, int B, int n_out, int n_choices, int& rows, int& cols) {
  if (head_kind == 1) { rows = B / n_choices; cols = n_choices; } else { rows = B; cols = n_out; }
}

// loss (fwd) or dlogits (bwd): one warp, rows processed in order.
__global__ void k_cls_ce(const float* __restrict__ logits, const int32_t* __restrict__ labels, int B,
                         int n_out, int n_choices, int head_kind, float* __restrict__ loss,
                         float* __restrict__ dlog) {
  pdl_enter();
  int rows, cols;
  ce_view(head_kind, B, n_out, n_choices, rows, cols);
  const int lane = threadIdx.x;
  float total = 0.f;
  for (int r = 0; r < rows; ++r) {
    const float* lr = logits + (int64_t)r * cols;
    float m = -INFINITY;
    for (int c = lane; c < cols; c += 32) m = fmaxf(m, lr[c]);
    m = warp_max(m);
    float z = 0.f;
    for (int c = lane; c < cols; c += 32) z += expf(lr[c] - m);
    z = warp_sum(z);
    const float lse = m + logf(z);
    total += lse - lr[labels[r]];
    if (dlog)
      for (int c = lane; c < cols; c += 32)
        dlog[(int64_t)r * cols + c] = (expf(lr[c] - lse) - (c == labels[r] ? 1.f : 0.f)) / (float)rows;
  }
  if (loss && lane == 0) *loss = total / (float)rows;
}

void head_cls_fwd(DType dt, const void* y, int B, int S, int H, const void* Wp, const void* bp,
                  const void* Wc, const void* bc, int n_out, void* p, float* logits,
                  const int32_t* labels, int n_choices, int head_kind, float* loss, Drop drop,
                  cudaStream_t s) {
  note_launch(3);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_pool_fwd<E>, cdiv((int64_t)B * H, 8), 256, 0, s, (const E*)y, B, S, H, (const E*)Wp, (const E*)bp, (E*)p);
    launch_k(k_cls_fwd<E>, cdiv((int64_t)B * n_out, 8), 256, 0, s, (const E*)p, B, H, (const E*)Wc, (const E*)bc, n_out, logits, drop);
  });
  launch_k(k_cls_ce, 1, 32, 0, s, logits, labels, B, n_out, n_choices, head_kind, loss, nullptr);
}

// dWc[o, j] = sum_b dlog[b, o] * drop(p)[b, j], dbc[o] = sum_b dlog[b, o].
// Block: 128 columns (lane owns 4 consecutive j, one Philox call per 4), warp w
// sums b = w, w+8, ... ascending; the 8 warp sums are added in warp order.
template <typename E>
__global__ void __launch_bounds__(256) k_cls_wgrad(const float* __restrict__ dlog, const E* __restrict__ p, int B,
                                                   int H, int n_out, float* __restrict__ dWc, float* __restrict__ dbc,
                                                   Drop drop) {
  pdl_enter();
  __shared__ float4 red[8][32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nblk = (H + 127) / 128;
  const int o = blockIdx.x / nblk, j = (blockIdx.x % nblk) * 128 + 4 * lane;
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  if (j < H)
    for (int b = warp; b < B; b += 8) {
      const float d = dlog[b * n_out + o];
      const float4 f = drop_factor4(drop, ((uint64_t)b * H + j) >> 2);
      acc.x += d * ldf(p + (int64_t)b * H + j) * f.x;
      acc.y += d * ldf(p + (int64_t)b * H + j + 1) * f.y;
      acc.z += d * ldf(p + (int64_t)b * H + j + 2) * f.z;
      acc.w += d * ldf(p + (int64_t)b * H + j + 3) * f.w;
    }
  red[warp][lane] = acc;
  __syncthreads();
  if (warp == 0 && j < H) {
    float4 t = red[0][lane];
    for (int w = 1; w < 8; ++w) {
      const float4 v = red[w][lane];
      t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
    }
    float* out = dWc + (int64_t)o * H + j;
    out[0] = t.x; out[1] = t.y; out[2] = t.z; out[3] = t.w;
  }
  if (blockIdx.x % nblk == 0 && threadIdx.x == 0) {
    float t = 0.f;
    for (int b = 0; b < B; ++b) t += dlog[b * n_out + o];
    dbc[o] = t;
  }
}

template <typename E>
__global__ void k_pool_dpre(const float* __restrict__ dlog, const E* __restrict__ p, const E* __restrict__ Wc,
                            int B, int H, int n_out, float* __restrict__ dpre, Drop drop) {
  pdl_enter();
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= B * H) return;
  const int b = i / H, j = i % H;
  float acc = 0.f;
  for (int o = 0; o < n_out; ++o) acc += dlog[b * n_out + o] * ldf(Wc + (int64_t)o * H + j);
  const float pv = ldf(p + i);
  dpre[i] = acc * drop_factor(drop, (uint64_t)b * H + j) * (1.f - pv * pv);
}

// dWp[j, k] = sum_b dpre[b, j] y[b, 0, k] (b ascending); dbp[j] = sum_b dpre[b, j].
// Block: 32 columns k (lane) x 64 rows j (warp w owns j0 + 8w .. +7); dpre's
// [B x 64] slab is staged in shared memory.
template <typename E>
__global__ void __launch_bounds__(256) k_pool_wgrad(const float* __restrict__ dpre, const E* __restrict__ y, int B,
                                                    int S, int H, float* __restrict__ dWp, float* __restrict__ dbp) {
  pdl_enter();
  extern __shared__ float sdp[];          // [B][64]
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int k = blockIdx.x * 32 + lane, j0 = blockIdx.y * 64;
  for (int i = threadIdx.x; i < B * 64; i += 256) {
    const int b = i >> 6, jj = j0 + (i & 63);
    sdp[i] = jj < H ? dpre[(int64_t)b * H + jj] : 0.f;
  }
  __syncthreads();
  float acc[8];
#pragma unroll
  for (int r = 0; r < 8; ++r) acc[r] = 0.f;
  if (k < H)
    for (int b = 0; b < B; ++b) {
      const float yv = ldf(y + (int64_t)b * S * H + k);
      const float* d = sdp + b * 64 + 8 * warp;
#pragma unroll
      for (int r = 0; r < 8; ++r) acc[r] += d[r] * yv;
    }
#pragma unroll
  for (int r = 0; r < 8; ++r) {
    const int j = j0 + 8 * warp + r;
    if (j < H && k < H) dWp[(int64_t)j * H + k] = acc[r];
  }
  if (blockIdx.x == 0) {
    const int jj = threadIdx.x;
    if (jj < 64 && j0 + jj < H) {
      float t = 0.f;
      for (int b = 0; b < B; ++b) t += sdp[b * 64 + jj];
      dbp[j0 + jj] = t;
    }
  }
}

// dy[b, 0, k] = sum_j dpre[b, j] Wp[j, k].  Block: 32 columns k (lane) x 8
// sequences; warp w sums j in [w H/8, (w+1) H/8) ascending, and the 8 warp
// partials are added in warp order.
template <typename E>
__global__ void __launch_bounds__(256) k_pool_dx(const float* __restrict__ dpre, const E* __restrict__ Wp, int B,
                                                 int S, int H, float* __restrict__ dy) {
  pdl_enter();
  __shared__ float red[8][8][33];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int k = blockIdx.x * 32 + lane, b0 = blockIdx.y * 8;
  const int jb = warp * H / 8, je = (warp + 1) * H / 8;
  float acc[8];
#pragma unroll
  for (int r = 0; r < 8; ++r) acc[r] = 0.f;
  if (k < H) {
#pragma unroll 4
    for (int j = jb; j < je; ++j) {
      const float w = ldf(Wp + (int64_t)j * H + k);
#pragma unroll
      for (int r = 0; r < 8; ++r)
        if (b0 + r < B) acc[r] += dpre[(int64_t)(b0 + r) * H + j] * w;
    }
  }
#pragma unroll
  for (int r = 0; r < 8; ++r) red[warp][r][lane] = acc[r];
  __syncthreads();
  if (warp == 0 && k < H) {
    for (int r = 0; r < 8; ++r) {
      if (b0 + r >= B) break;
      float t = red[0][r][lane];
      for (int w = 1; w < 8; ++w) t += red[w][r][lane];
      dy[(int64_t)(b0 + r) * S * H + k] = t;
    }
  }
}

void head_cls_bwd(DType dt, const void* y, int B, int S, int H, const void* Wp, const void* Wc, int n_out,
                  const void* p, const float* logits, const int32_t* labels, int n_choices, int head_kind,
                  float* scratch, float* dWp, float* dbp, float* dWc, float* dbc, float* dy, Drop drop,
                  cudaStream_t s) {
  float* dlog = scratch;
  note_launch(5);
  float* dpre = scratch + ((B * n_out + 3) / 4 * 4) + (int64_t)B * H;
  launch_k(k_cls_ce, 1, 32, 0, s, logits, labels, B, n_out, n_choices, head_kind, nullptr, dlog);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_cls_wgrad<E>, n_out * cdiv(H, 128), 256, 0, s, dlog, (const E*)p, B, H, n_out, dWc, dbc, drop);
    launch_k(k_pool_dpre<E>, cdiv(B * H, 256), 256, 0, s, dlog, (const E*)p, (const E*)Wc, B, H, n_out, dpre, drop);
    launch_k(k_pool_wgrad<E>, dim3(cdiv(H, 32), cdiv(H, 64)), 256, (size_t)B * 64 * 4, s, dpre, (const E*)y, B, S,
             H, dWp, dbp);
    launch_k(k_pool_dx<E>, dim3(cdiv(H, 32), cdiv(B, 8)), 256, 0, s, dpre, (const E*)Wp, B, S, H, dy);
  });
}

// ---- QA span head ----
template <typename E>
__global__ void k_qa_logits(const E* __restrict__ y, int T, int H, const E* __restrict__ Wq,
                            const E* __restrict__ bq, float* __restrict__ logits) {
  pdl_enter();
  const int t = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (t >= T) return;
  float a0 = 0.f, a1 = 0.f;
  for (int c = lane; c < H; c += 32) {
    const float v = ldf(y + (int64_t)t * H + c);
    a0 += v * ldf(Wq + c);
    a1 += v * ldf(Wq + H + c);
  }
  a0 = warp_sum(a0);
  a1 = warp_sum(a1);
  if (lane == 0) { logits[2 * t] = a0 + ldf(bq); logits[2 * t + 1] = a1 + ldf(bq + 1); }
}

// one warp; per sequence b and side j: masked softmax CE over s < len
__global__ void k_qa_ce(const float* __restrict__ logits, const int32_t* __restrict__ lengths,
                        const int32_t* __restrict__ labels, int B, int S, float* __restrict__ loss,
                        float* __restrict__ dlog) {
  pdl_enter();
  const int lane = threadIdx.x;
  float tot[2] = {0.f, 0.f};
  for (int b = 0; b < B; ++b) {
    const int len = lengths[b];
    for (int j = 0; j < 2; ++j) {
      float m = -INFINITY;
      for (int s = lane; s < len; s += 32) m = fmaxf(m, logits[2 * (b * S + s) + j]);
      m = warp_max(m);
      float z = 0.f;
      for (int s = lane; s < len; s += 32) z += expf(logits[2 * (b * S + s) + j] - m);
      z = warp_sum(z);
      const float lse = m + logf(z);
      const int lab = labels[2 * b + j];
      tot[j] += lse - logits[2 * (b * S + lab) + j];
      if (dlog)
        for (int s = lane; s < S; s += 32)
          dlog[2 * (b * S + s) + j] =
              s < len ? 0.5f * (expf(logits[2 * (b * S + s) + j] - lse) - (s == lab ? 1.f : 0.f)) / (float)B : 0.f;
    }
  }
  if (loss && lane == 0) *loss = 0.5f * (tot[0] / (float)B + tot[1] / (float)B);
}

void head_qa_fwd(DType dt, const void* y, int B, int S, int H, const void* Wq, const void* bq, float* logits,
                 const int32_t* lengths, const int32_t* labels, float* loss, cudaStream_t s) {
  const int T = B * S;
  note_launch(2);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_qa_logits<E>, cdiv(T, 8), 256, 0, s, (const E*)y, T, H, (const E*)Wq, (const E*)bq, logits);
  });
  launch_k(k_qa_ce, 1, 32, 0, s, logits, lengths, labels, B, S, loss, nullptr);
}

template <typename E>
__global__ void k_qa_dx(const float* __restrict__ dlog, const E* __restrict__ Wq, int T, int H, float* __restrict__ dy) {
  pdl_enter();
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= (int64_t)T * H) return;
  const int t = (int)(i / H), c = (int)(i % H);
  dy[i] = dlog[2 * t] * ldf(Wq + c) + dlog[2 * t + 1] * ldf(Wq + H + c);
}

// partials [NPART][2H + 2]: dWq rows then dbq
template <typename E>
__global__ void k_qa_wgrad_part(const float* __restrict__ dlog, const E* __restrict__ y, int T, int H,
                                float* __restrict__ part) {
  pdl_enter();
  const int ld = 2 * H + 2;
  for (int c = threadIdx.x; c < ld; c += blockDim.x) {
    float acc = 0.f;
    for (int t = blockIdx.x; t < T; t += NPART) {
      if (c < 2 * H) acc += dlog[2 * t + c / H] * ldf(y + (int64_t)t * H + c % H);
      else acc += dlog[2 * t + (c - 2 * H)];
    }
    part[(int64_t)blockIdx.x * ld + c] = acc;
  }
}

void head_qa_bwd(DType dt, const void* y, int B, int S, int H, const void* Wq, const float* logits,
                 const int32_t* lengths, const int32_t* labels, float* dlog, float* part, float* dWq,
                 float* dbq, float* dy, cudaStream_t s) {
  const int T = B * S;
  note_launch(3);
  launch_k(k_qa_ce, 1, 32, 0, s, logits, lengths, labels, B, S, nullptr, dlog);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_qa_dx<E>, cdiv((int64_t)T * H, 256), 256, 0, s, dlog, (const E*)Wq, T, H, dy);
    launch_k(k_qa_wgrad_part<E>, NPART, 256, 0, s, dlog, (const E*)y, T, H, part);
  });
  reduce_partials(part, 2 * H + 2, 2 * H, dWq, s);
  reduce_partials(part + 2 * H, 2 * H + 2, 2, dbq, s);
}

// ================================================================ LM head ===
// Block (1024 threads) per token row of the chunk; fixed-order block reductions.
MDEV float block_reduce(float v, bool is_max, float* sh) {
  v = is_max ? warp_max(v) : warp_sum(v);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  __syncthreads();
  if (l == 0) sh[w] = v;
  __syncthreads();
  float r = is_max ? -INFINITY : 0.f;
  if (threadIdx.x < 32) {
    r = threadIdx.x < (int)(blockDim.x >> 5) ? sh[threadIdx.x] : (is_max ? -INFINITY : 0.f);
    r = is_max ? warp_max(r) : warp_sum(r);
    if (threadIdx.x == 0) sh[32] = r;
  }
  __syncthreads();
  return sh[32];
}

MDEV bool lm_target(const int32_t* ids, const int32_t* lengths, int S, int t, int& tgt) {
  const int b = t / S, s = t % S;
  if (s + 1 >= lengths[b]) return false;
  tgt = ids[t + 1];
  return true;
}

__global__ void __launch_bounds__(1024) k_lm_ce_fwd(const float* __restrict__ logits, int64_t ldv, int V, int row0,
                                                    const int32_t* __restrict__ ids, const int32_t* __restrict__ lengths,
                                                    int S, float2* __restrict__ tokstat) {
  pdl_enter();
  __shared__ float sh[33];
  const int r = blockIdx.x, t = row0 + r;
  const float* lr = logits + (int64_t)r * ldv;
  float m = -INFINITY;
  for (int v = threadIdx.x; v < V; v += blockDim.x) m = fmaxf(m, lr[v]);
  m = block_reduce(m, true, sh);
  float z = 0.f;
  for (int v = threadIdx.x; v < V; v += blockDim.x) z += __expf(lr[v] - m);
  z = block_reduce(z, false, sh);
  if (threadIdx.x == 0) {
    const float lse = m + __logf(z);
    int tgt;
    const float nll = lm_target(ids, lengths, S, t, tgt) ? lse - lr[tgt] : 0.f;
    tokstat[t] = make_float2(lse, nll);
  }
}
void lm_ce_fwd(const float* logits, int64_t ldv, int V, int row0, int nrows, const int32_t* ids,
               const int32_t* lengths, int S, float2* tokstat, cudaStream_t s) {
  note_launch(1);
  launch_k(k_lm_ce_fwd, nrows, 1024, 0, s, logits, ldv, V, row0, ids, lengths, S, tokstat);
}

__global__ void __launch_bounds__(1024) k_lm_loss(const float2* __restrict__ tokstat, int T,
                                                  const int32_t* __restrict__ lengths, int B, float* __restrict__ loss) {
  pdl_enter();
  __shared__ float sh[33];
  float a = 0.f;
  for (int t = threadIdx.x; t < T; t += blockDim.x) a += tokstat[t].y;
  a = block_reduce(a, false, sh);
  float nv = 0.f;
  for (int b = threadIdx.x; b < B; b += blockDim.x) nv += (float)max(lengths[b] - 1, 0);
  nv = block_reduce(nv, false, sh);
  if (threadIdx.x == 0) *loss = a / fmaxf(nv, 1.f);
}
void lm_loss(const float2* tokstat, int T, const int32_t* lengths, int B, int S, float* loss, cudaStream_t s) {
  (void)S;
  note_launch(1);
  launch_k(k_lm_loss, 1, 1024, 0, s, tokstat, T, lengths, B, loss);
}

template <typename E>
__global__ void __launch_bounds__(256) k_lm_ce_bwd(const float* __restrict__ logits, int64_t ldv, int V, int row0,
                                                   const int32_t* __restrict__ ids, const int32_t* __restrict__ lengths,
                                                   int B, int S, const float2* __restrict__ tokstat, E* __restrict__ dlog) {
  pdl_enter();
  __shared__ float inv_n;
  if (threadIdx.x == 0) {
    int nv = 0;
    for (int b = 0; b < B; ++b) nv += max(lengths[b] - 1, 0);
    inv_n = 1.0f / (float)max(nv, 1);
  }
  __syncthreads();
  const int r = blockIdx.x, t = row0 + r;
  int tgt = -1;
  const bool valid = lm_target(ids, lengths, S, t, tgt);
  const float lse = tokstat[t].x;
  const float* lr = logits + (int64_t)r * ldv;
  E* dr = dlog + (int64_t)r * ldv;
  for (int v = threadIdx.x; v < V; v += blockDim.x)
    stf(dr + v, valid ? (__expf(lr[v] - lse) - (v == tgt ? 1.f : 0.f)) * inv_n : 0.f);
}
void lm_ce_bwd(DType dt, const float* logits, int64_t ldv, int V, int row0, int nrows, const int32_t* ids,
               const int32_t* lengths, int B, int S, const float2* tokstat, void* dlog, cudaStream_t s) {
  note_launch(1);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_lm_ce_bwd<E>, nrows, 256, 0, s, logits, ldv, V, row0, ids, lengths, B, S, tokstat, (E*)dlog);
  });
}

// ============================================================== optimizer ===

template <typename E>
__global__ void __launch_bounds__(256) k_adamw(E* __restrict__ w, float* __restrict__ master, const float* __restrict__ g,
                                               float* __restrict__ m, float* __restrict__ v, int64_t n, float lr, float b1,
                                               float b2, float eps, float wd, float bc1, float bc2, float gs) {
  pdl_enter();
  const float step = lr / bc1, rb2 = 1.0f / sqrtf(bc2), decay = 1.0f - lr * wd;
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * 4; i < n;
       i += (int64_t)gridDim.x * blockDim.x * 4) {
    const float4 g4 = *(const float4*)(g + i);
    float4 m4 = *(const float4*)(m + i), v4 = *(const float4*)(v + i);
    float p[4];
    if (master) {
      const float4 p4 = *(const float4*)(master + i);
      p[0] = p4.x; p[1] = p4.y; p[2] = p4.z; p[3] = p4.w;
    } else {
#pragma unroll
      for (int k = 0; k < 4; ++k) p[k] = ldf(w + i + k);
    }
    float gg[4] = {g4.x * gs, g4.y * gs, g4.z * gs, g4.w * gs};
    float mm[4] = {m4.x, m4.y, m4.z, m4.w}, vv[4] = {v4.x, v4.y, v4.z, v4.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      p[k] *= decay;
      mm[k] = b1 * mm[k] + (1.f - b1) * gg[k];
      vv[k] = b2 * vv[k] + (1.f - b2) * gg[k] * gg[k];
      p[k] -= step * mm[k] / (sqrtf(vv[k]) * rb2 + eps);
    }
    *(float4*)(m + i) = make_float4(mm[0], mm[1], mm[2], mm[3]);
    *(float4*)(v + i) = make_float4(vv[0], vv[1], vv[2], vv[3]);
    if (master) *(float4*)(master + i) = make_float4(p[0], p[1], p[2], p[3]);
    if constexpr (std::is_same<E, __nv_bfloat16>::value) {   // one 8-B store of the 4 bf16 weights
      __nv_bfloat162 lo = __floats2bfloat162_rn(p[0], p[1]), hi = __floats2bfloat162_rn(p[2], p[3]);
      *(uint2*)(w + i) = make_uint2(*(uint32_t*)&lo, *(uint32_t*)&hi);
    } else {
#pragma unroll
      for (int k = 0; k < 4; ++k) stf(w + i + k, p[k]);
    }
  }
}

void adamw(DType dt, void* w, float* master, const float* g, float* m, float* v, int64_t n, float lr,
           float b1, float b2, float eps, float wd, float bc1, float bc2, float gs, cudaStream_t s) {
  note_launch(1);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_adamw<E>, 148 * 8, 256, 0, s, (E*)w, master, g, m, v, n, lr, b1, b2, eps, wd, bc1, bc2, gs);
  });
}

template <typename E>
__global__ void k_cast_from(const float* __restrict__ src, E* __restrict__ dst, int64_t n) {
  pdl_enter();
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    stf(dst + i, src[i]);
}
template <typename E>
__global__ void k_cast_to(const E* __restrict__ src, float* __restrict__ dst, int64_t n) {
  pdl_enter();
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dst[i] = ldf(src + i);
}
void cast_from_f32(DType dt, const float* src, void* dst, int64_t n, cudaStream_t s) {
  note_launch(1);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_cast_from<E>, 592, 256, 0, s, src, (E*)dst, n);
  });
}
void cast_to_f32(DType dt, const void* src, float* dst, int64_t n, cudaStream_t s) {
  note_launch(1);
  dispatch(dt, [&](auto* tag) {
    using E = std::remove_pointer_t<decltype(tag)>;
    launch_k(k_cast_to<E>, 592, 256, 0, s, (const E*)src, dst, n);
  });
}

}  // namespace mimose
