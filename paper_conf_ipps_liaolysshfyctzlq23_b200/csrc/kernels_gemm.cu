// GEMM dispatch + the SIMT GEMM (fp32 mode, and the reference path of bf16
// mode).  The tcgen05/TMEM/TMA GEMM for bf16 lives in kernels_gemm_tc.cu.
//
// All linear layers of the layer ("Linear, GEMM ... the input-output
// tensor shapes have a deterministically linear correlation") go through
// gemm(): forward Y = X W^T (+ fused bias / GELU / dropout+residual), dgrad
// dX = dY W (+ GELU' or residual), wgrad dW = dY^T X (fp32, deterministic
// split-K: partials reduced in a fixed order).
#include "kernels.h"
#include "gemm_epi.cuh"

#include <cmath>
#include <cstdio>

namespace mimose {

bool gemm_tc(Epi epi, const GemmArgs& g, cudaStream_t st);   // kernels_gemm_tc.cu

static inline int cdiv(int64_t a, int64_t b) { return (int)((a + b - 1) / b); }

constexpr int SBM = 64, SBN = 64, SBK = 16;

template <typename E, int EPI>
__global__ void __launch_bounds__(256) k_gemm_simt(const GemmArgs g) {
  pdl_enter();
  __shared__ float As[SBK][SBM + 4];
  __shared__ float Bs[SBK][SBN + 4];
  const int tid = threadIdx.x, tx = tid % 16, ty = tid / 16;
  const int m0 = blockIdx.y * SBM, n0 = blockIdx.x * SBN;
  const int kper = cdiv_dev(g.K, g.split);
  const int kbeg = blockIdx.z * kper, kend = min(g.K, kbeg + kper);
  const E* A = (const E*)g.A;
  const E* B = (const E*)g.B;
  float acc[4][4] = {};
  for (int k0 = kbeg; k0 < kend; k0 += SBK) {
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      int mm, kk;
      if (g.a_sk == 1) { mm = tid / 4; kk = (tid % 4) * 4 + r; } else { kk = tid / 16; mm = (tid % 16) * 4 + r; }
      const int gm = m0 + mm, gk = k0 + kk;
      As[kk][mm] = (gm < g.M && gk < kend) ? ldf(A + (int64_t)gm * g.a_sm + (int64_t)gk * g.a_sk) : 0.f;
      int nn, kb;
      if (g.b_sk == 1) { nn = tid / 4; kb = (tid % 4) * 4 + r; } else { kb = tid / 16; nn = (tid % 16) * 4 + r; }
      const int gn = n0 + nn, gk2 = k0 + kb;
      Bs[kb][nn] = (gn < g.N && gk2 < kend) ? ldf(B + (int64_t)gn * g.b_sn + (int64_t)gk2 * g.b_sk) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < SBK; ++k) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) { a[i] = As[k][ty * 4 + i]; b[i] = Bs[k][tx * 4 + i]; }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] += a[i] * b[j];
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int m = m0 + ty * 4 + i, n = n0 + tx * 4 + j;
      if (m < g.M && n < g.N) epilogue<E, EPI>(g, m, n, acc[i][j]);
    }
}

template <typename E>
static void launch_simt(Epi epi, const GemmArgs& g, cudaStream_t st) {
  dim3 grid(cdiv(g.N, SBN), cdiv(g.M, SBM), g.split);
  switch (epi) {
    case EPI_STORE: launch_k(k_gemm_simt<E, EPI_STORE>, grid, 256, 0, st, g); break;
    case EPI_BIAS: launch_k(k_gemm_simt<E, EPI_BIAS>, grid, 256, 0, st, g); break;
    case EPI_BIAS_GELU: launch_k(k_gemm_simt<E, EPI_BIAS_GELU>, grid, 256, 0, st, g); break;
    case EPI_BIAS_DROP_RES: launch_k(k_gemm_simt<E, EPI_BIAS_DROP_RES>, grid, 256, 0, st, g); break;
    case EPI_GELU_BWD: launch_k(k_gemm_simt<E, EPI_GELU_BWD>, grid, 256, 0, st, g); break;
    case EPI_ACC_RES_F32: launch_k(k_gemm_simt<E, EPI_ACC_RES_F32>, grid, 256, 0, st, g); break;
    case EPI_BIAS_GELUT: launch_k(k_gemm_simt<E, EPI_BIAS_GELUT>, grid, 256, 0, st, g); break;
    case EPI_GELUT_BWD: launch_k(k_gemm_simt<E, EPI_GELUT_BWD>, grid, 256, 0, st, g); break;
    case EPI_BIAS_DROP_RESF32: launch_k(k_gemm_simt<E, EPI_BIAS_DROP_RESF32>, grid, 256, 0, st, g); break;
    case EPI_ACC_F32: launch_k(k_gemm_simt<E, EPI_ACC_F32>, grid, 256, 0, st, g); break;
    default: launch_k(k_gemm_simt<E, EPI_F32>, grid, 256, 0, st, g); break;
  }
}

void gemm(DType dt, Epi epi, const GemmArgs& g, cudaStream_t st, bool use_tc) {
  if (g.M <= 0 || g.N <= 0) return;
  note_launch(1);
  if (use_tc && dt == DT_BF16 && gemm_tc(epi, g, st)) return;
  if (dt == DT_F32) launch_simt<float>(epi, g, st);
  else launch_simt<__nv_bfloat16>(epi, g, st);
}

}  // namespace mimose
