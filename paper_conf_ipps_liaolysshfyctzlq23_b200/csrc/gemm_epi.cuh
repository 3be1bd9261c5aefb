// GEMM epilogues shared by the SIMT and tcgen05 GEMMs (device code only).
#pragma once
#include "kernels.h"

namespace mimose {

// erf-GELU and its derivative with a branch-free erf (Abramowitz & Stegun 7.1.26,
// |error| <= 1.5e-7, far below bf16 resolution): erf(x) = 1 - poly(t) exp(-x^2),
// t = 1/(1 + p|x|).  exp(-x^2) with x = u/sqrt(2) is exp(-u^2/2), which GELU'
// also needs, so the derivative costs one extra FMA.  (libdevice erff branches
// on |x|, which diverges inside a warp of GEMM-epilogue values.)
MDEV float erf_as(float x, float e /* = exp(-x^2) */) {
  const float ax = fabsf(x);
  const float t = __fdividef(1.0f, fmaf(0.3275911f, ax, 1.0f));
  float p = fmaf(1.061405429f, t, -1.453152027f);
  p = fmaf(p, t, 1.421413741f);
  p = fmaf(p, t, -0.284496736f);
  p = fmaf(p, t, 0.254829592f);
  const float r = 1.0f - p * t * e;
  return copysignf(r, x);
}
MDEV float gelu_f(float u) {
  const float e = __expf(-0.5f * u * u);
  return 0.5f * u * (1.0f + erf_as(u * 0.70710678118654752f, e));
}
MDEV float gelu_grad_f(float u) {
  const float e = __expf(-0.5f * u * u);
  return 0.5f * (1.0f + erf_as(u * 0.70710678118654752f, e)) + u * 0.39894228040143268f * e;
}

// GPT-2 "gelu_new": 0.5 u (1 + tanh(k0 (u + 0.044715 u^3))), tanh via one exp.
MDEV float tanh_fast(float z) { return 1.0f - __fdividef(2.0f, __expf(2.0f * z) + 1.0f); }
MDEV float gelu_tanh_f(float u) {
  const float z = 0.7978845608028654f * fmaf(0.044715f * u, u * u, u);
  return 0.5f * u * (1.0f + tanh_fast(z));
}
MDEV float gelu_tanh_grad_f(float u) {
  const float z = 0.7978845608028654f * fmaf(0.044715f * u, u * u, u);
  const float th = tanh_fast(z);
  return 0.5f * (1.0f + th) + 0.5f * u * (1.0f - th * th) * 0.7978845608028654f * fmaf(0.134145f, u * u, 1.0f);
}

// Epilogue of one output element.
template <typename E, int EPI>
MDEV void epilogue(const GemmArgs& g, int m, int n, float acc, int z = -1) {
  if (z < 0) z = blockIdx.z;
  const int64_t o = (int64_t)m * g.ldc + n;
  if constexpr (EPI == EPI_STORE) {
    stf((E*)g.C + o, acc);
  } else if constexpr (EPI == EPI_BIAS) {
    stf((E*)g.C + o, acc + ldf((const E*)g.bias + n));
  } else if constexpr (EPI == EPI_BIAS_GELU) {
    E* up = (E*)g.C + o;
    stf(up, acc + ldf((const E*)g.bias + n));
    stf((E*)g.C2 + o, gelu_f(ldf(up)));
  } else if constexpr (EPI == EPI_BIAS_DROP_RES) {
    const float t = acc + ldf((const E*)g.bias + n);
    ((float*)g.C)[o] = ldf((const E*)g.res + (int64_t)m * g.ldr + n) + t * drop_factor(g.drop, (uint64_t)o);
  } else if constexpr (EPI == EPI_GELU_BWD) {
    stf((E*)g.C + o, acc * gelu_grad_f(ldf((const E*)g.aux + (int64_t)m * g.ldx + n)));
  } else if constexpr (EPI == EPI_ACC_RES_F32) {
    ((float*)g.C)[o] = acc + ((const float*)g.res)[(int64_t)m * g.ldr + n];
  } else if constexpr (EPI == EPI_BIAS_GELUT) {
    E* up = (E*)g.C + o;
    stf(up, acc + ldf((const E*)g.bias + n));
    stf((E*)g.C2 + o, gelu_tanh_f(ldf(up)));
  } else if constexpr (EPI == EPI_GELUT_BWD) {
    stf((E*)g.C + o, acc * gelu_tanh_grad_f(ldf((const E*)g.aux + (int64_t)m * g.ldx + n)));
  } else if constexpr (EPI == EPI_BIAS_DROP_RESF32) {
    const float t = acc + ldf((const E*)g.bias + n);
    ((float*)g.C)[o] = ((const float*)g.res)[(int64_t)m * g.ldr + n] + t * drop_factor(g.drop, (uint64_t)o);
  } else if constexpr (EPI == EPI_ACC_F32) {
    ((float*)g.C)[o] += acc;
  } else if constexpr (EPI == EPI_NONE) {
    if (acc == 1234.5f) ((float*)g.C)[o] = acc;   // keep the value live
  } else {
    ((float*)g.C)[(int64_t)z * g.split_stride + o] = acc;
  }
}


}  // namespace mimose
