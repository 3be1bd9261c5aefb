// GEMM epilogues shared by the SIMT and tcgen05 GEMMs (device code only).
#pragma once
#include "kernels.h"

namespace mimose {

// Single-MUFU transcendentals.  The non-ftz __expf / __fdividef wrap each MUFU
// in denormal range fix-ups (FSETP + 2 conditional FMUL); every argument below
// is either >= 1 (rcp) or feeds a product where a flushed 2^-126 is exactly as
// good as the denormal, so the ftz forms are used directly.
MDEV float ex2_ftz(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
MDEV float rcp_ftz(float x) {
  float y;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// erf-GELU and its derivative with a branch-free erf (Abramowitz & Stegun 7.1.26,
// |error| <= 1.5e-7, far below bf16 resolution): erf(x) = 1 - poly(t) exp(-x^2),
// t = 1/(1 + p|x|).  exp(-x^2) with x = u/sqrt(2) is exp(-u^2/2), which GELU'
// also needs, so the derivative costs one extra FMA.  (libdevice erff branches
// on |x|, which diverges inside a warp of GEMM-epilogue values.)
MDEV float erf_as(float x, float e /* = exp(-x^2) */) {
  const float t = rcp_ftz(fmaf(0.3275911f, fabsf(x), 1.0f));
  float p = fmaf(1.061405429f, t, -1.453152027f);
  p = fmaf(p, t, 1.421413741f);
  p = fmaf(p, t, -0.284496736f);
  p = fmaf(p, t, 0.254829592f);
  return copysignf(fmaf(-p * t, e, 1.0f), x);
}
// erf(u / sqrt(2)) with the 1/sqrt(2) folded into the A&S constant
// (0.3275911 / sqrt(2)); the sign of u is the sign of u / sqrt(2).
MDEV float erf_s2(float u, float e /* = exp(-u^2/2) */) {
  const float t = rcp_ftz(fmaf(0.23164189922808f, fabsf(u), 1.0f));
  float p = fmaf(1.061405429f, t, -1.453152027f);
  p = fmaf(p, t, 1.421413741f);
  p = fmaf(p, t, -0.284496736f);
  p = fmaf(p, t, 0.254829592f);
  return copysignf(fmaf(-p * t, e, 1.0f), u);
}
// exp(-u^2/2) = 2^(u * (-log2(e)/2) * u)
MDEV float gauss_e(float u) { return ex2_ftz((u * -0.72134752044448170f) * u); }
MDEV float gelu_f(float u) {
  const float h = 0.5f * u;
  return fmaf(h, erf_s2(u, gauss_e(u)), h);
}
MDEV float gelu_grad_f(float u) {
  const float e = gauss_e(u);
  return fmaf(u * 0.39894228040143268f, e, fmaf(0.5f, erf_s2(u, e), 0.5f));
}

// Packed fp32x2 forms (sm_100 FFMA2 / FMUL2 / FADD2: two IEEE fp32 lanes per
// instruction, each lane rounding exactly like the scalar op).  The GEMM
// epilogue is issue-bound for the GELU epilogues; pairing halves the FMA-pipe
// instruction count.  Same operation sequence as gelu_f / gelu_grad_f, so the
// packed and scalar results are bit-identical.
MDEV uint64_t f2u(float2 a) { return ((uint64_t)__float_as_uint(a.y) << 32) | __float_as_uint(a.x); }
MDEV float2 u2f(uint64_t d) { return make_float2(__uint_as_float((uint32_t)d), __uint_as_float((uint32_t)(d >> 32))); }
MDEV float2 ffma2(float2 a, float2 b, float2 c) {
  uint64_t d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(f2u(a)), "l"(f2u(b)), "l"(f2u(c)));
  return u2f(d);
}
MDEV float2 fmul2(float2 a, float2 b) {
  uint64_t d;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(f2u(a)), "l"(f2u(b)));
  return u2f(d);
}
MDEV float2 fadd2(float2 a, float2 b) {
  uint64_t d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(f2u(a)), "l"(f2u(b)));
  return u2f(d);
}
MDEV float2 f2s(float c) { return make_float2(c, c); }
MDEV float2 erf_s2_x2(float2 u, float2 e) {
  const float2 d = ffma2(f2s(0.23164189922808f), make_float2(fabsf(u.x), fabsf(u.y)), f2s(1.0f));
  const float2 t = make_float2(rcp_ftz(d.x), rcp_ftz(d.y));
  float2 p = ffma2(f2s(1.061405429f), t, f2s(-1.453152027f));
  p = ffma2(p, t, f2s(1.421413741f));
  p = ffma2(p, t, f2s(-0.284496736f));
  p = ffma2(p, t, f2s(0.254829592f));
  const float2 pt = fmul2(p, t);
  const float2 r = ffma2(make_float2(-pt.x, -pt.y), e, f2s(1.0f));
  return make_float2(copysignf(r.x, u.x), copysignf(r.y, u.y));
}
MDEV float2 gauss_e_x2(float2 u) {
  const float2 a = fmul2(fmul2(u, f2s(-0.72134752044448170f)), u);
  return make_float2(ex2_ftz(a.x), ex2_ftz(a.y));
}
MDEV float2 gelu_x2(float2 u) {
  const float2 h = fmul2(f2s(0.5f), u);
  return ffma2(h, erf_s2_x2(u, gauss_e_x2(u)), h);
}
MDEV float2 gelu_grad_x2(float2 u) {
  const float2 e = gauss_e_x2(u);
  return ffma2(fmul2(u, f2s(0.39894228040143268f)), e, ffma2(f2s(0.5f), erf_s2_x2(u, e), f2s(0.5f)));
}

// Fast erf-GELU for the bf16 tcgen05 epilogues: the tanh form
// 0.5 u (1 + tanh(sqrt(2/pi) (u + 0.044715 u^3))) with one MUFU.TANH.  Its
// distance to the exact erf-GELU is <= 4.8e-4 (at u = 2.7, where a bf16 ulp is
// 1.6e-2) and that of its derivative to the exact GELU' <= 8.7e-4 (bf16 ulp
// 7.8e-3), so the stored bf16 values are within a small fraction of an ulp of
// the exact ones (reading R-G).  The fp32 (SIMT) path keeps the exact
// erf forms above.  Backward uses this function's own derivative.
MDEV float tanh_apx(float x) {
  float y;
  asm("tanh.approx.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
MDEV float gelu_fast(float u) {
  const float z = u * fmaf(0.035677408136300125f, u * u, 0.7978845608028654f);
  const float h = 0.5f * u;
  return fmaf(h, tanh_apx(z), h);
}
MDEV float gelu_grad_fast(float u) {
  const float u2 = u * u;
  const float t = tanh_apx(u * fmaf(0.035677408136300125f, u2, 0.7978845608028654f));
  const float dz = fmaf(0.10703222440890037f, u2, 0.7978845608028654f);
  return fmaf(0.5f * u * fmaf(-t, t, 1.0f), dz, fmaf(0.5f, t, 0.5f));
}
MDEV float2 gelu_fast_x2(float2 u) {
  const float2 u2 = fmul2(u, u);
  const float2 z = fmul2(u, ffma2(f2s(0.035677408136300125f), u2, f2s(0.7978845608028654f)));
  const float2 t = make_float2(tanh_apx(z.x), tanh_apx(z.y));
  const float2 h = fmul2(f2s(0.5f), u);
  return ffma2(h, t, h);
}
MDEV float2 gelu_grad_fast_x2(float2 u) {
  const float2 u2 = fmul2(u, u);
  const float2 z = fmul2(u, ffma2(f2s(0.035677408136300125f), u2, f2s(0.7978845608028654f)));
  const float2 t = make_float2(tanh_apx(z.x), tanh_apx(z.y));
  const float2 dz = ffma2(f2s(0.10703222440890037f), u2, f2s(0.7978845608028654f));
  const float2 omt = ffma2(make_float2(-t.x, -t.y), t, f2s(1.0f));
  return ffma2(fmul2(fmul2(f2s(0.5f), u), omt), dz, ffma2(f2s(0.5f), t, f2s(0.5f)));
}

// GPT-2 "gelu_new": 0.5 u (1 + tanh(k0 (u + 0.044715 u^3))), tanh via one exp:
// tanh z = 1 - 2 / (2^(2 log2(e) z) + 1) (inf -> 1, 0 -> -1 at the extremes).
MDEV float tanh_fast(float z) { return fmaf(-2.0f, rcp_ftz(ex2_ftz(2.8853900817779268f * z) + 1.0f), 1.0f); }
MDEV float gelu_tanh_f(float u) {
  const float z = 0.7978845608028654f * fmaf(0.044715f * u, u * u, u);
  const float h = 0.5f * u;
  return fmaf(h, tanh_fast(z), h);
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
