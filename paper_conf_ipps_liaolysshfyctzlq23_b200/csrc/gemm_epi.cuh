// GEMM epilogues shared by the SIMT and tcgen05 GEMMs (device code only).
#pragma once
#include "kernels.h"

namespace mimose {

MDEV float gelu_f(float u) { return 0.5f * u * (1.0f + erff(u * 0.70710678118654752f)); }
MDEV float gelu_grad_f(float u) {
  return 0.5f * (1.0f + erff(u * 0.70710678118654752f)) + u * 0.39894228040143268f * expf(-0.5f * u * u);
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
  } else {
    ((float*)g.C)[(int64_t)z * g.split_stride + o] = acc;
  }
}


}  // namespace mimose
