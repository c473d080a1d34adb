// epilogue.cuh — the per-element GEMM epilogue shared by every tcgen05 GEMM kernel
// (single CTA, CTA pair, skinny, split-K): a given output element is computed with the
// same fp32 instruction sequence whatever kernel or tile produced its accumulator, which
// the bitwise tile-width / cross-L tests rely on.
#pragma once

#include "common.cuh"
#include "kernels.h"

namespace arlo {

// Epilogue arithmetic of 4 consecutive columns of one row: acc + bias, then GELU or
// + residual (two bf16x2 words ua, ub), RNE-packed to two bf16x2 words.  Paired fp32
// instructions (FADD2 / FFMA2); shared by every GEMM kernel so the result of an element
// does not depend on the tile shape that produced it.
template <int EPI>
__device__ __forceinline__ void epi_pack4(const uint32_t* r, float4 b4, uint32_t ua, uint32_t ub, uint32_t& p0,
                                          uint32_t& p1) {
#if defined(ARLO_EPI_SCALAR)  // A/B only: the previous scalar epilogue arithmetic
  float v0 = __uint_as_float(r[0]) + b4.x, v1 = __uint_as_float(r[1]) + b4.y;
  float v2 = __uint_as_float(r[2]) + b4.z, v3 = __uint_as_float(r[3]) + b4.w;
  if (EPI == EPI_BIAS_GELU) {
    v0 = gelu_erf_fast(v0); v1 = gelu_erf_fast(v1); v2 = gelu_erf_fast(v2); v3 = gelu_erf_fast(v3);
  }
  if (EPI == EPI_BIAS_RESID) {
    const float2 fa = unpack_bf16x2(ua), fb = unpack_bf16x2(ub);
    v0 += fa.x; v1 += fa.y; v2 += fb.x; v3 += fb.y;
  }
  p0 = pack_bf16x2(v0, v1);
  p1 = pack_bf16x2(v2, v3);
  return;
#endif
  float2 x0 = __fadd2_rn(make_float2(__uint_as_float(r[0]), __uint_as_float(r[1])), make_float2(b4.x, b4.y));
  float2 x1 = __fadd2_rn(make_float2(__uint_as_float(r[2]), __uint_as_float(r[3])), make_float2(b4.z, b4.w));
  if (EPI == EPI_BIAS_GELU) {
    x0 = gelu2_erf_fast(x0);
    x1 = gelu2_erf_fast(x1);
  }
  if (EPI == EPI_BIAS_RESID) {
    x0 = __fadd2_rn(x0, unpack_bf16x2(ua));
    x1 = __fadd2_rn(x1, unpack_bf16x2(ub));
  }
  p0 = pack_bf16x2(x0.x, x0.y);
  p1 = pack_bf16x2(x1.x, x1.y);
}

// Epilogue arithmetic of one column pair of a row for the LayerNorm-fold modes (paired fp32;
// the tile, skinny and split-K kernels share it):
//  EPI_LNFOLD(_GELU): x = acc * rstd + (nrm * s + c), nrm = -rstd * mean (rowst = (nrm, rstd)); GELU;
//  EPI_RESID_LN: x = (acc + b) + LN(r), LN(r) = ((r - mean) * rstd) * gamma + beta
//    (rowst = (mean, rstd) of the residual row; mean 0 / rstd 1 / gamma 1 / beta 0 = plain residual
//    is not used: a plain residual passes rowst.y < 0).
template <int EPI>
__device__ __forceinline__ uint32_t epi_fold_pair(float2 a, float2 v0, float2 v1, float2 v2, uint32_t ru, float2 rowst) {
  float2 x;
  if constexpr (EPI == EPI_LNFOLD || EPI == EPI_LNFOLD_GELU) {  // v0 = s, v1 = c
    x = __ffma2_rn(a, f2(rowst.y), __ffma2_rn(f2(rowst.x), v0, v1));
    if (EPI == EPI_LNFOLD_GELU) x = gelu2_erf_fast(x);
  } else {  // v0 = bias, v1 = gamma, v2 = beta
    float2 rr = unpack_bf16x2(ru);
    if (rowst.y >= 0.f) rr = __ffma2_rn(__fmul2_rn(__fadd2_rn(rr, f2(-rowst.x)), f2(rowst.y)), v1, v2);
    x = __fadd2_rn(__fadd2_rn(a, v0), rr);
  }
  return pack_bf16x2(x.x, x.y);
}

}  // namespace arlo
