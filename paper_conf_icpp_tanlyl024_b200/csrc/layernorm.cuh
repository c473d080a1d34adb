// layernorm.cuh — the per-row LayerNorm shared by the LayerNorm / embedding kernels and the
// LayerNorm prologue of the persistent GEMMs (steps a5 / a8; BERT [17], PAPER.md:L422;
// reading S3: biased variance, eps inside the square root).  One warp per row: the row in
// registers, two-pass fp32 statistics with warp-shuffle sums, RNE to the output type.  The
// arithmetic is written with explicit _rn intrinsics, so both call sites compute a row with
// the same instruction sequence (bitwise-equal rows, tests: LN prologue vs LN kernel).
#pragma once

#include "common.cuh"
#include "kernels.h"

namespace arlo {

template <typename T> struct Vec;
template <> struct Vec<bf16> {
  static constexpr int N = 8;  // 16 B
  static __device__ __forceinline__ void load(const bf16* p, float* f, bool dep = false) {
    uint4 u = dep ? ld_dep_v4(p) : __ldg(reinterpret_cast<const uint4*>(p));
    float2 a = unpack_bf16x2(u.x), b = unpack_bf16x2(u.y), c = unpack_bf16x2(u.z), d = unpack_bf16x2(u.w);
    f[0] = a.x; f[1] = a.y; f[2] = b.x; f[3] = b.y; f[4] = c.x; f[5] = c.y; f[6] = d.x; f[7] = d.y;
  }
  static __device__ __forceinline__ void store(bf16* p, const float* f) {
    uint4 u;
    u.x = pack_bf16x2(f[0], f[1]); u.y = pack_bf16x2(f[2], f[3]);
    u.z = pack_bf16x2(f[4], f[5]); u.w = pack_bf16x2(f[6], f[7]);
    *reinterpret_cast<uint4*>(p) = u;
  }
};
template <> struct Vec<float> {
  static constexpr int N = 4;
  static __device__ __forceinline__ void load(const float* p, float* f, bool dep = false) {
    float4 v;
    if (dep) {
      const uint4 u = ld_dep_v4(p);
      v = make_float4(__uint_as_float(u.x), __uint_as_float(u.y), __uint_as_float(u.z), __uint_as_float(u.w));
    } else {
      v = __ldg(reinterpret_cast<const float4*>(p));
    }
    f[0] = v.x; f[1] = v.y; f[2] = v.z; f[3] = v.w;
  }
  static __device__ __forceinline__ void store(float* p, const float* f) {
    *reinterpret_cast<float4*>(p) = make_float4(f[0], f[1], f[2], f[3]);
  }
};

// Normalise the row held in v[MAXV][VN] (only vectors lane + 32 i < nvec valid) and store it.
// g, b point to the shared-memory copies of gamma / beta.
template <typename T, int MAXV>
__device__ __forceinline__ void ln_finish(float (&v)[MAXV][Vec<T>::N], int nvec, int H, int lane,
                                          const float* g, const float* b,
                                          float eps, T* __restrict__ out_row) {
  constexpr int VN = Vec<T>::N;
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < MAXV; ++i) {
    if (lane + 32 * i < nvec) {
#pragma unroll
      for (int j = 0; j < VN; ++j) s += v[i][j];
    }
  }
  const float mean = warp_sum(s) / (float)H;
  float q = 0.f;
#pragma unroll
  for (int i = 0; i < MAXV; ++i) {
    if (lane + 32 * i < nvec) {
#pragma unroll
      for (int j = 0; j < VN; ++j) {
        const float d = __fsub_rn(v[i][j], mean);
        q = __fmaf_rn(d, d, q);
      }
    }
  }
  const float var = warp_sum(q) / (float)H;
  const float rstd = 1.0f / sqrtf(var + eps);
#pragma unroll
  for (int i = 0; i < MAXV; ++i) {
    const int vi = lane + 32 * i;
    if (vi < nvec) {
      const int c0 = vi * VN;
      float gg[VN], bb[VN], o[VN];
#pragma unroll
      for (int j = 0; j < VN; j += 4) {
        const float4 g4 = *reinterpret_cast<const float4*>(g + c0 + j);
        const float4 b4 = *reinterpret_cast<const float4*>(b + c0 + j);
        gg[j] = g4.x; gg[j + 1] = g4.y; gg[j + 2] = g4.z; gg[j + 3] = g4.w;
        bb[j] = b4.x; bb[j + 1] = b4.y; bb[j + 2] = b4.z; bb[j + 3] = b4.w;
      }
#pragma unroll
      for (int j = 0; j < VN; ++j) o[j] = __fmaf_rn(__fmul_rn(__fsub_rn(v[i][j], mean), rstd), gg[j], bb[j]);
      Vec<T>::store(out_row + c0, o);
    }
  }
}

// ---------------------------------------------------------------------------------------------
// LayerNorm as the prologue of the GEMM that consumes its output (QKV after LN2 of the previous
// layer, FFN1 after LN1): every warp of the persistent grid normalises rows r = gw, gw + nw, ...
// (gw = global warp index, nw = warps in the grid) and stores x = LN(y); a grid-wide barrier then
// makes x visible to the TMA loads of the main loop.  Removes the LayerNorm kernel and its launch
// boundary.
template <int MAXV>
__device__ __forceinline__ void ln_prologue_rows(const LnPrologue& lp, int gw, int nw, int lane) {
  constexpr int VN = 8;
  const int nvec = lp.H / VN;
  for (int row = gw; row < lp.rows; row += nw) {
    float v[MAXV][VN];
    const bf16* src = reinterpret_cast<const bf16*>(lp.y) + (size_t)row * lp.H;
#pragma unroll
    for (int i = 0; i < MAXV; ++i)
      if (lane + 32 * i < nvec) Vec<bf16>::load(src + (lane + 32 * i) * VN, v[i], true);
    ln_finish<bf16, MAXV>(v, nvec, lp.H, lane, lp.g, lp.b, lp.eps, reinterpret_cast<bf16*>(lp.x) + (size_t)row * lp.H);
  }
}

// Every thread of every CTA of the grid calls this (the grid is persistent: all CTAs resident).
__device__ __forceinline__ void ln_prologue(const LnPrologue& lp) {
  const int lane = threadIdx.x & 31, nwarp = blockDim.x >> 5;
  const int gw = blockIdx.x * nwarp + (threadIdx.x >> 5), nw = gridDim.x * nwarp;
  switch ((lp.H / 8 + 31) / 32) {
    case 1: ln_prologue_rows<1>(lp, gw, nw, lane); break;
    case 2: ln_prologue_rows<2>(lp, gw, nw, lane); break;
    case 3: ln_prologue_rows<3>(lp, gw, nw, lane); break;
    case 4: ln_prologue_rows<4>(lp, gw, nw, lane); break;
  }
  asm volatile("fence.proxy.async.global;" ::: "memory");  // x is read next by TMA (async proxy)
  grid_barrier(lp.bar);
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

}  // namespace arlo
