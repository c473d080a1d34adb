// head.cu — step a9: CLS pooler + classifier of a discriminative model.
//
// logits[b] = W_c tanh(W_p x[b, 0] + b_p) + b_c (BERT pooler on position 0
// and a linear classifier, [17] PAPER.md:L422; discriminative models predict
// "labels or classifications"; reading S8).  One CTA per
// sequence; warp-per-output dot products with lanes striding K (coalesced
// 16-byte weight loads), fp32 accumulation, fp32 logits.  Latency-bound:
// B <= 64 rows of H x H then C x H.
#include "common.cuh"
#include "kernels.h"

namespace arlo {
namespace {

template <typename T>
__device__ __forceinline__ float dot_row(const T* __restrict__ w, const float* __restrict__ x, int H, int lane);

template <>
__device__ __forceinline__ float dot_row<bf16>(const bf16* __restrict__ w, const float* __restrict__ x, int H,
                                               int lane) {
  float s = 0.f;
  for (int k = lane * 8; k < H; k += 256) {
    const uint4 u = __ldg(reinterpret_cast<const uint4*>(w + k));
    const float2 a = unpack_bf16x2(u.x), b = unpack_bf16x2(u.y), c = unpack_bf16x2(u.z), d = unpack_bf16x2(u.w);
    s = fmaf(a.x, x[k], s); s = fmaf(a.y, x[k + 1], s); s = fmaf(b.x, x[k + 2], s); s = fmaf(b.y, x[k + 3], s);
    s = fmaf(c.x, x[k + 4], s); s = fmaf(c.y, x[k + 5], s); s = fmaf(d.x, x[k + 6], s); s = fmaf(d.y, x[k + 7], s);
  }
  return warp_sum(s);
}

template <>
__device__ __forceinline__ float dot_row<float>(const float* __restrict__ w, const float* __restrict__ x, int H,
                                                int lane) {
  float s = 0.f;
  for (int k = lane * 4; k < H; k += 128) {
    const float4 u = __ldg(reinterpret_cast<const float4*>(w + k));
    s = fmaf(u.x, x[k], s); s = fmaf(u.y, x[k + 1], s); s = fmaf(u.z, x[k + 2], s); s = fmaf(u.w, x[k + 3], s);
  }
  return warp_sum(s);
}

template <typename T>
__global__ void __launch_bounds__(512) head_kernel(int L, int H, int C, const T* __restrict__ x,
                                                   const T* __restrict__ w_p, const float* __restrict__ b_p,
                                                   const T* __restrict__ w_c, const float* __restrict__ b_c,
                                                   float* __restrict__ logits) {
  extern __shared__ float sh[];
  float* xs = sh;       // CLS row, fp32
  float* ps = sh + H;   // pooled
  const int b = blockIdx.x;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  const T* xr = x + (size_t)b * L * H;  // position 0 of sequence b
  for (int k = threadIdx.x; k < H; k += blockDim.x) xs[k] = Elem<T>::to_f(xr[k]);
  __syncthreads();
  for (int j = warp; j < H; j += nw) {
    const float v = dot_row<T>(w_p + (size_t)j * H, xs, H, lane);
    if (lane == 0) ps[j] = tanhf(v + b_p[j]);
  }
  __syncthreads();
  for (int c = warp; c < C; c += nw) {
    const float v = dot_row<T>(w_c + (size_t)c * H, ps, H, lane);
    if (lane == 0) logits[(size_t)b * C + c] = v + b_c[c];
  }
}

}  // namespace

cudaError_t launch_head(DType dt, int B, int L, int H, int C, const void* x, const void* w_p, const float* b_p,
                        const void* w_c, const float* b_c, float* logits, cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  const size_t smem = 2 * (size_t)H * sizeof(float);
  if (dt == DT_BF16)
    head_kernel<bf16><<<B, 512, smem, s>>>(L, H, C, (const bf16*)x, (const bf16*)w_p, b_p, (const bf16*)w_c, b_c,
                                           logits);
  else
    head_kernel<float><<<B, 512, smem, s>>>(L, H, C, (const float*)x, (const float*)w_p, b_p, (const float*)w_c,
                                            b_c, logits);
  return cudaGetLastError();
}

}  // namespace arlo
