// head.cu — step a9: CLS pooler + classifier of a discriminative model.
//
// pooled[b] = tanh(W_p x[b, 0] + b_p);  logits[b] = W_c pooled[b] + b_c
// (BERT pooler on position 0 and a linear classifier, [17] PAPER.md:L422;
// discriminative models predict "labels or classifications", PAPER.md:L33-35;
// reading S8).  Latency-bound (B <= 64 rows): the pooler spreads its H output
// features over H/8 x ceil(B/8) CTAs; each warp owns one feature and 8
// sequences, reads its W_p row once (coalesced 16-byte loads, lanes striding
// K) against the 8 CLS rows staged in shared memory as fp32, and keeps 8
// fp32 partial sums.  A second tiny kernel applies the classifier.  Every
// reduction order is fixed, so a sequence's logits do not depend on B.
#include "common.cuh"
#include "kernels.h"

namespace arlo {
namespace {

constexpr int kRows = 8;   // sequences per CTA
constexpr int kFeat = 8;   // output features per CTA (one per warp)

template <typename T> struct Ld8;
template <> struct Ld8<bf16> {
  static constexpr int N = 8;
  static __device__ __forceinline__ void load(const bf16* p, float* f) {
    const uint4 u = __ldg(reinterpret_cast<const uint4*>(p));
    float2 a = unpack_bf16x2(u.x), b = unpack_bf16x2(u.y), c = unpack_bf16x2(u.z), d = unpack_bf16x2(u.w);
    f[0] = a.x; f[1] = a.y; f[2] = b.x; f[3] = b.y; f[4] = c.x; f[5] = c.y; f[6] = d.x; f[7] = d.y;
  }
};
template <> struct Ld8<float> {
  static constexpr int N = 4;
  static __device__ __forceinline__ void load(const float* p, float* f) {
    const float4 u = __ldg(reinterpret_cast<const float4*>(p));
    f[0] = u.x; f[1] = u.y; f[2] = u.z; f[3] = u.w;
  }
};

template <typename T>
__global__ void __launch_bounds__(256) pooler_kernel(int B, int L, int H, const T* __restrict__ x,
                                                     const T* __restrict__ w_p, const float* __restrict__ b_p,
                                                     float* __restrict__ pooled) {
  extern __shared__ float xs[];  // [kRows][H]
  pdl_begin();
  const int b0 = blockIdx.y * kRows;
  const int nb = min(kRows, B - b0);
  for (int i = threadIdx.x; i < kRows * H; i += blockDim.x) {
    const int r = i / H, k = i - r * H;
    xs[i] = r < nb ? Elem<T>::to_f(x[(size_t)(b0 + r) * L * H + k]) : 0.f;  // position 0 of sequence b0+r
  }
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int j = blockIdx.x * kFeat + warp;
  if (j >= H) return;
  constexpr int VN = Ld8<T>::N;
  float acc[kRows];
#pragma unroll
  for (int r = 0; r < kRows; ++r) acc[r] = 0.f;
  const T* wr = w_p + (size_t)j * H;
  for (int k = lane * VN; k < H; k += 32 * VN) {
    float wv[VN];
    Ld8<T>::load(wr + k, wv);
#pragma unroll
    for (int r = 0; r < kRows; ++r) {
#pragma unroll
      for (int e = 0; e < VN; ++e) acc[r] = fmaf(wv[e], xs[r * H + k + e], acc[r]);
    }
  }
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    const float v = warp_sum(acc[r]);
    if (lane == 0 && r < nb) pooled[(size_t)(b0 + r) * H + j] = tanhf(v + b_p[j]);
  }
}

template <typename T>
__global__ void __launch_bounds__(64) classifier_kernel(int H, int C, const float* __restrict__ pooled,
                                                        const T* __restrict__ w_c, const float* __restrict__ b_c,
                                                        float* __restrict__ logits) {
  pdl_begin();
  const int b = blockIdx.x;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const float* p = pooled + (size_t)b * H;
  for (int c = warp; c < C; c += 2) {
    const T* wr = w_c + (size_t)c * H;
    float s = 0.f;
    for (int k = lane; k < H; k += 32) s = fmaf(Elem<T>::to_f(wr[k]), p[k], s);
    s = warp_sum(s);
    if (lane == 0) logits[(size_t)b * C + c] = s + b_c[c];
  }
}

template <typename T>
cudaError_t launch_t(int B, int L, int H, int C, const void* x, const void* w_p, const float* b_p, const void* w_c,
                     const float* b_c, float* pooled, float* logits, cudaStream_t s) {
  const size_t smem = (size_t)kRows * H * sizeof(float);
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(pooler_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * 2048 * 4);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  dim3 grid((H + kFeat - 1) / kFeat, (B + kRows - 1) / kRows);
  cudaError_t e = launch_k(pooler_kernel<T>, grid, dim3(256), smem, s, B, L, H, (const T*)x, (const T*)w_p, b_p,
                           pooled);
  if (e != cudaSuccess) return e;
  return launch_k(classifier_kernel<T>, dim3(B), dim3(64), 0, s, H, C, (const float*)pooled, (const T*)w_c, b_c,
                  logits);
}

}  // namespace

cudaError_t launch_head(DType dt, int B, int L, int H, int C, const void* x, const void* w_p, const float* b_p,
                        const void* w_c, const float* b_c, float* pooled, float* logits, cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  if (H > 2048) return cudaErrorInvalidValue;
  return dt == DT_BF16 ? launch_t<bf16>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s)
                       : launch_t<float>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s);
}

}  // namespace arlo
