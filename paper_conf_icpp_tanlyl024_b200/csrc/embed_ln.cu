// embed_ln.cu — steps a1 (embedding gather + LayerNorm) and a5/a8 (LayerNorm).
//
// BERT embedding and post-LN LayerNorm (Devlin et al. [17], PAPER.md:L422;
// SURVEY.md §8(a) rows a1, a5, a8; reading S3: biased variance, eps inside the
// square root; reading S4/S7: token type 0, pad positions t >= len use id 0).
//
// HBM-bound: one warp per row, 128-bit loads/stores, row held in registers,
// two-pass mean/variance from registers (no second read), warp-shuffle
// reductions, fp32 statistics, RNE conversion to bf16.  Algorithmic bytes per
// row: LN 2*H*sizeof(T) (+8H for gamma/beta, L2-resident); embedding
// 3*H*sizeof(T) read (word, pos, type) + H*sizeof(T) written.
#include "common.cuh"
#include "kernels.h"
#include "layernorm.cuh"

namespace arlo {

namespace {

#ifndef ARLO_LN_ROWS
#define ARLO_LN_ROWS 16  // rows (warps) per CTA: 16 -> 4.08 us at M=4096 vs 4.40 (8), 4.10 (32) (round-1 A/B)
#endif
constexpr int kRowsPerBlock = ARLO_LN_ROWS;  // one warp per row
#ifndef ARLO_LN_SMEM
#define ARLO_LN_SMEM 1  // stage gamma / beta in shared memory (A/B: 0 reads them through L1)
#endif
constexpr int kLnThreads = 32 * kRowsPerBlock;

// gamma / beta are weights, independent of the predecessor kernel: every CTA stages them in
// shared memory BEFORE the PDL wait, so their L2 round trip overlaps the previous kernel's tail
// instead of sitting between the row statistics and the normalisation.
__device__ __forceinline__ void stage_affine(int H, const float* __restrict__ g, const float* __restrict__ b,
                                             float* sg, float* sb) {
  for (int i = threadIdx.x * 4; i < H; i += blockDim.x * 4) {
    *reinterpret_cast<float4*>(sg + i) = __ldg(reinterpret_cast<const float4*>(g + i));
    *reinterpret_cast<float4*>(sb + i) = __ldg(reinterpret_cast<const float4*>(b + i));
  }
  __syncthreads();
}

template <typename T, int MAXV>
__global__ void __launch_bounds__(kLnThreads) layernorm_kernel(int M, int H, const T* __restrict__ in,
                                                        const float* __restrict__ g,
                                                        const float* __restrict__ b, float eps,
                                                        T* __restrict__ out) {
  constexpr int VN = Vec<T>::N;
#if ARLO_LN_SMEM
  extern __shared__ float s_aff[];  // [gamma H | beta H]
  pdl_launch_dependents();
  stage_affine(H, g, b, s_aff, s_aff + H);
  const float* ga = s_aff;
  const float* be = s_aff + H;
#else  // A/B: gamma / beta straight from L1/L2 (no shared memory: CTAs fit beside a GEMM's)
  pdl_launch_dependents();
  const float* ga = g;
  const float* be = b;
#endif
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int row = blockIdx.x * kRowsPerBlock + (threadIdx.x >> 5);
  if (row >= M) return;
  const int nvec = H / VN;
  const T* src = in + (size_t)row * H;
  float v[MAXV][VN];
#pragma unroll
  for (int i = 0; i < MAXV; ++i)
    if (lane + 32 * i < nvec) Vec<T>::load(src + (lane + 32 * i) * VN, v[i], true);  // predecessor's output
  ln_finish<T, MAXV>(v, nvec, H, lane, ga, be, eps, out + (size_t)row * H);
}

template <typename T, int MAXV>
__global__ void __launch_bounds__(kLnThreads) embed_ln_kernel(int B, int L, int H, int vocab,
                                                       const int32_t* __restrict__ ids,
                                                       const int32_t* __restrict__ lengths,
                                                       const T* __restrict__ word,
                                                       const T* __restrict__ pos,
                                                       const T* __restrict__ type,
                                                       const float* __restrict__ g,
                                                       const float* __restrict__ b, float eps,
                                                       T* __restrict__ out, int32_t* err_flag) {
  constexpr int VN = Vec<T>::N;
  extern __shared__ float s_aff[];  // [gamma H | beta H]
  pdl_launch_dependents();
  stage_affine(H, g, b, s_aff, s_aff + H);
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int row = blockIdx.x * kRowsPerBlock + (threadIdx.x >> 5);
  if (row >= B * L) return;
  const int bi = row / L, t = row - bi * L;
  int id = 0;
  if (t < __ldg(lengths + bi)) {
    id = __ldg(ids + row);
    if (id < 0 || id >= vocab) {
      if (lane == 0 && err_flag) *err_flag = 1;
      id = 0;
    }
  }
  const int nvec = H / VN;
  const T* wr = word + (size_t)id * H;
  const T* pr = pos + (size_t)t * H;
  float v[MAXV][VN];
#pragma unroll
  for (int i = 0; i < MAXV; ++i) {
    const int vi = lane + 32 * i;
    if (vi < nvec) {
      float a[VN], p[VN], c[VN];
      Vec<T>::load(wr + vi * VN, a);
      Vec<T>::load(pr + vi * VN, p);
      Vec<T>::load(type + vi * VN, c);
#pragma unroll
      for (int j = 0; j < VN; ++j) v[i][j] = a[j] + p[j] + c[j];
    }
  }
  ln_finish<T, MAXV>(v, nvec, H, lane, s_aff, s_aff + H, eps, out + (size_t)row * H);
}

// LayerNorm fold (runtime.cu): a GEMM consuming LN(y) = (y - mu) rstd * gamma + beta runs on y with
//   W'[n, k] = bf16(W[n, k] * gamma[k]),  s[n] = sum_k W'[n, k],  c[n] = sum_k W[n, k] beta[k] + b[n]
// and the epilogue out = rstd * acc - rstd * mu * s[n] + c[n].  One warp per output row n; the sums
// in fp64 (lane-strided, then a fixed shuffle tree), computed once per weight set.
__global__ void __launch_bounds__(128) fold_weights_kernel(int N, int K, const bf16* __restrict__ W,
                                                           const float* __restrict__ gamma,
                                                           const float* __restrict__ beta, const float* __restrict__ b,
                                                           bf16* __restrict__ Wf, float* __restrict__ s,
                                                           float* __restrict__ c) {
  const int n = blockIdx.x * 4 + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (n >= N) return;
  double ss = 0.0, cc = 0.0;
  for (int k = lane; k < K; k += 32) {
    const float w = __bfloat162float(W[(size_t)n * K + k]);
    const bf16 wf = __float2bfloat16_rn(w * gamma[k]);
    Wf[(size_t)n * K + k] = wf;
    ss += (double)__bfloat162float(wf);
    cc += (double)w * (double)beta[k];
  }
  for (int o = 16; o > 0; o >>= 1) {
    ss += __shfl_xor_sync(0xffffffffu, ss, o);
    cc += __shfl_xor_sync(0xffffffffu, cc, o);
  }
  if (lane == 0) {
    s[n] = (float)ss;
    c[n] = (float)(cc + (double)b[n]);
  }
}

}  // namespace

cudaError_t launch_fold_weights(int N, int K, const void* W, const float* gamma, const float* beta, const float* b,
                                void* Wf, float* s, float* c, cudaStream_t st) {
  fold_weights_kernel<<<(N + 3) / 4, 128, 0, st>>>(N, K, (const bf16*)W, gamma, beta, b, (bf16*)Wf, s, c);
  return cudaGetLastError();
}

#define ARLO_MAXV_SWITCH(maxv, ...)            \
  switch (maxv) {                              \
    case 1: { constexpr int MV = 1; __VA_ARGS__; } break; \
    case 2: { constexpr int MV = 2; __VA_ARGS__; } break; \
    case 3: { constexpr int MV = 3; __VA_ARGS__; } break; \
    case 4: { constexpr int MV = 4; __VA_ARGS__; } break; \
    case 6: { constexpr int MV = 6; __VA_ARGS__; } break; \
    case 8: { constexpr int MV = 8; __VA_ARGS__; } break; \
    default: return cudaErrorInvalidValue;     \
  }

static int round_maxv(int nvec) {
  int m = (nvec + 31) / 32;
  if (m <= 4) return m;
  if (m <= 6) return 6;
  if (m <= 8) return 8;
  return -1;
}

cudaError_t launch_layernorm(DType dt, int M, int H, const void* in, const float* g, const float* b,
                             float eps, void* out, cudaStream_t s) {
  if (M <= 0) return cudaSuccess;
  const int vn = dt == DT_BF16 ? 8 : 4;
  if (H % vn) return cudaErrorInvalidValue;
  const int maxv = round_maxv(H / vn);
  dim3 grid((M + kRowsPerBlock - 1) / kRowsPerBlock), block(kLnThreads);
  if (dt == DT_BF16) {
    ARLO_MAXV_SWITCH(maxv, return launch_k(layernorm_kernel<bf16, MV>, grid, block, ARLO_LN_SMEM ? 8 * H : 0, s,
        M, H, (const bf16*)in, g, b, eps, (bf16*)out));
  } else {
    ARLO_MAXV_SWITCH(maxv, return launch_k(layernorm_kernel<float, MV>, grid, block, ARLO_LN_SMEM ? 8 * H : 0, s,
        M, H, (const float*)in, g, b, eps, (float*)out));
  }
  return cudaGetLastError();
}

cudaError_t launch_embed_ln(DType dt, int B, int L, int H, int vocab, const int32_t* ids,
                            const int32_t* lengths, const void* word, const void* pos,
                            const void* type, const float* g, const float* b, float eps, void* out,
                            int32_t* err_flag, cudaStream_t s) {
  if (B * L <= 0) return cudaSuccess;
  const int vn = dt == DT_BF16 ? 8 : 4;
  if (H % vn) return cudaErrorInvalidValue;
  const int maxv = round_maxv(H / vn);
  dim3 grid((B * L + kRowsPerBlock - 1) / kRowsPerBlock), block(kLnThreads);
  if (dt == DT_BF16) {
    ARLO_MAXV_SWITCH(maxv, return launch_k(embed_ln_kernel<bf16, MV>, grid, block, 8 * H, s,
        B, L, H, vocab, ids, lengths, (const bf16*)word, (const bf16*)pos, (const bf16*)type, g, b,
        eps, (bf16*)out, err_flag));
  } else {
    ARLO_MAXV_SWITCH(maxv, return launch_k(embed_ln_kernel<float, MV>, grid, block, 8 * H, s,
        B, L, H, vocab, ids, lengths, (const float*)word, (const float*)pos, (const float*)type, g,
        b, eps, (float*)out, err_flag));
  }
  return cudaGetLastError();
}

}  // namespace arlo
