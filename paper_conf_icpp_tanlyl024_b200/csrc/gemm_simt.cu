// gemm_simt.cu — FFMA GEMM with the same fused epilogues.
//
// out[M,N] = epi(A[M,K] W[N,K]^T + bias) in true fp32 FFMA (no TF32): the
// fp32 "check mode" of the north_star (logits within 1e-4 of the fp64
// oracle).  Not a performance path: the bf16 runtime uses gemm_tc.cu.
// Classic 64x64x16 shared-memory tiling, 256 threads, 4x4 outputs each, K
// reduced strictly in increasing order.
#include "common.cuh"
#include "kernels.h"

namespace arlo {
namespace {

constexpr int TM = 64, TN = 64, TK = 16;

template <typename T, int EPI>
__global__ void __launch_bounds__(256) gemm_simt_kernel(int M, int N, int K, const T* __restrict__ A,
                                                        const T* __restrict__ W,
                                                        const float* __restrict__ bias,
                                                        const T* __restrict__ resid,
                                                        T* __restrict__ out) {
  __shared__ float As[TK][TM + 4];
  __shared__ float Ws[TK][TN + 4];
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  const int m0 = blockIdx.y * TM, n0 = blockIdx.x * TN;
  float acc[4][4] = {};
  // loader mapping: 256 threads x 4 elements = 64 rows x 16 k
  const int lr = threadIdx.x / 4, lk = (threadIdx.x % 4) * 4;
  for (int k0 = 0; k0 < K; k0 += TK) {
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int am = m0 + lr;
      As[lk + j][lr] = am < M ? Elem<T>::to_f(A[(size_t)am * K + k0 + lk + j]) : 0.f;
      Ws[lk + j][lr] = Elem<T>::to_f(W[(size_t)(n0 + lr) * K + k0 + lk + j]);
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < TK; ++k) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        a[i] = As[k][ty * 4 + i];
        b[i] = Ws[k][tx * 4 + i];
      }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int m = m0 + ty * 4 + i;
    if (m >= M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int n = n0 + tx * 4 + j;
      float v = acc[i][j] + bias[n];
      if (EPI == EPI_BIAS_GELU) v = gelu_erf(v);
      if (EPI == EPI_BIAS_RESID) v += Elem<T>::to_f(resid[(size_t)m * N + n]);
      out[(size_t)m * N + n] = Elem<T>::from_f(v);
    }
  }
}

template <typename T>
cudaError_t launch_t(int M, int N, int K, const void* A, const void* W, const float* bias,
                     const void* resid, void* out, int epi, cudaStream_t s) {
  dim3 grid(N / TN, (M + TM - 1) / TM), block(256);
  const T* a = (const T*)A;
  const T* w = (const T*)W;
  const T* r = (const T*)resid;
  T* o = (T*)out;
  switch (epi) {
    case EPI_BIAS: gemm_simt_kernel<T, EPI_BIAS><<<grid, block, 0, s>>>(M, N, K, a, w, bias, r, o); break;
    case EPI_BIAS_GELU: gemm_simt_kernel<T, EPI_BIAS_GELU><<<grid, block, 0, s>>>(M, N, K, a, w, bias, r, o); break;
    case EPI_BIAS_RESID: gemm_simt_kernel<T, EPI_BIAS_RESID><<<grid, block, 0, s>>>(M, N, K, a, w, bias, r, o); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_gemm_simt(DType dt, int M, int N, int K, const void* A, const void* W,
                             const float* bias, const void* resid, void* out, int epi,
                             cudaStream_t s) {
  if (M <= 0) return cudaSuccess;
  if (N % TN || K % TK) return cudaErrorInvalidValue;
  return dt == DT_BF16 ? launch_t<bf16>(M, N, K, A, W, bias, resid, out, epi, s)
                       : launch_t<float>(M, N, K, A, W, bias, resid, out, epi, s);
}

}  // namespace arlo
