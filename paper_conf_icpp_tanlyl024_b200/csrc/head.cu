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

// 16-byte vectors of T: VN = 16 / sizeof(T) elements.
template <typename T>
__device__ __forceinline__ void unpack16(const uint4& u, float* f) {
  if constexpr (sizeof(T) == 2) {
    float2 a = unpack_bf16x2(u.x), b = unpack_bf16x2(u.y), c = unpack_bf16x2(u.z), d = unpack_bf16x2(u.w);
    f[0] = a.x; f[1] = a.y; f[2] = b.x; f[3] = b.y; f[4] = c.x; f[5] = c.y; f[6] = d.x; f[7] = d.y;
  } else {
    f[0] = __uint_as_float(u.x); f[1] = __uint_as_float(u.y); f[2] = __uint_as_float(u.z); f[3] = __uint_as_float(u.w);
  }
}

// MAXV = 16-byte vectors per lane of one H-row, ceil(H * sizeof(T) / 512): a warp's W row and
// (kRows * 32 == 256 threads) a thread's share of the kRows staged CLS rows both take MAXV
// registers of 16 B, so the register count follows H (173 registers at a fixed 16 limited the
// pooler to one CTA per SM: 31 us at B = 32).

// The warp's W_p row is loaded into registers BEFORE the PDL wait (weights never depend
// on the previous kernel); the CLS rows are then staged with every 16-byte load of a thread
// issued before any shared-memory store (one L2 round trip, not one per element).
// Classifier logit (sequence row, label c) by one warp: lane-strided 16-byte loads of the W_c row
// and of the pooled row, fixed fma order, then warp_sum.  Shared by the classifier kernel and the
// pooler's last-CTA classifier, so both give a sequence's logits bitwise alike.
template <typename T, int MAXV>
__device__ __forceinline__ float classifier_dot(const uint4 (&wv)[MAXV], const float* p, int nvec, int lane) {
  constexpr int VN = 16 / sizeof(T);
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < MAXV; ++i) {
    const int v = lane + 32 * i;
    if (v < nvec) {
      float w[VN];
      unpack16<T>(wv[i], w);
#pragma unroll
      for (int e = 0; e < VN; e += 4) {
        const uint4 qu = ld_dep_v4(p + v * VN + e);
        const float4 q = make_float4(__uint_as_float(qu.x), __uint_as_float(qu.y), __uint_as_float(qu.z),
                                     __uint_as_float(qu.w));
        s = fmaf(w[e], q.x, s);
        s = fmaf(w[e + 1], q.y, s);
        s = fmaf(w[e + 2], q.z, s);
        s = fmaf(w[e + 3], q.w, s);
      }
    }
  }
  return warp_sum(s);
}

template <typename T, int MAXV>
__device__ __forceinline__ void load_wrow(uint4 (&wv)[MAXV], const T* __restrict__ w, int row, int H, int lane) {
  constexpr int VN = 16 / sizeof(T);
  const uint4* wr = reinterpret_cast<const uint4*>(w + (size_t)row * H);
#pragma unroll
  for (int i = 0; i < MAXV; ++i)
    if (lane + 32 * i < H / VN) wv[i] = __ldg(wr + lane + 32 * i);
}

// HeadCls (runtimes): the classifier runs in the pooler's grid.  Every CTA of a sequence group
// (blockIdx.y) counts itself in cnt[blockIdx.y] after its pooled features are written (release);
// the last one (acquire) computes the group's logits with classifier_dot and resets the counter
// for the next replay.  One dependent launch less per forward.
struct HeadCls {
  const void* w_c;
  const float* b_c;
  float* logits;
  int C;
  unsigned* cnt;  // [ceil(B / 8)] zero-initialised, or nullptr: separate classifier kernel
};

template <typename T, int MAXV>
__global__ void __launch_bounds__(256) pooler_kernel(int B, int L, int H, const T* __restrict__ x,
                                                     const T* __restrict__ w_p, const float* __restrict__ b_p,
                                                     float* __restrict__ pooled, const HeadLn ln, const HeadCls hc) {
  // [kRows][nvec] raw 16-byte vectors of T: lane-consecutive vectors are bank-conflict free
  // (fp32 staging with 8 floats per lane put lanes 4 apart on the same banks: 8-way STS,
  // 2x LDS.128 wavefronts; the pooler was shared-memory bound at 22 us for b = 32)
  extern __shared__ uint4 xs[];
  constexpr int VN = 16 / sizeof(T);
  pdl_launch_dependents();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int j = blockIdx.x * kFeat + warp;
  const int nvec = H / VN;  // 16-byte vectors per row
  uint4 wv[MAXV];
  if (j < H) {
    const uint4* wr = reinterpret_cast<const uint4*>(w_p + (size_t)j * H);
#pragma unroll
    for (int i = 0; i < MAXV; ++i)
      if (lane + 32 * i < nvec) wv[i] = __ldg(wr + lane + 32 * i);
  }
  pdl_wait();
  const int b0 = blockIdx.y * kRows;
  const int nb = min(kRows, B - b0);
  // LayerNorm fold: the CLS rows are the last layer's un-normalised output y; normalise them while
  // staging (x = bf16((y - mean) rstd * gamma + beta), layernorm.cuh's per-element arithmetic)
  __shared__ float2 s_ms[kRows];
  if (sizeof(T) == 2 && ln.st != nullptr) {
    if (threadIdx.x < nb)
      s_ms[threadIdx.x] = fold_row_stats(ln.st, (size_t)(b0 + threadIdx.x) * L, ln.st_ld, H / 32, H, ln.eps);
    __syncthreads();
  }
  {
    constexpr int kPer = MAXV;  // kRows * nvec / 256 <= MAXV vectors per thread
    static_assert(kRows * 32 == 256, "one staged vector per thread per 32 of a row");
    uint4 u[kPer];
#pragma unroll
    for (int t = 0; t < kPer; ++t) {
      const int i = threadIdx.x + 256 * t;
      const int r = i / nvec, c = i - r * nvec;
      if (r < nb) u[t] = ld_dep_v4(reinterpret_cast<const uint4*>(x + (size_t)(b0 + r) * L * H) + c);
    }
#pragma unroll
    for (int t = 0; t < kPer; ++t) {
      const int i = threadIdx.x + 256 * t;
      const int r = i / nvec, c = i - r * nvec;
      if (sizeof(T) == 2 && ln.st != nullptr && r < nb) {
        const float2 ms = s_ms[r];
        uint32_t w[4] = {u[t].x, u[t].y, u[t].z, u[t].w};
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int col = c * 8 + 2 * e;
          const float2 y = unpack_bf16x2(w[e]);
          const float o0 = __fmaf_rn(__fmul_rn(__fsub_rn(y.x, ms.x), ms.y), __ldg(ln.gamma + col), __ldg(ln.beta + col));
          const float o1 = __fmaf_rn(__fmul_rn(__fsub_rn(y.y, ms.x), ms.y), __ldg(ln.gamma + col + 1),
                                     __ldg(ln.beta + col + 1));
          w[e] = pack_bf16x2(o0, o1);
        }
        u[t] = make_uint4(w[0], w[1], w[2], w[3]);
      }
      if (r < kRows) xs[r * nvec + c] = r < nb ? u[t] : make_uint4(0, 0, 0, 0);
    }
  }
  __syncthreads();
  if (j < H) {
  float acc[kRows];
#pragma unroll
  for (int r = 0; r < kRows; ++r) acc[r] = 0.f;
#pragma unroll
  for (int i = 0; i < MAXV; ++i) {
    const int v = lane + 32 * i;
    if (v < nvec) {
      float w[VN];
      unpack16<T>(wv[i], w);
#pragma unroll
      for (int r = 0; r < kRows; ++r) {
        float xv[VN];
        unpack16<T>(xs[r * nvec + v], xv);
#pragma unroll
        for (int e = 0; e < VN; ++e) acc[r] = fmaf(w[e], xv[e], acc[r]);
      }
    }
  }
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    const float v = warp_sum(acc[r]);
    if (lane == 0 && r < nb) pooled[(size_t)(b0 + r) * H + j] = tanhf(v + b_p[j]);
  }
  }
  if (hc.cnt == nullptr) return;
  __shared__ int s_last;
  __syncthreads();  // this CTA's pooled features are written
  if (threadIdx.x == 0) {
    __threadfence();
    s_last = atomicAdd(hc.cnt + blockIdx.y, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  for (int t = warp; t < nb * hc.C; t += kFeat) {
    const int r = t / hc.C, c = t - r * hc.C;
    uint4 wv[MAXV];
    load_wrow<T, MAXV>(wv, (const T*)hc.w_c, c, H, lane);
    const float s = classifier_dot<T, MAXV>(wv, pooled + (size_t)(b0 + r) * H, nvec, lane);
    if (lane == 0) hc.logits[(size_t)(b0 + r) * hc.C + c] = s + hc.b_c[c];
  }
  if (threadIdx.x == 0) hc.cnt[blockIdx.y] = 0;  // (every CTA of the group has counted itself)
}

// One warp per (sequence, label): 16-byte loads of the W_c row (before the PDL wait) and of
// the pooled row, fixed lane-strided order then a warp_sum, so logits do not depend on B.
template <typename T, int MAXV>
__global__ void __launch_bounds__(64) classifier_kernel(int H, int C, const float* __restrict__ pooled,
                                                        const T* __restrict__ w_c, const float* __restrict__ b_c,
                                                        float* __restrict__ logits) {
  constexpr int VN = 16 / sizeof(T);
  pdl_launch_dependents();
  const int b = blockIdx.x;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nvec = H / VN;
  for (int c = warp; c < C; c += 2) {
    uint4 wv[MAXV];
    load_wrow<T, MAXV>(wv, w_c, c, H, lane);
    if (c == warp) pdl_wait();
    const float s = classifier_dot<T, MAXV>(wv, pooled + (size_t)b * H, nvec, lane);
    if (lane == 0) logits[(size_t)b * C + c] = s + b_c[c];
  }
  if (warp >= C) pdl_wait();
}

template <typename T, int MAXV>
cudaError_t launch_t(int B, int L, int H, int C, const void* x, const void* w_p, const float* b_p, const void* w_c,
                     const float* b_c, float* pooled, float* logits, cudaStream_t s, HeadLn ln, unsigned* cnt) {
  const size_t smem = (size_t)kRows * H * sizeof(T);
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t e = once_per_device(attr_done, [] {
    cudaError_t r = cudaFuncSetAttribute(pooler_kernel<T, MAXV>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         kRows * 2048 * 4);
    if (r == cudaSuccess)
      r = cudaFuncSetAttribute(pooler_kernel<T, MAXV>, cudaFuncAttributePreferredSharedMemoryCarveout,
                               cudaSharedmemCarveoutMaxShared);
    return r; });
  if (e != cudaSuccess) return e;
  dim3 grid((H + kFeat - 1) / kFeat, (B + kRows - 1) / kRows);
  e = launch_k(pooler_kernel<T, MAXV>, grid, dim3(256), smem, s, B, L, H, (const T*)x, (const T*)w_p,
                           b_p, pooled, ln, HeadCls{w_c, b_c, logits, C, cnt});
  if (e != cudaSuccess || cnt != nullptr) return e;
  return launch_k(classifier_kernel<T, MAXV>, dim3(B), dim3(64), 0, s, H, C, (const float*)pooled, (const T*)w_c,
                  b_c, logits);
}

template <typename T>
cudaError_t launch_dt(int B, int L, int H, int C, const void* x, const void* w_p, const float* b_p, const void* w_c,
                      const float* b_c, float* pooled, float* logits, cudaStream_t s, HeadLn ln, unsigned* cnt) {
  const int maxv = (H * (int)sizeof(T) + 511) / 512;
  switch (maxv) {
    case 1: return launch_t<T, 1>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s, ln, cnt);
    case 2: return launch_t<T, 2>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s, ln, cnt);
    case 3: return launch_t<T, 3>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s, ln, cnt);
    case 4: return launch_t<T, 4>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s, ln, cnt);
    case 5: case 6: return launch_t<T, 6>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s, ln, cnt);
    case 7: case 8: return launch_t<T, 8>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s, ln, cnt);
    default: return launch_t<T, 16>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s, ln, cnt);
  }
}

}  // namespace

cudaError_t launch_head(DType dt, int B, int L, int H, int C, const void* x, const void* w_p, const float* b_p,
                        const void* w_c, const float* b_c, float* pooled, float* logits, cudaStream_t s, HeadLn ln,
                        unsigned* cnt) {
  if (B <= 0) return cudaSuccess;
  if (H > 2048 || H % 8) return cudaErrorInvalidValue;
  return dt == DT_BF16 ? launch_dt<bf16>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s, ln, cnt)
                       : launch_dt<float>(B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, s, HeadLn{}, cnt);
}

}  // namespace arlo
