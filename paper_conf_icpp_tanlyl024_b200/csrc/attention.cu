// attention.cu — step a3: padding-masked multi-head attention of a static [B, L] batch.
//
// o[b,t,head] = softmax_j(q_t . k_j / sqrt(64), j < len_b) v_j  for every
// query row t < L of sequence b (BERT self-attention [17], PAPER.md:L422;
// zero-padded static shape PAPER.md:L37, L101; mask from lengths, reading S4).
//
// The padding premise of the paper (padded positions are wasted work,
// PAPER.md:L101-103) is applied where it is free: key tiles whose first key is
// >= len_b are never loaded or multiplied, and query tiles lying wholly at
// t >= len_b are written as zeros (their rows are never read by a real token;
// reading S5).  A real query row's result depends only on keys < len_b, so it
// is bitwise identical for every runtime L >= len_b.
//
// bf16 path: flash-attention style, one CTA per (64-query tile, head,
// sequence), 4 warps x 16 query rows, S = QK^T and O += PV on mma.sync
// m16n8k16 (bf16 in, fp32 accumulate), online softmax in fp32 with exp2,
// K/V 64-key tiles double-buffered in 128B-XOR-swizzled shared memory via
// cp.async.  fp32 check mode: one warp per query row, exact fp32 FFMA.
#include "common.cuh"
#include "kernels.h"

namespace arlo {
namespace {

constexpr int D = 64;       // head dim (all configs)
constexpr int QT = 64;      // query rows per CTA
constexpr int KT = 64;      // keys per tile

__device__ __forceinline__ uint32_t swz(int row, int chunk) {  // byte offset in a [64][128B] tile
  return (uint32_t)(row * 128 + ((chunk ^ (row & 7)) << 4));
}

__device__ __forceinline__ void cp_async16(uint32_t saddr, const void* g, bool valid) {
  const int n = valid ? 16 : 0;  // zero-fill when out of range
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(saddr), "l"(g), "r"(n) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3) : "r"(addr));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3) : "r"(addr));
}
__device__ __forceinline__ void mma16816(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

// Load a [64 rows][64 dims] bf16 tile (row stride ld elements) into swizzled smem.
__device__ __forceinline__ void load_tile(uint32_t sbase, const bf16* g, int ld, int row0, int rows_valid) {
  for (int i = threadIdx.x; i < 64 * 8; i += 128) {
    const int r = i >> 3, c = i & 7;
    const bool ok = (row0 + r) < rows_valid;
    const bf16* src = g + (size_t)(ok ? r : 0) * ld + c * 8;
    cp_async16(sbase + swz(r, c), src, ok);
  }
}

__global__ void __launch_bounds__(128) attn_bf16_kernel(int L, int heads, const bf16* __restrict__ qkv,
                                                        const int32_t* __restrict__ lengths,
                                                        bf16* __restrict__ o) {
  __shared__ __align__(128) uint8_t sQ[QT * 128];
  __shared__ __align__(128) uint8_t sK[2][KT * 128];
  __shared__ __align__(128) uint8_t sV[2][KT * 128];
  const int qt = blockIdx.x, h = blockIdx.y, b = blockIdx.z;
  const int H = heads * D, ld = 3 * H;
  const int len = __ldg(lengths + b);
  const int q0 = qt * QT;
  const size_t row_base = (size_t)b * L;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (q0 >= len) {  // wholly padded query tile (or empty slot): zeros
    for (int i = threadIdx.x; i < QT * 8; i += 128) {
      const int r = i >> 3, c = i & 7;
      if (q0 + r < L)
        *reinterpret_cast<uint4*>(o + (row_base + q0 + r) * H + h * D + c * 8) = make_uint4(0, 0, 0, 0);
    }
    return;
  }
  const bf16* gq = qkv + row_base * ld + h * D;
  const bf16* gk = gq + H;
  const bf16* gv = gq + 2 * H;
  const uint32_t aQ = (uint32_t)__cvta_generic_to_shared(sQ);
  const uint32_t aK[2] = {(uint32_t)__cvta_generic_to_shared(sK[0]), (uint32_t)__cvta_generic_to_shared(sK[1])};
  const uint32_t aV[2] = {(uint32_t)__cvta_generic_to_shared(sV[0]), (uint32_t)__cvta_generic_to_shared(sV[1])};

  const int n_kt = (len + KT - 1) / KT;
  load_tile(aQ, gq + (size_t)q0 * ld, ld, q0, L);
  load_tile(aK[0], gk, ld, 0, L);
  load_tile(aV[0], gv, ld, 0, L);
  cp_async_commit();

  // softmax in base 2: p = 2^(s * scale*log2e - m)
  const float sl2 = 0.125f * 1.4426950408889634f;
  float m_i[2] = {-INFINITY, -INFINITY}, l_i[2] = {0.f, 0.f};
  float acc_o[8][4];
#pragma unroll
  for (int i = 0; i < 8; ++i) acc_o[i][0] = acc_o[i][1] = acc_o[i][2] = acc_o[i][3] = 0.f;
  uint32_t qf[4][4];
  const int g = lane >> 2, t4 = lane & 3;

  for (int kt = 0; kt < n_kt; ++kt) {
    const int cur = kt & 1;
    if (kt + 1 < n_kt) {
      load_tile(aK[cur ^ 1], gk + (size_t)(kt + 1) * KT * ld, ld, (kt + 1) * KT, L);
      load_tile(aV[cur ^ 1], gv + (size_t)(kt + 1) * KT * ld, ld, (kt + 1) * KT, L);
      cp_async_commit();
      cp_async_wait<1>();
    } else {
      cp_async_wait<0>();
    }
    __syncthreads();
    if (kt == 0) {
#pragma unroll
      for (int ks = 0; ks < 4; ++ks) {
        const int i = lane >> 3;
        const int r = warp * 16 + (i & 1) * 8 + (lane & 7);
        ldsm_x4(aQ + swz(r, ks * 2 + (i >> 1)), qf[ks][0], qf[ks][1], qf[ks][2], qf[ks][3]);
      }
    }
    // S = Q K^T for this warp's 16 rows x 64 keys
    float s[8][4];
#pragma unroll
    for (int i = 0; i < 8; ++i) s[i][0] = s[i][1] = s[i][2] = s[i][3] = 0.f;
#pragma unroll
    for (int ks = 0; ks < 4; ++ks) {
#pragma unroll
      for (int np = 0; np < 4; ++np) {  // pairs of 8-key n-tiles
        const int i = lane >> 3;
        const int r = (np * 2 + (i >> 1)) * 8 + (lane & 7);
        uint32_t b0, b1, b2, b3;
        ldsm_x4(aK[cur] + swz(r, ks * 2 + (i & 1)), b0, b1, b2, b3);
        mma16816(s[2 * np], qf[ks], b0, b1);
        mma16816(s[2 * np + 1], qf[ks], b2, b3);
      }
    }
    // mask keys >= len (only the last tile can hold any), online softmax
    const int kbase = kt * KT;
    float mx[2] = {-INFINITY, -INFINITY};
#pragma unroll
    for (int nt = 0; nt < 8; ++nt) {
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int key = kbase + nt * 8 + t4 * 2 + (e & 1);
        if (key >= len) s[nt][e] = -INFINITY;
        mx[e >> 1] = fmaxf(mx[e >> 1], s[nt][e]);
      }
    }
    float scale_o[2];
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      mx[r] = fmaxf(mx[r], __shfl_xor_sync(0xffffffffu, mx[r], 1));
      mx[r] = fmaxf(mx[r], __shfl_xor_sync(0xffffffffu, mx[r], 2));
      const float m_new = fmaxf(m_i[r], mx[r] * sl2);  // key 0 is always real: finite
      scale_o[r] = exp2f(m_i[r] - m_new);
      m_i[r] = m_new;
    }
    float rs[2] = {0.f, 0.f};
    uint32_t pf[4][4];  // P as bf16 A fragments, 4 k-steps of 16 keys
#pragma unroll
    for (int nt = 0; nt < 8; ++nt) {
      float p[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int key = kbase + nt * 8 + t4 * 2 + (e & 1);
        p[e] = key < len ? exp2f(s[nt][e] * sl2 - m_i[e >> 1]) : 0.f;
        rs[e >> 1] += p[e];
      }
      const int ks = nt >> 1, hi = nt & 1;
      pf[ks][hi * 2 + 0] = pack_bf16x2(p[0], p[1]);
      pf[ks][hi * 2 + 1] = pack_bf16x2(p[2], p[3]);
    }
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      rs[r] += __shfl_xor_sync(0xffffffffu, rs[r], 1);
      rs[r] += __shfl_xor_sync(0xffffffffu, rs[r], 2);
      l_i[r] = l_i[r] * scale_o[r] + rs[r];
    }
#pragma unroll
    for (int dt = 0; dt < 8; ++dt) {
      acc_o[dt][0] *= scale_o[0]; acc_o[dt][1] *= scale_o[0];
      acc_o[dt][2] *= scale_o[1]; acc_o[dt][3] *= scale_o[1];
    }
    // O += P V
#pragma unroll
    for (int ks = 0; ks < 4; ++ks) {
#pragma unroll
      for (int dp = 0; dp < 4; ++dp) {
        const int i = lane >> 3;
        const int r = ks * 16 + (i & 1) * 8 + (lane & 7);
        uint32_t b0, b1, b2, b3;
        ldsm_x4_t(aV[cur] + swz(r, dp * 2 + (i >> 1)), b0, b1, b2, b3);
        // A fragment order for m16n8k16: a0 (g, k 0-7), a1 (g+8, k 0-7), a2 (g, k 8-15), a3 (g+8, k 8-15)
        const uint32_t a[4] = {pf[ks][0], pf[ks][1], pf[ks][2], pf[ks][3]};
        mma16816(acc_o[2 * dp], a, b0, b1);
        mma16816(acc_o[2 * dp + 1], a, b2, b3);
      }
    }
    __syncthreads();  // buffer `cur` is refilled by the next iteration's prefetch
  }
  // normalise and store
  const float inv0 = 1.f / l_i[0], inv1 = 1.f / l_i[1];
  const int r0 = q0 + warp * 16 + g, r1 = r0 + 8;
#pragma unroll
  for (int dt = 0; dt < 8; ++dt) {
    const int col = h * D + dt * 8 + t4 * 2;
    if (r0 < L)
      *reinterpret_cast<uint32_t*>(o + (row_base + r0) * H + col) = pack_bf16x2(acc_o[dt][0] * inv0, acc_o[dt][1] * inv0);
    if (r1 < L)
      *reinterpret_cast<uint32_t*>(o + (row_base + r1) * H + col) = pack_bf16x2(acc_o[dt][2] * inv1, acc_o[dt][3] * inv1);
  }
}

// fp32 check mode: one warp per (query row, head); lane owns dims 2*lane, 2*lane+1.
__global__ void __launch_bounds__(128) attn_f32_kernel(int B, int L, int heads, const float* __restrict__ qkv,
                                                       const int32_t* __restrict__ lengths,
                                                       float* __restrict__ o) {
  const int H = heads * D, ld = 3 * H;
  const int gw = blockIdx.x * 4 + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (gw >= B * L * heads) return;
  const int h = gw % heads, row = gw / heads;
  const int b = row / L, t = row - b * L;
  const int len = __ldg(lengths + b);
  float* orow = o + (size_t)row * H + h * D;
  if ((t / QT) * QT >= len) {  // same zero rule as the bf16 path
    orow[2 * lane] = 0.f;
    orow[2 * lane + 1] = 0.f;
    return;
  }
  const float* qrow = qkv + (size_t)row * ld + h * D;
  const float q0 = qrow[2 * lane], q1 = qrow[2 * lane + 1];
  float m = -INFINITY, l = 0.f, a0 = 0.f, a1 = 0.f;
  for (int j = 0; j < len; ++j) {
    const float* krow = qkv + ((size_t)b * L + j) * ld + H + h * D;
    const float* vrow = krow + H;
    const float sc = warp_sum(fmaf(q0, krow[2 * lane], q1 * krow[2 * lane + 1])) * 0.125f;
    const float mn = fmaxf(m, sc);
    const float corr = expf(m - mn), p = expf(sc - mn);
    l = l * corr + p;
    a0 = a0 * corr + p * vrow[2 * lane];
    a1 = a1 * corr + p * vrow[2 * lane + 1];
    m = mn;
  }
  orow[2 * lane] = a0 / l;
  orow[2 * lane + 1] = a1 / l;
}

}  // namespace

cudaError_t launch_attention(DType dt, int B, int L, int heads, const void* qkv, const int32_t* lengths,
                             void* o, cudaStream_t s) {
  if (B <= 0 || L <= 0) return cudaSuccess;
  if (dt == DT_BF16) {
    dim3 grid((L + QT - 1) / QT, heads, B);
    attn_bf16_kernel<<<grid, 128, 0, s>>>(L, heads, (const bf16*)qkv, lengths, (bf16*)o);
  } else {
    const long warps = (long)B * L * heads;
    attn_f32_kernel<<<(unsigned)((warps + 3) / 4), 128, 0, s>>>(B, L, heads, (const float*)qkv, lengths,
                                                                 (float*)o);
  }
  return cudaGetLastError();
}

}  // namespace arlo
