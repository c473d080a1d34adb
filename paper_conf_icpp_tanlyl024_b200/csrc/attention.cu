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
// bf16 path (attn_tc_kernel): flash attention on the 5th-gen tensor cores —
// tcgen05.mma with S and O accumulators in TMEM, operands staged by TMA, one
// CTA per (128-query tile, head, sequence), 128-key tiles, L <= 512.
// fp32 check mode: one warp per query row, exact fp32 FFMA.
#include "common.cuh"
#include "kernels.h"
#include "ptx.cuh"

namespace arlo {
namespace {

constexpr int D = 64;        // head dim (all configs)
constexpr int AQ = 128;      // queries per q-tile (TMEM lanes)
constexpr int NQ = 2;        // q-tiles per CTA: their softmax and MMAs interleave
constexpr int AK = 128;      // keys per tile
constexpr int kMaxKT = 4;    // L <= 512
constexpr int kSoftWarps = 4 * NQ;            // warps 0..7: q-tile w/4, TMEM lane quarter w%4
constexpr int kProdWarp = kSoftWarps;         // warp 8: TMA
constexpr int kMmaWarp = kSoftWarps + 1;      // warp 9: MMA
constexpr int kAttnThreads = 32 * (kSoftWarps + 2);
constexpr int kTileBytes = 128 * 128;         // 128 rows x 64 bf16 (128 B), SWIZZLE_128B
constexpr int kPBytes = 2 * kTileBytes;       // P: 128 queries x 128 keys = two 64-key K-blocks
constexpr int kAttnSmem = 1024 + kTileBytes * (NQ + 2 * kMaxKT) + NQ * kPBytes + 256;
constexpr uint32_t kTmemCols = 512;           // S (NQ x 128) + O (NQ x 64)
constexpr uint32_t kOCol = NQ * AK;
// lazy rescale: keep a stale row max unless a tile's max exceeds it by > 2^8 in p
constexpr float kRescaleLog2 = 8.0f;
static_assert(kAttnSmem <= 232448, "attention smem");

__device__ __forceinline__ bool valid_key(int key, int len) { return key < len; }

// One CTA = (two 128-query tiles, head, sequence), 128-key tiles.  Per q-tile
// qi: S_qi,j = Q_qi K_j^T (M=128, N=128, K=64) and O_qi += P_qi,j V_j (M=128,
// N=64, K=128; V is an MN-major B operand) on tcgen05 with S_qi and O_qi in
// TMEM.  Four softmax warps per q-tile (thread = query row) read S from TMEM,
// keep a lazily-rescaled running max (O rescaled in TMEM only when a tile
// raises a row max by > 2^8 in p), write P as bf16 into 128B-swizzled smem
// (the A operand of the PV MMA) and accumulate the fp32 row sum.  The two
// q-tiles' softmax and MMAs interleave (one's softmax runs while the other's
// S/PV MMAs execute); Q, every K_j and V_j (<= 4 tiles, L <= 512) are loaded
// once by TMA and shared by both q-tiles.  Key tiles starting at >= len are
// never loaded or multiplied; keys >= len inside the last tile get p = 0.
__global__ void __launch_bounds__(kAttnThreads, 1)
attn_tc_kernel(const __grid_constant__ CUtensorMap tm, int L, int heads, const int32_t* __restrict__ lengths,
               bf16* __restrict__ o) {
  const int h = blockIdx.y, b = blockIdx.z;
  const int H = heads * D;
  const int len = __ldg(lengths + b);
  const int q0 = blockIdx.x * (NQ * AQ);
  const int row_base = b * L;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (q0 >= len) {  // every q-tile wholly padded (or empty slot): zeros
    const int rows = min(NQ * AQ, L - q0);
    for (int i = threadIdx.x; i < rows * 8; i += kAttnThreads) {
      const int r = i >> 3, c = i & 7;
      *reinterpret_cast<uint4*>(o + (size_t)(row_base + q0 + r) * H + h * D + c * 8) = make_uint4(0, 0, 0, 0);
    }
    return;
  }
  const int n_kt = (len + AK - 1) / AK;
  const int nq = (q0 + AQ < len) ? 2 : 1;  // live q-tiles (the second may be wholly padded)

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + NQ * kTileBytes;
  uint8_t* sV = sK + kMaxKT * kTileBytes;
  uint8_t* sP = sV + kMaxKT * kTileBytes;
  uint64_t* bar_k = reinterpret_cast<uint64_t*>(sP + NQ * kPBytes);
  uint64_t* bar_v = bar_k + kMaxKT;
  uint64_t* s_full = bar_v + kMaxKT;
  uint64_t* p_full = s_full + NQ;
  uint64_t* pv_done = p_full + NQ;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(pv_done + NQ);

  if (warp == kProdWarp && lane == 0) {
    ptx::tma_prefetch_desc(&tm);
    for (int j = 0; j < kMaxKT; ++j) {
      ptx::mbar_init(&bar_k[j], 1);
      ptx::mbar_init(&bar_v[j], 1);
    }
    for (int i = 0; i < NQ; ++i) {
      ptx::mbar_init(&s_full[i], 1);
      ptx::mbar_init(&p_full[i], 4);
      ptx::mbar_init(&pv_done[i], 1);
    }
    ptx::fence_mbar_init();
  }
  if (warp == kMmaWarp) ptx::tmem_alloc(tmem_slot, kTmemCols);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == kProdWarp) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0) {
      ptx::mbar_arrive_expect_tx(&bar_k[0], (nq + 1) * kTileBytes);
      for (int qi = 0; qi < nq; ++qi) ptx::tma_load_2d(sQ + qi * kTileBytes, &tm, &bar_k[0], h * D, row_base + q0 + qi * AQ);
      ptx::tma_load_2d(sK, &tm, &bar_k[0], H + h * D, row_base);
      for (int j = 1; j < n_kt; ++j) {
        ptx::mbar_arrive_expect_tx(&bar_k[j], kTileBytes);
        ptx::tma_load_2d(sK + j * kTileBytes, &tm, &bar_k[j], H + h * D, row_base + j * AK);
      }
      for (int j = 0; j < n_kt; ++j) {
        ptx::mbar_arrive_expect_tx(&bar_v[j], kTileBytes);
        ptx::tma_load_2d(sV + j * kTileBytes, &tm, &bar_v[j], 2 * H + h * D, row_base + j * AK);
      }
    }
  } else if (warp == kMmaWarp) {
    // ------------------------------------------------------------- MMA issuer
    if (lane == 0) {
      constexpr uint32_t idesc_s = ptx::idesc_bf16_f32(AQ, AK);
      constexpr uint32_t idesc_pv = ptx::idesc_bf16_f32_bmn(AQ, D);
      auto issue_s = [&](int qi, int j) {
        ptx::mbar_wait(&bar_k[j], 0);
        ptx::tc_fence_after();
        const uint32_t q_addr = ptx::smem_u32(sQ + qi * kTileBytes);
        const uint32_t k_addr = ptx::smem_u32(sK + j * kTileBytes);
#pragma unroll
        for (int k = 0; k < D / 16; ++k)
          ptx::mma_bf16_ss(tmem + qi * AK, ptx::desc_k_sw128(q_addr + k * 32), ptx::desc_k_sw128(k_addr + k * 32),
                           idesc_s, k > 0);
        ptx::mma_commit(&s_full[qi]);
      };
      for (int qi = 0; qi < nq; ++qi) issue_s(qi, 0);
      for (int j = 0; j < n_kt; ++j) {
        for (int qi = 0; qi < nq; ++qi) {
          ptx::mbar_wait(&p_full[qi], j & 1);  // P_qi,j written, S_qi buffer consumed
          ptx::mbar_wait(&bar_v[j], 0);
          ptx::tc_fence_after();
          const uint32_t p_addr = ptx::smem_u32(sP + qi * kPBytes);
          const uint32_t v_addr = ptx::smem_u32(sV + j * kTileBytes);
#pragma unroll
          for (int ks = 0; ks < AK / 16; ++ks)
            ptx::mma_bf16_ss(tmem + kOCol + qi * D,
                             ptx::desc_k_sw128(p_addr + (ks >> 2) * kTileBytes + (ks & 3) * 32),
                             ptx::desc_mn_sw128(v_addr + ks * 2048, 0), idesc_pv, (j | ks) != 0);
          ptx::mma_commit(&pv_done[qi]);
          if (j + 1 < n_kt) issue_s(qi, j + 1);
        }
      }
    }
  } else {
    // ----------------------------------------------------------------- softmax
    const int qi = warp >> 2, quarter = warp & 3;
    const int r = quarter * 32 + lane;  // query row within q-tile qi == TMEM lane
    const int qrow = q0 + qi * AQ + r;
    if (qi < nq) {
      const uint32_t t_lane = tmem + ((uint32_t)(quarter * 32) << 16);
      const uint32_t t_s = t_lane + qi * AK;
      const uint32_t t_o = t_lane + kOCol + qi * D;
      const float c = 0.125f * 1.4426950408889634f;  // 1/sqrt(64) * log2(e)
      float m = -INFINITY, l = 0.f;
      uint8_t* pbuf = sP + qi * kPBytes;
      for (int j = 0; j < n_kt; ++j) {
        ptx::mbar_wait(&s_full[qi], j & 1);
        ptx::tc_fence_after();
        const bool full_tile = (j + 1) * AK <= len;
        float tmax = -INFINITY;
#pragma unroll
        for (int ch = 0; ch < AK / 32; ++ch) {
          uint32_t v[32];
          ptx::tmem_ld_32x32b_x32(t_s + ch * 32, v);
          ptx::tmem_wait_ld();
#pragma unroll
          for (int e = 0; e < 32; ++e) {
            if (full_tile || valid_key(j * AK + ch * 32 + e, len)) tmax = fmaxf(tmax, __uint_as_float(v[e]));
          }
        }
        // P buffer (and O) are read / accumulated by PV_{j-1}: wait for it
        if (j > 0) {
          ptx::mbar_wait(&pv_done[qi], (j - 1) & 1);
          ptx::tc_fence_after();
        }
        if (j == 0) {
          m = tmax;
        } else if (__any_sync(0xffffffffu, (tmax - m) * c > kRescaleLog2)) {
          // warp-uniform branch (tcgen05.ld/st are warp-collective): rows whose
          // max rose by > 2^8 rescale O and l, the others multiply by 1
          float alpha = 1.f;
          if ((tmax - m) * c > kRescaleLog2) {
            alpha = ex2_approx((m - tmax) * c);
            l *= alpha;
            m = tmax;
          }
#pragma unroll
          for (int half = 0; half < 2; ++half) {
            uint32_t v[32];
            ptx::tmem_ld_32x32b_x32(t_o + half * 32, v);
            ptx::tmem_wait_ld();
#pragma unroll
            for (int e = 0; e < 32; ++e) v[e] = __float_as_uint(__uint_as_float(v[e]) * alpha);
            ptx::tmem_st_32x32b_x32(t_o + half * 32, v);
          }
          ptx::tmem_wait_st();
        }
        const float mc = m * c;
#pragma unroll
        for (int ch = 0; ch < AK / 32; ++ch) {
          uint32_t v[32];
          ptx::tmem_ld_32x32b_x32(t_s + ch * 32, v);
          ptx::tmem_wait_ld();
          uint32_t pk[16];
#pragma unroll
          for (int e = 0; e < 32; e += 2) {
            float p0 = ex2_approx(fmaf(__uint_as_float(v[e]), c, -mc));
            float p1 = ex2_approx(fmaf(__uint_as_float(v[e + 1]), c, -mc));
            if (!full_tile) {
              if (!valid_key(j * AK + ch * 32 + e, len)) p0 = 0.f;
              if (!valid_key(j * AK + ch * 32 + e + 1, len)) p1 = 0.f;
            }
            l += p0 + p1;
            pk[e >> 1] = pack_bf16x2(p0, p1);
          }
          // keys ch*32 .. +31 -> K-block ch/2, 16-byte chunks (ch%2)*4 .. +3 of row r
          uint8_t* rowp = pbuf + (ch >> 1) * kTileBytes + r * 128;
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const int chunk = (ch & 1) * 4 + i;
            *reinterpret_cast<uint4*>(rowp + ((chunk ^ (r & 7)) << 4)) =
                make_uint4(pk[4 * i], pk[4 * i + 1], pk[4 * i + 2], pk[4 * i + 3]);
          }
        }
        ptx::fence_proxy_async_smem();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&p_full[qi]);
      }
      // O = (sum_j P_j V_j) / l
      ptx::mbar_wait(&pv_done[qi], (n_kt - 1) & 1);
      ptx::tc_fence_after();
      const float inv = 1.f / l;
      uint4* orow = reinterpret_cast<uint4*>(o + (size_t)(row_base + qrow) * H + h * D);
#pragma unroll
      for (int half = 0; half < 2; ++half) {
        uint32_t v[32];
        ptx::tmem_ld_32x32b_x32(t_o + half * 32, v);
        ptx::tmem_wait_ld();
        if (qrow < L) {
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            uint4 u;
            u.x = pack_bf16x2(__uint_as_float(v[8 * i + 0]) * inv, __uint_as_float(v[8 * i + 1]) * inv);
            u.y = pack_bf16x2(__uint_as_float(v[8 * i + 2]) * inv, __uint_as_float(v[8 * i + 3]) * inv);
            u.z = pack_bf16x2(__uint_as_float(v[8 * i + 4]) * inv, __uint_as_float(v[8 * i + 5]) * inv);
            u.w = pack_bf16x2(__uint_as_float(v[8 * i + 6]) * inv, __uint_as_float(v[8 * i + 7]) * inv);
            orow[half * 4 + i] = u;
          }
        }
      }
    } else if (qrow < L) {
      // second q-tile wholly padded: zero rows
      uint4* orow = reinterpret_cast<uint4*>(o + (size_t)(row_base + qrow) * H + h * D);
#pragma unroll
      for (int i = 0; i < 8; ++i) orow[i] = make_uint4(0, 0, 0, 0);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == kMmaWarp) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, kTmemCols);
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
  if ((t / AQ) * AQ >= len) {  // same zero rule as the bf16 path (128-row q-tiles)
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

bool attn_plan(AttnPlan* p, DType dt, int B, int L, int heads, const void* qkv) {
  p->B = B; p->L = L; p->heads = heads; p->dt = dt; p->qkv = qkv;
  if (dt != DT_BF16) return true;
  if (L > AK * kMaxKT) return false;
  return encode_tmap_bf16_2d(&p->tm, qkv, (uint64_t)3 * heads * D, (uint64_t)B * L, 64, 128, 128);
}

cudaError_t attn_launch(const AttnPlan& p, const int32_t* lengths, void* o, cudaStream_t s) {
  if (p.B <= 0 || p.L <= 0) return cudaSuccess;
  if (p.dt == DT_BF16) {
    static bool attr = false;
    if (!attr) {
      cudaError_t e = cudaFuncSetAttribute(attn_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kAttnSmem);
      if (e != cudaSuccess) return e;
      attr = true;
    }
    dim3 grid((p.L + NQ * AQ - 1) / (NQ * AQ), p.heads, p.B);
    attn_tc_kernel<<<grid, kAttnThreads, kAttnSmem, s>>>(p.tm, p.L, p.heads, lengths, (bf16*)o);
  } else {
    const long warps = (long)p.B * p.L * p.heads;
    attn_f32_kernel<<<(unsigned)((warps + 3) / 4), 128, 0, s>>>(p.B, p.L, p.heads, (const float*)p.qkv, lengths,
                                                                 (float*)o);
  }
  return cudaGetLastError();
}

}  // namespace arlo
