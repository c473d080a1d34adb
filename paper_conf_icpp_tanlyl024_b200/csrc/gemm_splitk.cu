// gemm_splitk.cu — split-K weight-streaming GEMM of the latency (batch-1) runtimes
// (steps a2, a4, a6, a7 at small M = b*L).
//
//   out[M,N] = epi(A[M,K] W[N,K]^T + bias[N]),  epi in {identity, GELU_erf, +residual}
//
// The paper's runtimes serve one request at a time ("we set the batch size for all
// runtimes to 1", §5).  At M = L <= 512 rows a projection reads its whole
// weight matrix for 2*M flops per weight element: far below the B200 ridge (SURVEY.md
// §8(d)), so it is bound by how fast the weights stream from HBM, and, when only a few
// dozen CTAs each walk the full K (the tile kernels: N/BN CTAs), by the serial chain of
// K/16 tcgen05.mma of each CTA.  This kernel spreads every weight matrix over ~148 CTAs:
//
//  * a thread-block cluster of S CTAs per (BN-column tile, 128-row block); CTA s of the
//    cluster streams the W slice [n0, n0+BN) x [s*kc, (s+1)*kc) (kc = K/S) and the same
//    K range of A through a TMA ring (W requested before the PDL wait: weights never depend
//    on the previous kernel), and accumulates its partial sum in TMEM (M=128 tcgen05.mma,
//    K=16 steps);
//  * each CTA copies its fp32 partial to its own shared memory (over its operand ring, idle by
//    then); after a cluster barrier the
//    rows are reduced over distributed shared memory in the FIXED order
//    ((p_0 + p_1) + p_2) + ... + p_{S-1}, each row quad by exactly one CTA, then the shared
//    epilogue (bias, GELU, residual, or the LATENCY family's residual + on-the-fly LayerNorm
//    with the output's granule statistics; RNE to bf16; epilogue.cuh) and a direct store.
//
// S = splitk_factor(N, K) depends on the weight shape only, never on M, so every runtime of
// the latency family produces each output element with the same sequence of fp32 additions:
// a request's logits are bitwise equal across the latency runtimes of every L (the cross-L
// contract of SURVEY.md §7 holds within the family; the throughput family, whose tile
// kernels add the K chain in one accumulator, agrees to bf16 rounding).  The tile width
// BN may vary with M: it changes which CTA computes an element, not how.
#include <cuda.h>

#include <cstdlib>

#include "common.cuh"
#include "epilogue.cuh"
#include "kernels.h"
#include "ptx.cuh"

namespace arlo {
namespace {

constexpr int BM = 128, BK = 64;
constexpr int kThreads = 192;      // warps 0-3: TMEM -> smem partial; warp 4: TMA; warp 5: MMA; all: reduction
constexpr int kMaxSplits = 8;      // portable cluster size
constexpr int kSmemOptIn = 232448;  // 227 KB
constexpr int kMaxStages = 12;

template <int BN>
struct SkRed {
  static constexpr int LD = BN + 4;  // fp32 row stride of the partial (spreads rows over banks)
  static constexpr int BYTES = BM * LD * 4;
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int TMEM_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
};

template <int BN, int EPI>
__global__ void __launch_bounds__(kThreads, 1)
gemm_splitk_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   bf16* __restrict__ out, int M, int N, int kc, int a_rows, int stages, int a_stage,
                   const float* __restrict__ bias, const bf16* __restrict__ resid, int ldr, const FoldArgs fa) {
  using R = SkRed<BN>;
  // EPI_RESID_LN: (mean, rstd) of the residual rows of this 128-row block, from their granule
  // statistics (fa.st_in); rstd < 0 marks a plain residual (no statistics: layer 0's input)
  __shared__ float2 rs[EPI == EPI_RESID_LN ? BM : 1];
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = sA + stages * a_stage;
  // [BM][LD] fp32 partial, over the operand ring: it is written only after the last MMA has
  // completed (tfull), when no stage is read or written any more
  float* red = reinterpret_cast<float*>(smem);
  const int ring = stages * (a_stage + R::B_BYTES);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + (ring > R::BYTES ? ring : R::BYTES));
  uint64_t* empty = full + stages;
  uint64_t* tfull = empty + stages;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tfull + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t S = gridDim.x;  // the cluster spans x
  const uint32_t rank = ptx::cluster_ctarank();
  const int n0 = blockIdx.y * BN, m0 = blockIdx.z * BM;
  const int k0 = (int)rank * kc;
  const int kblocks = kc / BK;
  const uint32_t stage_tx = (uint32_t)(a_rows * BK * 2 + R::B_BYTES);

  if (warp == 4 && lane == 0) {
    ptx::tma_prefetch_desc(&tmA);
    ptx::tma_prefetch_desc(&tmB);
    for (int i = 0; i < stages; ++i) {
      ptx::mbar_init(&full[i], 1);
      ptx::mbar_init(&empty[i], 1);
    }
    ptx::mbar_init(tfull, 1);
    ptx::fence_mbar_init();
  }
  if (warp == 5) ptx::tmem_alloc(tmem_slot, R::TMEM_COLS);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_launch_dependents();

  if (warp == 4) {
    if (lane == 0) {
      // the whole W slice of this CTA (up to `stages` k-blocks) before the PDL wait, A after it
      const int pre = kblocks < stages ? kblocks : stages;
      for (int kb = 0; kb < pre; ++kb) {
        ptx::mbar_arrive_expect_tx(&full[kb], stage_tx);
        ptx::tma_load_2d(sB + kb * R::B_BYTES, &tmB, &full[kb], k0 + kb * BK, n0);
      }
      pdl_wait();
      for (int kb = 0; kb < pre; ++kb) ptx::tma_load_2d(sA + kb * a_stage, &tmA, &full[kb], k0 + kb * BK, m0);
      int stage = pre % stages;
      uint32_t phase = pre == stages ? 1 : 0;
      for (int kb = pre; kb < kblocks; ++kb) {
        ptx::mbar_wait(&empty[stage], phase ^ 1);
        ptx::mbar_arrive_expect_tx(&full[stage], stage_tx);
        ptx::tma_load_2d(sB + stage * R::B_BYTES, &tmB, &full[stage], k0 + kb * BK, n0);
        ptx::tma_load_2d(sA + stage * a_stage, &tmA, &full[stage], k0 + kb * BK, m0);
        if (++stage == stages) { stage = 0; phase ^= 1; }
      }
    }
  } else if (warp == 5) {
    // converged warp, one elected lane issues (see gemm_skinny_kernel)
    constexpr uint32_t idesc = ptx::idesc_bf16_f32(BM, BN);
    int stage = 0;
    uint32_t phase = 0;
#pragma unroll 1
    for (int kb = 0; kb < kblocks; ++kb) {
      ptx::mbar_wait(&full[stage], phase);
      ptx::tc_fence_after();
      const uint32_t a_addr = ptx::smem_u32(sA + stage * a_stage);
      const uint32_t b_addr = ptx::smem_u32(sB + stage * R::B_BYTES);
#pragma unroll
      for (int k = 0; k < BK / 16; ++k)
        ptx::mma_bf16_ss_w(tmem, ptx::desc_k_sw128(a_addr + k * 32), ptx::desc_k_sw128(b_addr + k * 32), idesc,
                           (kb | k) != 0);
      ptx::mma_commit_w(&empty[stage]);
      if (++stage == stages) { stage = 0; phase ^= 1; }
    }
    ptx::mma_commit_w(tfull);
  } else {
    if constexpr (EPI == EPI_RESID_LN) {  // the residual rows' statistics, overlapping the main loop
      pdl_wait();
      const int grow = m0 + warp * 32 + lane;
      rs[warp * 32 + lane] = fa.st_in != nullptr && grow < M
                                 ? fold_row_stats(fa.st_in, (size_t)grow * fa.st_in_stride, fa.st_ld, N / 32, N, fa.eps)
                                 : make_float2(0.f, -1.f);
    }
    // partial -> own shared memory: thread = row (TMEM lane), BN fp32 columns
    ptx::mbar_wait(tfull, 0);
    ptx::tc_fence_after();
    const int row = warp * 32 + lane;
    const uint32_t t_row = tmem + ((uint32_t)(warp * 32) << 16);
#pragma unroll
    for (int c0 = 0; c0 < BN; c0 += 16) {
      uint32_t r[16];
      ptx::tmem_ld_32x32b_x16(t_row + c0, r);
      ptx::tmem_wait_ld();
      float4* dst = reinterpret_cast<float4*>(red + row * R::LD + c0);
#pragma unroll
      for (int j = 0; j < 4; ++j)
        dst[j] = make_float4(__uint_as_float(r[4 * j]), __uint_as_float(r[4 * j + 1]), __uint_as_float(r[4 * j + 2]),
                             __uint_as_float(r[4 * j + 3]));
    }
  }
  ptx::tc_fence_before();
  ptx::cluster_sync();  // every CTA's partial is in its shared memory and visible cluster-wide
  pdl_wait();           // (residual reads below; a no-op once passed)

  // fixed-order reduction over the cluster: row quads striped over the S CTAs
  constexpr int Q = BN / 4;
  const int rows_valid = M - m0 < BM ? M - m0 : BM;
  const int items = rows_valid * Q;
  for (int it = (int)rank * kThreads + threadIdx.x; it < items; it += (int)S * kThreads) {
    const int row = it / Q, q = it - row * Q;
    const float* src = red + row * R::LD + q * 4;
    float4 acc = ptx::ld_shared_cluster_v4(ptx::mapa_shared(src, 0));
    for (uint32_t s = 1; s < S; ++s) {
      const float4 v = ptx::ld_shared_cluster_v4(ptx::mapa_shared(src, s));
      acc.x += v.x;
      acc.y += v.y;
      acc.z += v.z;
      acc.w += v.w;
    }
    const int grow = m0 + row, col = n0 + q * 4;
    const float4 b4 = __ldg(reinterpret_cast<const float4*>(bias + col));
    uint32_t ua = 0, ub = 0;
    if (EPI == EPI_BIAS_RESID || EPI == EPI_RESID_LN) {
      const uint2 u = ld_dep_v2(resid + (size_t)grow * ldr + col);
      ua = u.x;
      ub = u.y;
    }
    uint32_t p0, p1;
    if constexpr (EPI == EPI_RESID_LN) {
      // y = (acc + b) + LN(r) (epilogue.cuh), then the (sum y, sum y^2) of the 32-column granule of
      // the bf16 outputs: each quad's sums in column order, then an xor tree over the granule's 8
      // quads, which are 8 consecutive lanes (Q and kThreads are multiples of 8, so a granule is
      // either wholly inside this iteration or wholly outside it).  A function of N and K only, so
      // every runtime of the family produces each statistic alike.
      const float4 g4 = fa.v1 ? __ldg(reinterpret_cast<const float4*>(fa.v1 + col)) : make_float4(0.f, 0.f, 0.f, 0.f);
      const float4 e4 = fa.v2 ? __ldg(reinterpret_cast<const float4*>(fa.v2 + col)) : make_float4(0.f, 0.f, 0.f, 0.f);
      const float2 rowst = rs[row];
      p0 = epi_fold_pair<EPI>(make_float2(acc.x, acc.y), make_float2(b4.x, b4.y), make_float2(g4.x, g4.y),
                              make_float2(e4.x, e4.y), ua, rowst);
      p1 = epi_fold_pair<EPI>(make_float2(acc.z, acc.w), make_float2(b4.z, b4.w), make_float2(g4.z, g4.w),
                              make_float2(e4.z, e4.w), ub, rowst);
      const float2 y0 = unpack_bf16x2(p0), y1 = unpack_bf16x2(p1);
      float s1 = y0.x, s2 = y0.x * y0.x;
      s1 += y0.y; s2 = fmaf(y0.y, y0.y, s2);
      s1 += y1.x; s2 = fmaf(y1.x, y1.x, s2);
      s1 += y1.y; s2 = fmaf(y1.y, y1.y, s2);
      const unsigned gmask = 0xffu << (lane & 24);
#pragma unroll
      for (int o = 1; o < 8; o <<= 1) {
        s1 += __shfl_xor_sync(gmask, s1, o);
        s2 += __shfl_xor_sync(gmask, s2, o);
      }
      if ((lane & 7) == 0 && fa.st_out != nullptr)
        reinterpret_cast<float2*>(fa.st_out)[(size_t)(col / 32) * fa.st_ld + grow] = make_float2(s1, s2);
    } else {
      const uint32_t r4[4] = {__float_as_uint(acc.x), __float_as_uint(acc.y), __float_as_uint(acc.z),
                              __float_as_uint(acc.w)};
      epi_pack4<EPI>(r4, b4, ua, ub, p0, p1);
    }
    *reinterpret_cast<uint2*>(out + (size_t)grow * N + col) = make_uint2(p0, p1);
  }
  ptx::cluster_sync();  // no CTA leaves (releasing its shared memory) while a peer still reads it
  if (warp == 5) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, R::TMEM_COLS);
  }
}

template <int BN, int EPI>
cudaError_t launch_cfg(const TcGemmPlan& p, cudaStream_t s) {
  auto kern = gemm_splitk_kernel<BN, EPI>;
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t e = once_per_device(attr_done, [&] {
    return cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemOptIn - 2048); });
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(p.splits, p.N / BN, (p.M + BM - 1) / BM);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = p.smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = p.splits;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, p.tmA, p.tmB, (bf16*)p.out, p.M, p.N, p.kc, p.a_rows, p.stages, p.a_stage,
                            p.bias, (const bf16*)p.resid, p.ldr, p.fold);
}

template <int BN>
cudaError_t launch_bn(const TcGemmPlan& p, cudaStream_t s) {
  switch (p.epi) {
    case EPI_BIAS: return launch_cfg<BN, EPI_BIAS>(p, s);
    case EPI_BIAS_GELU: return launch_cfg<BN, EPI_BIAS_GELU>(p, s);
    case EPI_BIAS_RESID: return launch_cfg<BN, EPI_BIAS_RESID>(p, s);
    case EPI_RESID_LN: return launch_cfg<BN, EPI_RESID_LN>(p, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace

// Split factor: the smallest divisor S <= 8 of K/64 that puts >= 120 CTAs on the weights of
// one 128-row block at BN = 32 with at most 12 k-blocks (48 MMAs) per CTA; failing that, the
// largest such divisor.  BERT-base: QKV 2, out-proj 6, FFN1 2, FFN2 6; BERT-large: 2, 4, 1, 8.
int splitk_factor(int N, int K) {
  const int kb = K / BK;
  int best = 1;
  for (int s = 1; s <= kMaxSplits; ++s) {
    if (kb % s) continue;
    best = s;
    if ((N / 32) * s >= 120 && kb / s <= 12) break;
  }
  return best;
}

// Tile width: the narrowest of 32 / 64 / 128 / 192 that keeps the grid within two CTAs per SM.
// (The LATENCY family times the widths instead: at most 22 six-CTA clusters are resident at once
// on B200 (ncu launch__cluster_max_active), so the width that keeps a GEMM in one wave of clusters
// can be wider than this rule's.)
int splitk_bn(int M, int N, int S) {
  const long mblocks = (M + BM - 1) / BM;
  const long cap = 2L * num_sms();
  for (int bn : {32, 64, 128, 192})
    if (N % bn == 0 && (long)(N / bn) * S * mblocks <= cap) return bn;
  return N % 128 == 0 ? 128 : N % 64 == 0 ? 64 : 32;
}

bool tc_plan_gemm_splitk(TcGemmPlan* p, int M, int N, int K, const void* A, int lda, const void* W,
                         const float* bias, const void* resid, int ldr, void* out, int epi, int bn) {
  if (M <= 0 || N % 64 || K % 64 || K <= 0 || lda < K || lda % 8 || ldr < N || ldr % 8) return false;
  const int S = splitk_factor(N, K);
  if (bn == 0) bn = splitk_bn(M, N, S);
  if ((bn != 32 && bn != 64 && bn != 128 && bn != 192) || N % bn) return false;
  const int kc = K / S, kblocks = kc / BK;
  const int a_rows = M < BM ? ((M + 7) & ~7) : BM;
  const int a_stage = ((a_rows * BK * 2) + 1023) & ~1023;
  const int b_stage = bn * BK * 2;
  const int red = BM * (bn + 4) * 4;
  const long ctas = (long)S * (N / bn) * ((M + BM - 1) / BM);
  // two CTAs per SM when the grid exceeds one wave, else the whole opt-in budget
  // (less 2 KB for the kernel's static shared memory: the EPI_RESID_LN row statistics)
  int budget = ctas > num_sms() ? kSmemOptIn / 2 - 2048 : kSmemOptIn - 2048;
  if (const char* e = getenv("ARLO_SPLITK_SMEM")) budget = atoi(e);  // A/B: per-CTA smem budget (bytes)
  const int fixed = 1024 + 8 * 64;  // (the partial `red` lives over the operand ring)
  int stages = (budget - fixed) / (a_stage + b_stage);
  if (stages > kMaxStages) stages = kMaxStages;
  if (stages < 2) stages = 2;  // (a budget too small for two stages is exceeded)
  if (stages > kblocks) stages = kblocks;
  p->M = M; p->N = N; p->K = K; p->BN = bn; p->epi = epi; p->grid = (int)ctas; p->ew = 4;
  p->pair = false; p->skinny = false; p->ln = false; p->splitk = true; p->fold = FoldArgs{}; p->lnp = LnPrologue{};
  p->splits = S; p->kc = kc; p->stages = stages; p->a_stage = a_stage; p->a_rows = a_rows;
  p->smem = fixed + (stages * (a_stage + b_stage) > red ? stages * (a_stage + b_stage) : red);
  p->bias = bias; p->resid = resid; p->ldr = ldr; p->out = out;
  if (!encode_tmap_bf16_2d(&p->tmA, A, (uint64_t)K, (uint64_t)M, BK, a_rows, 128, (uint64_t)lda)) return false;
  if (!encode_tmap_bf16_2d(&p->tmB, W, (uint64_t)K, (uint64_t)N, BK, bn, 128)) return false;
  return true;
}

cudaError_t splitk_launch(const TcGemmPlan& p, cudaStream_t s) {
  switch (p.BN) {
    case 32: return launch_bn<32>(p, s);
    case 64: return launch_bn<64>(p, s);
    case 128: return launch_bn<128>(p, s);
    case 192: return launch_bn<192>(p, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace arlo
