// gemm_tc.cu — tcgen05/TMEM/TMA GEMM with fused epilogues (steps a2, a4, a6, a7).
//
//   out[M,N] = epi(A[M,K] W[N,K]^T + bias[N]),  epi in {identity, GELU_erf, +residual}
//
// The projections of every BERT layer (QKV, attention output, FFN1, FFN2;
// Devlin et al. [17]) on the padded static shape M = b*L of a
// per-length runtime (§3.3: "GPUs are most efficient at matrix
// multiplication when the sequence length is a multiple of the tile size").
//
// Blackwell design (not a port of anything in the paper, whose runtimes are
// TensorRT engines for sm_86):
//  * persistent CTAs (grid = min(tiles, #SMs)), static round-robin tile order
//    (N fastest), single-CTA 128 x BN tiles or CTA-pair (cta_group::2) 256 x BN tiles;
//  * warps 0..EW-1 = epilogue (EW = 8; Roles<EW>):
//    warp w reads TMEM lane quarter w % 4 and the 32-column chunks w/4, w/4 + EW/4, ...;
//    tcgen05.ld, bias / GELU / residual on paired fp32 instructions, RNE to bf16,
//    st.shared into a 64B-swizzled staging tile, TMA bulk tensor store.  Two TMEM
//    accumulator stages let the epilogue of tile i overlap the main loop of tile i+1;
//  * warp EW = TMA producer: 128x64 A tile + BNx64 W tile per stage, 128-byte
//    swizzle, STAGES-deep smem ring guarded by full/empty mbarriers;
//  * warp EW+1 = MMA issuer: the converged warp runs the loop, one elected lane issues
//    tcgen05.mma.kind::f16 (M=128 or 256, N=BN, K=16) into the TMEM fp32 accumulator;
//    tcgen05.commit frees smem stages and signals the epilogue.
// Row results never depend on M, the tile width or the grid: the K loop of
// every output element is the same sequence of K=16 MMAs (cross-L bitwise
// invariance, SURVEY.md §7 "Cross-L argmax agreement").
#include <cuda.h>

#include "common.cuh"
#include "epilogue.cuh"
#include "kernels.h"
#include "layernorm.cuh"
#include "ptx.cuh"

namespace arlo {
namespace {

constexpr int BM = 128, BK = 64;
#ifndef ARLO_EPI_WARPS
#define ARLO_EPI_WARPS 8
#endif
constexpr int kEpiWarps = ARLO_EPI_WARPS;      // warps 0..kEpiWarps-1: kEpiGroups per TMEM lane quarter
constexpr int kEpiGroups = kEpiWarps / 4;      // column groups of an accumulator tile
constexpr int kProducerWarp = kEpiWarps;       // warp 8: TMA producer
constexpr int kMmaWarp = kEpiWarps + 1;        // warp 9: MMA issuer
constexpr int kThreads = 32 * (kEpiWarps + 2);
constexpr int kAccStages = 2;
constexpr int kStgBytes = 32 * 64;             // one 32-row x 32-col bf16 staging tile (SWIZZLE_64B)
#ifndef ARLO_STG_BUFS
#define ARLO_STG_BUFS 2
#endif
constexpr int kStgBufs = ARLO_STG_BUFS;
#ifndef ARLO_EPI_PAIRS
#define ARLO_EPI_PAIRS 1  // A/B hook: 0 = one chunk per store step for the bias / GELU epilogues
#endif
#ifndef ARLO_EPI_EARLY_LD
#define ARLO_EPI_EARLY_LD 0  // A/B hook: 1 = the next step's first TMEM load before the second chunk's math
#endif
#ifndef ARLO_EPI_PAIRS_RESID
#define ARLO_EPI_PAIRS_RESID 1  // A/B hook: 0 = one chunk per store step for the residual epilogue
#endif         // staging tiles per epilogue warp (TMA stores in flight)
// Per epilogue warp: kStgBufs output staging tiles, then the bias of the warp's chunks of the
// current tile (32 fp32 per chunk, <= 4 chunks), staged before the accumulator wait so that the
// epilogue math reads bias from shared memory, not from L2 (a cold __ldg per chunk cost ~400
// cycles of the ~1100-cycle chunk: tools/gemm_trace.py sub-stamps, profiles/r02_gemm_sweep.txt).
#ifndef ARLO_BIAS_SMEM
#define ARLO_BIAS_SMEM 1  // A/B hook: 0 reads bias with __ldg inside the chunk loop
#endif
constexpr int kBiasWarpBytes = ARLO_BIAS_SMEM ? 4 * 32 * 4 : 0;
// Column vectors an epilogue stages per warp and chunk: bias (EPI 0-2), s and c (LN fold), bias,
// gamma and beta (residual + on-the-fly LayerNorm).  The fold epilogues always stage them.
constexpr int nvec_of(int epi) { return epi == EPI_RESID_LN ? 3 : epi >= EPI_LNFOLD ? 2 : 1; }
constexpr int col_warp_bytes(int epi) { return epi >= EPI_LNFOLD ? 4 * 32 * 4 * nvec_of(epi) : kBiasWarpBytes; }
constexpr bool is_resid(int epi) { return epi == EPI_BIAS_RESID || epi == EPI_RESID_LN; }
constexpr int kWarpStg = kStgBufs * kStgBytes + kBiasWarpBytes;
constexpr int kStagingBytes = kEpiWarps * kWarpStg;

// Warp-role layout of the persistent kernels for EW epilogue warps (EW / 4 column groups per
// TMEM lane quarter), then the TMA producer and the MMA warp.  EW = 8.  Round 1 ran the GELU
// epilogue (then two MUFU ops per element) with EW = 12 at M <= 8192; with the one-MUFU GELU
// (A&S 7.1.28) and the two-chunk store step, 8 warps win at every M (FFN1 M = 2048 / 4096 / 8192:
// 737 / 953 / 1132 vs 710 / 927 / 1100 TF; profiles/r02_epilogue_pairs_ab.txt).  The
// bias / residual epilogues lose with 12 (fewer smem stages, more residual traffic in flight).
// ARLO_GELU_EW12_MAX_M keeps the 12-warp instantiation reachable for A/B runs.
template <int EW>
struct Roles {
  static_assert(EW % 4 == 0, "epilogue warps cover the four TMEM lane quarters");
  static constexpr int kEpi = EW, kGroups = EW / 4, kProducer = EW, kMma = EW + 1, kThreads = 32 * (EW + 2);
  static constexpr int kStaging = EW * kWarpStg;
};
constexpr int kSmemBudget = 229376;            // 224 KB of the 227 KB opt-in maximum

// Optional event trace (tools/gemm_trace.py): when g_trace != nullptr every CTA
// writes %globaltimer stamps to g_trace[blockIdx.x * 64 + slot].  One
// predictable branch per event; never set in production.
__device__ unsigned long long* g_trace = nullptr;
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void trace(int slot) {
  if (g_trace != nullptr && slot < 64) g_trace[blockIdx.x * 64 + slot] = gtimer();
}
// clock64 sub-stamps of the epilogue of a CTA's first tile (warp 0, lane 0): slots 32..63
__device__ __forceinline__ void trace_clk(int slot) {
  if (g_trace != nullptr && slot < 64) g_trace[blockIdx.x * 64 + slot] = clock64();
}

// Tile rasterisation of the persistent kernels: N fastest.  The CTAs (pairs) running at
// the same time then cover a few whole row blocks of A (each A row block is read from
// DRAM once and shared through L2 by the N/BN tiles of its row) and every column of W
// (<= 8 MB, L2-resident).  The M-fastest order read A about 6x from DRAM at
// M = 32768 (ncu: 441 MB vs 72 MB of operands; cuBLAS 78 MB), costing power and clock.
__device__ __forceinline__ int tile_m(int tile, int num_m, int num_n) {
#if defined(ARLO_RASTER_M)  // A/B only: the previous M-fastest order
  return tile % num_m;
#else
  return tile / num_n;
#endif
}
__device__ __forceinline__ int tile_n(int tile, int num_m, int num_n) {
#if defined(ARLO_RASTER_M)
  return tile / num_m;
#else
  return tile % num_n;
#endif
}

constexpr int tmem_cols_for(int n) {
  return n <= 32 ? 32 : n <= 64 ? 64 : n <= 128 ? 128 : n <= 256 ? 256 : 512;
}

// PAIR = false: one CTA computes a 128 x BN tile; PAIR = true: a CTA pair
// (cluster of 2, cta_group::2) computes a 256 x BN tile, each CTA holding 128
// rows of A, BN/2 rows of W and its 128 x BN half of the accumulator.
// Residual epilogue (EPI_BIAS_RESID, ARLO_RESID_TMA): the producer TMA-loads the CTA's 128 x BN
// residual tile into shared memory ({32 columns x 128 rows} boxes, 64-byte swizzle = the output
// staging layout) while the main loop runs; the epilogue reads the residual from there, writes the
// bf16 result in place and TMA-stores it from the same buffer.  The residual's L2 round trip left
// the critical path of the epilogue (it cost ~1000-1300 of a ~1800-cycle chunk, gemm_trace
// sub-stamps) and the per-warp output staging tiles are not needed.
#ifndef ARLO_RESID_TMA
#define ARLO_RESID_TMA 1
#endif
template <int BN>
constexpr int resid_buf_bytes() { return BN * 128 * 2; }

template <int BN, bool PAIR, int RESERVE = 0, int EW = kEpiWarps, bool RESID_BUF = false, int COLB = kBiasWarpBytes>
struct TcCfg {
  static constexpr int kStagingBytes =
      RESID_BUF ? EW * COLB + resid_buf_bytes<BN>() : EW * (kStgBufs * kStgBytes + COLB);
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_ROWS = PAIR ? BN / 2 : BN;
  static constexpr int B_BYTES = B_ROWS * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES_FIT = (kSmemBudget - kStagingBytes - RESERVE) / STAGE_BYTES;
  static constexpr int STAGES = STAGES_FIT > 8 ? 8 : STAGES_FIT;
  static constexpr int TMEM_COLS = tmem_cols_for(kAccStages * BN);
  static constexpr int BAR_BYTES = 8 * (2 * STAGES + 2 * kAccStages + 2) + 16;
  static constexpr int SMEM = 1024 + STAGES * STAGE_BYTES + kStagingBytes + BAR_BYTES + RESERVE;
  static_assert(SMEM <= 232448, "shared memory budget");
};

// Epilogue of one accumulator tile for one warp: TMEM lane quarter q (32
// rows) and the 32-column chunks cg, cg + G, cg + 2G, ... of the tile (G =
// kEpiGroups warps share a quarter).  For each chunk: tcgen05.ld (the next
// chunk's load and residual are issued before this chunk is computed), bias /
// GELU / residual in fp32, RNE to bf16, st.shared into a 64-byte-swizzled
// 32x32 staging tile, then one TMA bulk tensor store of the tile (coalesced,
// asynchronous; rows >= M clipped by the tensor map).  `release()` fires once
// the warp's last TMEM load has completed.
constexpr int CW = 32;  // chunk width: TMEM load / staging tile / TMA box (columns)

#ifndef ARLO_EPI_DIRECT
#define ARLO_EPI_DIRECT 0  // 1: store rows straight from registers instead of smem staging + TMA (A/B)
#endif

// Residual of this warp's first chunk of a tile (row row0 + lane, columns n0 + 32 cg ...): the
// residual never depends on the MMA, so the epilogue warps load it BEFORE waiting for the
// accumulator, taking its L2 latency off the exposed epilogue of one-round GEMMs.
template <int BN, int EPI>
__device__ __forceinline__ void prefetch_first_resid(uint4 (&rv)[CW / 8], const bf16* resid, int row0, int lane,
                                                     int n0, int cg, int M, int ldr) {
  if (!is_resid(EPI) || cg * CW >= BN) return;  // (a warp without chunks loads nothing)
  const int row = row0 + lane;
  if (row >= M) return;
  const uint4* res4 = reinterpret_cast<const uint4*>(resid + (size_t)row * ldr + n0) + cg * (CW / 8);
#pragma unroll
  for (int j = 0; j < CW / 8; ++j) rv[j] = ld_dep_v4(res4 + j);
}

// Column vectors of this warp's chunks cg, cg + G, ... of the tile at column n0 -> the warp's
// slots [chunk k][vector v][32 columns] (lane j writes column 32 c + j; the math reads float4
// broadcasts): bias, or s and c (LN fold), or bias, gamma and beta (residual LN).  Called before
// the accumulator wait; the warp's previous tile has finished reading the slots.
template <int BN, int EPI, int kEpiGroups>
__device__ __forceinline__ void stage_colv(float* sv, const float* __restrict__ v0, const FoldArgs& fa, int n0, int cg,
                                           int lane) {
  constexpr int NCH = BN / CW;
  constexpr int NCMAX = (NCH + kEpiGroups - 1) / kEpiGroups;
  constexpr int NV = nvec_of(EPI);
  static_assert(NCMAX * CW * 4 * NV <= col_warp_bytes(EPI) || (!ARLO_BIAS_SMEM && EPI < EPI_LNFOLD), "column slots");
  if (!ARLO_BIAS_SMEM && EPI < EPI_LNFOLD) return;
#pragma unroll
  for (int k = 0; k < NCMAX; ++k) {
    const int c = cg + k * kEpiGroups;
    if (c < NCH) {
      const int col = n0 + c * CW + lane;
      sv[(k * NV) * CW + lane] = __ldg(v0 + col);
      if (NV >= 2) sv[(k * NV + 1) * CW + lane] = fa.v1 ? __ldg(fa.v1 + col) : 0.f;
      if (NV >= 3) sv[(k * NV + 2) * CW + lane] = fa.v2 ? __ldg(fa.v2 + col) : 0.f;
    }
  }
  __syncwarp();
}


// epi_fold_pair (the per-pair arithmetic of the LayerNorm-fold modes) is in epilogue.cuh.
template <int EPI>
__device__ __forceinline__ void epi_fold_chunk(const uint32_t* acc, const float* sv, const uint32_t* ru, float2 rowst,
                                               uint32_t* pk) {
  constexpr int NV = nvec_of(EPI);
  const float4* s0 = reinterpret_cast<const float4*>(sv);
  const float4* s1 = s0 + CW / 4;
  const float4* s2 = s1 + CW / 4;
#pragma unroll
  for (int j = 0; j < CW / 4; ++j) {  // 4 columns: 2 pairs
    const float4 a0 = s0[j], a1 = s1[j];
    const float4 a2 = NV >= 3 ? s2[j] : make_float4(0.f, 0.f, 0.f, 0.f);
    const float2 x0 = make_float2(__uint_as_float(acc[4 * j]), __uint_as_float(acc[4 * j + 1]));
    const float2 x1 = make_float2(__uint_as_float(acc[4 * j + 2]), __uint_as_float(acc[4 * j + 3]));
    pk[2 * j] = epi_fold_pair<EPI>(x0, make_float2(a0.x, a0.y), make_float2(a1.x, a1.y), make_float2(a2.x, a2.y),
                                   ru[2 * j], rowst);
    pk[2 * j + 1] = epi_fold_pair<EPI>(x1, make_float2(a0.z, a0.w), make_float2(a1.z, a1.w),
                                       make_float2(a2.z, a2.w), ru[2 * j + 1], rowst);
  }
}

// (sum y, sum y^2) of 16 packed bf16 words (32 columns) in column order, continuing (s1, s2).
__device__ __forceinline__ float2 fold_granule(const uint32_t* pk, int nw, float2 acc) {
  float s1 = acc.x, s2 = acc.y;
#pragma unroll
  for (int j = 0; j < 16; ++j) {
    if (j < nw) {
      const float2 y = unpack_bf16x2(pk[j]);
      s1 += y.x; s2 = fmaf(y.x, y.x, s2);
      s1 += y.y; s2 = fmaf(y.y, y.y, s2);
    }
  }
  return make_float2(s1, s2);
}

template <int BN, int EPI, int kEpiGroups, typename Release>
__device__ __forceinline__ void epilogue_tile(uint32_t t_acc, int q, int cg, int lane, int row0, int n0, int M,
                                              int ldr, const float* __restrict__ bias,
                                              const bf16* __restrict__ resid, const CUtensorMap* tmC,
                                              uint8_t* stg, int& sc, Release release, bf16* __restrict__ outp,
                                              int N, const uint4* rv_first, uint8_t* rbuf = nullptr,
                                              const float* sbias = nullptr, float2 rowst = make_float2(0.f, 1.f),
                                              float* st_out = nullptr, int st_ld = 0) {
  static_assert(BN % CW == 0, "tile width must be a multiple of 32");
  constexpr int NCH = BN / CW;                                 // chunks per row block
  constexpr int NCMAX = (NCH + kEpiGroups - 1) / kEpiGroups;  // chunks per warp (max)
  constexpr int RV = CW / 8;                                   // 16-byte residual vectors per row per chunk
  const int nc = (NCH - cg + kEpiGroups - 1) / kEpiGroups;     // this warp's chunks (warp-uniform)
  const int row = row0 + lane;
  const bool row_ok = row < M;
  const uint4* res4 = reinterpret_cast<const uint4*>(resid + (size_t)(row_ok ? row : 0) * ldr + n0);
  const uint32_t t_row = t_acc + ((uint32_t)(q * 32) << 16);
  if (nc <= 0) {
    ptx::tc_fence_before();
    __syncwarp();
    if (lane == 0) release();
    return;
  }
  const bool stamp = threadIdx.x == 0 && g_trace != nullptr && sc < 64;  // (sc: chunks stored so far)
  const bool first_tile = sc == 0;
  if (stamp && first_tile) trace_clk(32);
  // the fold epilogues load one TMEM chunk at a time (their extra operands otherwise spill)
  constexpr int NB = EPI >= EPI_LNFOLD ? 1 : 2;
  uint32_t r[NB][CW];
  uint4 rv[2][RV];
  const bool rsm = rbuf != nullptr;  // residual tile in shared memory (TMA-prefetched), output in place
  constexpr int NV = nvec_of(EPI);
  if (is_resid(EPI) && row_ok && !rsm) {  // prefetched by the caller before the accumulator wait
#pragma unroll
    for (int j = 0; j < RV; ++j) rv[0][j] = rv_first[j];
  }
  ptx::tmem_ld_32x32b_x32(t_row + cg * CW, r[0]);
  ptx::tmem_wait_ld();
  if (stamp && first_tile) trace_clk(33);
  // Bias / GELU epilogues: two chunks per step.  Both chunks' math runs back to back (the second
  // chunk's TMEM load overlaps the first's math), then one proxy fence, one warp sync and two TMA
  // stores from the two staging tiles: half the fixed per-chunk store cost (fence + sync + issue +
  // staging wait were ~500 of a ~1000-cycle chunk, tools/gemm_trace.py).  Same per-element
  // arithmetic (epi_pack4): bitwise the one-chunk loop.  8 epilogue warps only: with 12 (GELU at
  // M <= 8192, <= 144 registers per thread) the second live chunk spilled and the pair loop lost
  // (FFN1 M = 4096 948 -> 928 TF; at M = 16384, 8 warps: 1097 -> 1197 TF, gpurun A/B).
  if constexpr ((EPI == EPI_BIAS || EPI == EPI_BIAS_GELU) && ARLO_EPI_PAIRS && !ARLO_EPI_DIRECT &&
                kEpiGroups < 3) {
    static_assert(kStgBufs >= 2, "chunk-pair epilogue needs two staging tiles per warp");
    auto chunk_math = [&](const uint32_t* rr, int kk, uint32_t* pk) {
      const float4* bias4 = ARLO_BIAS_SMEM ? reinterpret_cast<const float4*>(sbias) + kk * (CW / 4)
                                           : reinterpret_cast<const float4*>(bias + n0 + (cg + kk * kEpiGroups) * CW);
#pragma unroll
      for (int j = 0; j < CW / 4; ++j) {
        const float4 b4 = ARLO_BIAS_SMEM ? bias4[j] : __ldg(bias4 + j);
        epi_pack4<EPI>(&rr[4 * j], b4, 0u, 0u, pk[2 * j], pk[2 * j + 1]);
      }
    };
    auto stage = [&](const uint32_t* pk, uint8_t* buf) {
#pragma unroll
      for (int j = 0; j < CW / 8; ++j) {
        const int sw = j ^ ((lane >> 1) & 3);  // TMA 64B swizzle of a 64-byte row
        *reinterpret_cast<uint4*>(buf + lane * (CW * 2) + sw * 16) =
            make_uint4(pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
      }
    };
#pragma unroll 1
    for (int k = 0; k < nc; k += 2) {
      const bool two = k + 1 < nc, more = k + 2 < nc;
      const int c0 = cg + k * kEpiGroups, c1 = c0 + kEpiGroups;
      if (stamp && first_tile && k < 12) trace_clk(34 + 5 * (k / 2));
      if (two) ptx::tmem_ld_32x32b_x32(t_row + c1 * CW, r[1]);  // overlaps chunk k's math
      uint32_t pk[CW / 2];
      chunk_math(r[0], k, pk);
      if (stamp && first_tile && k < 12) trace_clk(35 + 5 * (k / 2));
      if (sc > 0) {  // the previous step's TMA stores have finished reading both staging tiles
        if (lane == 0) ptx::bulk_wait_read<0>();
        __syncwarp();
      }
      if (stamp && first_tile && k < 12) trace_clk(36 + 5 * (k / 2));
      stage(pk, stg);
      if (two) ptx::tmem_wait_ld();
      if (!more) {  // every TMEM load of this warp has completed: hand the accumulator back
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) release();
      }
      if (ARLO_EPI_EARLY_LD && more) ptx::tmem_ld_32x32b_x32(t_row + (c1 + kEpiGroups) * CW, r[0]);
      if (two) {
        chunk_math(r[1], k + 1, pk);
        stage(pk, stg + kStgBytes);
      }
      if (!ARLO_EPI_EARLY_LD && more) ptx::tmem_ld_32x32b_x32(t_row + (c1 + kEpiGroups) * CW, r[0]);
      ptx::fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) {
        ptx::tma_store_2d(tmC, stg, n0 + c0 * CW, row0);
        if (two) ptx::tma_store_2d(tmC, stg + kStgBytes, n0 + c1 * CW, row0);
        ptx::bulk_commit();
      }
      sc += two ? 2 : 1;
      if (stamp && first_tile && k < 12) trace_clk(37 + 5 * (k / 2));
      if (more) ptx::tmem_wait_ld();
      if (stamp && first_tile && k < 12) trace_clk(38 + 5 * (k / 2));
    }
    return;
  }
  // Residual epilogue, residual tile TMA-prefetched into shared memory (the default): the same
  // two-chunk step, each chunk written in place over its residual and TMA-stored from there.
  if constexpr (EPI == EPI_BIAS_RESID && ARLO_EPI_PAIRS_RESID && !ARLO_EPI_DIRECT && kEpiGroups < 3) {
    if (rsm) {
      auto chunk = [&](const uint32_t* rr, int kk, uint8_t* rch) {
        const float4* bias4 = ARLO_BIAS_SMEM ? reinterpret_cast<const float4*>(sbias) + kk * (CW / 4)
                                             : reinterpret_cast<const float4*>(bias + n0 + (cg + kk * kEpiGroups) * CW);
        uint32_t pk[CW / 2];
#pragma unroll
        for (int j = 0; j < CW / 8; ++j) {  // 8 columns: one 16-byte residual vector
          const int sw = j ^ ((lane >> 1) & 3);
          const uint4 u = *reinterpret_cast<const uint4*>(rch + lane * (CW * 2) + sw * 16);
          const float4 b0 = ARLO_BIAS_SMEM ? bias4[2 * j] : __ldg(bias4 + 2 * j);
          const float4 b1 = ARLO_BIAS_SMEM ? bias4[2 * j + 1] : __ldg(bias4 + 2 * j + 1);
          epi_pack4<EPI>(&rr[8 * j], b0, u.x, u.y, pk[4 * j], pk[4 * j + 1]);
          epi_pack4<EPI>(&rr[8 * j + 4], b1, u.z, u.w, pk[4 * j + 2], pk[4 * j + 3]);
        }
#pragma unroll
        for (int j = 0; j < CW / 8; ++j) {
          const int sw = j ^ ((lane >> 1) & 3);
          *reinterpret_cast<uint4*>(rch + lane * (CW * 2) + sw * 16) =
              make_uint4(pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
        }
      };
#pragma unroll 1
      for (int k = 0; k < nc; k += 2) {
        const bool two = k + 1 < nc, more = k + 2 < nc;
        const int c0 = cg + k * kEpiGroups, c1 = c0 + kEpiGroups;
        uint8_t* rch0 = rbuf + c0 * (BM * CW * 2) + q * (32 * CW * 2);
        uint8_t* rch1 = rbuf + c1 * (BM * CW * 2) + q * (32 * CW * 2);
        if (stamp && first_tile && k < 12) trace_clk(34 + 5 * (k / 2));
        if (two) ptx::tmem_ld_32x32b_x32(t_row + c1 * CW, r[1]);  // overlaps chunk k's math
        chunk(r[0], k, rch0);
        if (stamp && first_tile && k < 12) trace_clk(35 + 5 * (k / 2));
        if (two) ptx::tmem_wait_ld();
        if (!more) {  // every TMEM load of this warp has completed: hand the accumulator back
          ptx::tc_fence_before();
          __syncwarp();
          if (lane == 0) release();
        }
        if (stamp && first_tile && k < 12) trace_clk(36 + 5 * (k / 2));
        if (ARLO_EPI_EARLY_LD && more) ptx::tmem_ld_32x32b_x32(t_row + (c1 + kEpiGroups) * CW, r[0]);
        if (two) chunk(r[1], k + 1, rch1);
        if (!ARLO_EPI_EARLY_LD && more) ptx::tmem_ld_32x32b_x32(t_row + (c1 + kEpiGroups) * CW, r[0]);
        ptx::fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) {
          ptx::tma_store_2d(tmC, rch0, n0 + c0 * CW, row0);
          if (two) ptx::tma_store_2d(tmC, rch1, n0 + c1 * CW, row0);
          ptx::bulk_commit();
        }
        sc += two ? 2 : 1;
        if (stamp && first_tile && k < 12) trace_clk(37 + 5 * (k / 2));
        if (more) ptx::tmem_wait_ld();
        if (stamp && first_tile && k < 12) trace_clk(38 + 5 * (k / 2));
      }
      return;
    }
  }
#pragma unroll
  for (int k = 0; k < NCMAX; ++k) {
    if (k >= nc) break;
    const int c = cg + k * kEpiGroups;  // chunk index within the tile
    const int cur = NB == 2 ? (k & 1) : 0, nxt = NB == 2 ? (cur ^ 1) : 0;
    if (NB == 1 && k > 0) {
      ptx::tmem_ld_32x32b_x32(t_row + c * CW, r[0]);
      if (is_resid(EPI) && row_ok && !rbuf) {
#pragma unroll
        for (int j = 0; j < RV; ++j) rv[0][j] = ld_dep_v4(res4 + c * RV + j);
      }
      ptx::tmem_wait_ld();
    }
    if (stamp && first_tile && k < 6) trace_clk(34 + 5 * k);
    // this chunk's 32 rows x 32 columns in the residual buffer (64-byte rows, 64B swizzle)
    uint8_t* rchunk = rsm ? rbuf + c * (BM * CW * 2) + q * (32 * CW * 2) : nullptr;
    if (is_resid(EPI) && rsm) {
#pragma unroll
      for (int j = 0; j < RV; ++j)
        rv[cur][j] = *reinterpret_cast<const uint4*>(rchunk + lane * (CW * 2) + ((j ^ ((lane >> 1) & 3)) * 16));
    }
    if (NB == 2 && k + 1 < nc) {
      ptx::tmem_ld_32x32b_x32(t_row + (c + kEpiGroups) * CW, r[nxt]);
      if (is_resid(EPI) && row_ok && !rsm) {
#pragma unroll
        for (int j = 0; j < RV; ++j) rv[nxt][j] = ld_dep_v4(res4 + (c + kEpiGroups) * RV + j);
      }
    }
    uint32_t pk[CW / 2];
    if constexpr (EPI < EPI_LNFOLD) {
      const float4* bias4 = ARLO_BIAS_SMEM ? reinterpret_cast<const float4*>(sbias) + k * (CW / 4)
                                           : reinterpret_cast<const float4*>(bias + n0 + c * CW);
#pragma unroll
      for (int j = 0; j < CW / 4; ++j) {
        const float4 b4 = ARLO_BIAS_SMEM ? bias4[j] : __ldg(bias4 + j);
        uint32_t ua = 0, ub = 0;
        if (EPI == EPI_BIAS_RESID) {
          const uint4 u = rv[cur][j >> 1];
          ua = (j & 1) ? u.z : u.x;
          ub = (j & 1) ? u.w : u.y;
        }
        epi_pack4<EPI>(&r[cur][4 * j], b4, ua, ub, pk[2 * j], pk[2 * j + 1]);
      }
    } else {
      const float* sv = sbias + k * NV * CW;  // this chunk's column vectors
      epi_fold_chunk<EPI>(&r[cur][0], sv, reinterpret_cast<const uint32_t*>(rv[cur]), rowst, pk);
      if (EPI == EPI_RESID_LN && st_out != nullptr && row_ok)  // granule (= chunk) statistics of the output
        reinterpret_cast<float2*>(st_out)[(size_t)((n0 + c * CW) / 32) * st_ld + row] =
            fold_granule(pk, 16, make_float2(0.f, 0.f));
    }
    if (ARLO_EPI_DIRECT) {
      if (row_ok) {
        uint4* o4 = reinterpret_cast<uint4*>(outp + (size_t)row * N + n0 + c * CW);
#pragma unroll
        for (int j = 0; j < CW / 8; ++j) o4[j] = make_uint4(pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
      }
      ptx::tmem_wait_ld();
      if (k == (nc >= 2 ? nc - 2 : 0)) {
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) release();
      }
      continue;
    }
    if (stamp && first_tile && k < 6) trace_clk(35 + 5 * k);
    // staging buffer sc % kStgBufs was last used kStgBufs chunks ago: make sure its TMA store has read it
    // (the residual epilogue stores in place from the residual buffer instead)
    uint8_t* buf = rsm ? rchunk : stg + (sc % kStgBufs) * kStgBytes;
    if (!rsm && sc >= kStgBufs) {
      if (lane == 0) ptx::bulk_wait_read<kStgBufs - 1>();
      __syncwarp();
    }
    if (stamp && first_tile && k < 6) trace_clk(36 + 5 * k);
#pragma unroll
    for (int j = 0; j < CW / 8; ++j) {
      // TMA 64B swizzle of a 64-byte row: 16-byte chunk index ^= address bits [7:8]
      const int sw = j ^ ((lane >> 1) & 3);
      *reinterpret_cast<uint4*>(buf + lane * (CW * 2) + sw * 16) =
          make_uint4(pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
    }
    ptx::fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) {
      ptx::tma_store_2d(tmC, buf, n0 + c * CW, row0);
      ptx::bulk_commit();
    }
    ++sc;
    if (stamp && first_tile && k < 6) trace_clk(37 + 5 * k);
    ptx::tmem_wait_ld();
    if (stamp && first_tile && k < 6) trace_clk(38 + 5 * k);
    if (k == (nc >= 2 ? nc - 2 : 0)) {  // the last TMEM load of this warp has completed
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) release();
    }
  }
}

template <int BN, int EPI, int EW>
__global__ void __launch_bounds__(Roles<EW>::kThreads, 1)
gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
               const __grid_constant__ CUtensorMap tmC, const __grid_constant__ CUtensorMap tmR, int M, int N, int K,
               const float* __restrict__ bias,
               const bf16* __restrict__ resid, int ldr, bf16* __restrict__ outp, const LnPrologue lnp,
               const FoldArgs fa) {
  constexpr bool kResidBuf = ARLO_RESID_TMA && is_resid(EPI);
  constexpr int kColB = col_warp_bytes(EPI);
  using C = TcCfg<BN, false, 0, EW, kResidBuf, kColB>;
  using R = Roles<EW>;
  constexpr int kEpiWarps = R::kEpi, kEpiGroups = R::kGroups, kProducerWarp = R::kProducer, kMmaWarp = R::kMma;
  constexpr int kStagingBytes = C::kStagingBytes;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * C::A_BYTES;
  uint8_t* sStg = sB + C::STAGES * C::B_BYTES;
  uint8_t* rbuf = sStg + kEpiWarps * kColB;  // (kResidBuf) the CTA's 128 x BN residual tile
  uint64_t* full = reinterpret_cast<uint64_t*>(sStg + kStagingBytes);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;
  uint64_t* tempty = tfull + kAccStages;
  uint64_t* rfull = tempty + kAccStages;  // residual tile landed (producer: expect_tx + TMA)
  uint64_t* rfree = rfull + 1;            // residual buffer read and stored from (one arrive per epilogue warp)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(rfree + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int num_m = (M + BM - 1) / BM;
  const int num_n = N / BN;
  const int tiles = num_m * num_n;
  const int kblocks = K / BK;

  if (warp == kProducerWarp && lane == 0) {
    ptx::tma_prefetch_desc(&tmA);
    ptx::tma_prefetch_desc(&tmB);
    ptx::tma_prefetch_desc(&tmC);
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < kAccStages; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], kEpiWarps);  // one arrive per epilogue warp
    }
    ptx::mbar_init(rfull, 1);
    ptx::mbar_init(rfree, kEpiWarps);
    if (kResidBuf) ptx::tma_prefetch_desc(&tmR);
    ptx::fence_mbar_init();
  }
  if (warp == kMmaWarp) ptx::tmem_alloc(tmem_slot, C::TMEM_COLS);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  pdl_launch_dependents();  // setup above overlapped the previous kernel's tail

  // W never depends on the previous kernel: the first tile's first STAGES W tiles are
  // requested before the PDL wait (and before the LayerNorm prologue), its A tiles after it
  const int pre = blockIdx.x < tiles ? (kblocks < C::STAGES ? kblocks : C::STAGES) : 0;
  if (warp == kProducerWarp && lane == 0) {
    const int n0 = tile_n(blockIdx.x, num_m, num_n) * BN;
    for (int kb = 0; kb < pre; ++kb) {
      ptx::mbar_arrive_expect_tx(&full[kb], C::STAGE_BYTES);
      ptx::tma_load_2d(sB + kb * C::B_BYTES, &tmB, &full[kb], kb * BK, n0);
    }
  }
  if constexpr (EPI != EPI_BIAS_RESID) {
    if (lnp.y != nullptr) {  // A = LN(y), computed by the whole grid first (layernorm.cuh)
      pdl_wait();
      ln_prologue(lnp);
    }
  }

  if (warp == kProducerWarp) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0) {
      pdl_wait();
      if (threadIdx.x == kProducerWarp * 32) trace(0);
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x, ++it) {
        const int m0 = tile_m(tile, num_m, num_n) * BM, n0 = tile_n(tile, num_m, num_n) * BN;
        trace(2 + 6 * it);
        // residual tile: issued as soon as the previous tile's epilogue has freed the buffer (polled
        // between k-blocks so the main loop never waits for it), at the latest after the last k-block
        bool r_issued = !kResidBuf;
        auto issue_resid = [&]() {
          ptx::mbar_arrive_expect_tx(rfull, (uint32_t)resid_buf_bytes<BN>());
          for (int c = 0; c < BN / CW; ++c)
            ptx::tma_load_2d(rbuf + c * (BM * CW * 2), &tmR, rfull, n0 + c * CW, m0);
          r_issued = true;
        };
        for (int kb = 0; kb < kblocks; ++kb) {
          if (it == 0 && kb < pre) {
            ptx::tma_load_2d(sA + stage * C::A_BYTES, &tmA, &full[stage], kb * BK, m0);
          } else {
            ptx::mbar_wait(&empty[stage], phase ^ 1);
            ptx::mbar_arrive_expect_tx(&full[stage], C::STAGE_BYTES);
            ptx::tma_load_2d(sA + stage * C::A_BYTES, &tmA, &full[stage], kb * BK, m0);
            ptx::tma_load_2d(sB + stage * C::B_BYTES, &tmB, &full[stage], kb * BK, n0);
          }
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
          if (!r_issued && (it == 0 || ptx::mbar_test(rfree, (it - 1) & 1))) issue_resid();
        }
        if (!r_issued) {
          ptx::mbar_wait(rfree, (it - 1) & 1);
          issue_resid();
        }
      }
    } else {
      pdl_wait();
    }
  } else if (warp == kMmaWarp) {
    // ------------------------------------------------------------- MMA issuer
    pdl_wait();
    {  // converged warp, elected lane issues (see gemm_tc_pair_kernel)
      constexpr uint32_t idesc = ptx::idesc_bf16_f32(BM, BN);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      int it = 0;
      for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x, ++it) {
        ptx::mbar_wait(&tempty[acc], acc_phase ^ 1);
        ptx::tc_fence_after();
        if (lane == 0) trace(3 + 6 * it);
        const uint32_t d_tmem = tmem_base + acc * BN;
        for (int kb = 0; kb < kblocks; ++kb) {
          ptx::mbar_wait(&full[stage], phase);
          ptx::tc_fence_after();
          if (kb == 0 && lane == 0) trace(4 + 6 * it);
          const uint32_t a_addr = ptx::smem_u32(sA + stage * C::A_BYTES);
          const uint32_t b_addr = ptx::smem_u32(sB + stage * C::B_BYTES);
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            ptx::mma_bf16_ss_w(d_tmem, ptx::desc_k_sw128(a_addr + k * 32),
                               ptx::desc_k_sw128(b_addr + k * 32), idesc, (kb | k) != 0);
          }
          ptx::mma_commit_w(&empty[stage]);
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
        }
        ptx::mma_commit_w(&tfull[acc]);
        if (lane == 0) trace(5 + 6 * it);
        if (++acc == kAccStages) { acc = 0; acc_phase ^= 1; }
      }
    }
  } else {
    // --------------------------------------------------------------- epilogue
    // warp w may only touch TMEM lanes 32*(w%4)..+31 (rows of the tile); the
    // two warps sharing a quarter take one column half each.
    pdl_wait();
    const int q = warp & 3, cg = warp >> 2;
    uint8_t* stg = kResidBuf ? nullptr : sStg + warp * (kStgBufs * kStgBytes + kColB);
    float* sbias = reinterpret_cast<float*>(kResidBuf ? sStg + warp * kColB : stg + kStgBufs * kStgBytes);
    int sc = 0;
    int acc = 0;
    uint32_t acc_phase = 0;
    int it = 0;
    for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x, ++it) {
      const int m0 = tile_m(tile, num_m, num_n) * BM, n0 = tile_n(tile, num_m, num_n) * BN;
      uint4 rv0[CW / 8];
      if (!kResidBuf) prefetch_first_resid<BN, EPI>(rv0, resid, m0 + q * 32, lane, n0, cg, M, ldr);
      stage_colv<BN, EPI, kEpiGroups>(sbias, bias, fa, n0, cg, lane);
      // LayerNorm fold: this row's statistics (of A's rows, or of the residual rows)
      float2 rowst = make_float2(0.f, -1.f);
      if constexpr (EPI >= EPI_LNFOLD) {
        const int grow = m0 + q * 32 + lane;
        const int Hs = EPI == EPI_RESID_LN ? N : K;
        if (fa.st_in != nullptr && grow < M) {
          const float2 ms = fold_row_stats(fa.st_in, (size_t)grow * fa.st_in_stride, fa.st_ld, Hs / 32, Hs, fa.eps);
          rowst = EPI == EPI_RESID_LN ? ms : make_float2(-ms.x * ms.y, ms.y);
        } else if (EPI != EPI_RESID_LN) {
          rowst = make_float2(0.f, 1.f);
        }
      }
      ptx::mbar_wait(&tfull[acc], acc_phase);
      if (kResidBuf) ptx::mbar_wait(rfull, it & 1);  // this tile's residual has landed
      ptx::tc_fence_after();
      if (warp == 0 && lane == 0) trace(6 + 6 * it);
      uint64_t* te = &tempty[acc];
      epilogue_tile<BN, EPI, kEpiGroups>(tmem_base + acc * BN, q, cg, lane, m0 + q * 32, n0, M, ldr, bias, resid,
                                         &tmC, stg, sc, [te]() { ptx::mbar_arrive(te); }, outp, N, rv0,
                                         kResidBuf ? rbuf : nullptr, sbias, rowst, fa.st_out, fa.st_ld);
      if (kResidBuf) {  // the buffer is free once this warp's in-place TMA stores have read it
        if (lane == 0) ptx::bulk_wait_read<0>();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(rfree);
      }
      if (warp == 0 && lane == 0) trace(7 + 6 * it);
      if (++acc == kAccStages) { acc = 0; acc_phase ^= 1; }
    }
    if (lane == 0) ptx::bulk_wait<0>();
  }

  ptx::tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) trace(1);
  if (warp == kMmaWarp) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem_base, C::TMEM_COLS);
  }
}

// CTA-pair kernel: cluster (2,1,1); the pair computes 256 x BN tiles with
// tcgen05.mma.cta_group::2 issued by the leader (rank 0).  Each CTA's TMA
// loads its 128 rows of A and its BN/2 rows of W and counts the bytes on the
// leader's full barrier; the leader's commits arrive on both CTAs' empty and
// tfull barriers (multicast); both CTAs' epilogue warps arrive on the
// leader's tempty barrier.  Halves the L2->SM operand traffic per FLOP and
// deepens the smem pipeline relative to the single-CTA kernel.
template <int BN, int EPI, int EW>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(Roles<EW>::kThreads, 1)
gemm_tc_pair_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                    const __grid_constant__ CUtensorMap tmC, const __grid_constant__ CUtensorMap tmR, int M, int N,
                    int K, const float* __restrict__ bias,
                    const bf16* __restrict__ resid, int ldr, bf16* __restrict__ outp, const LnPrologue lnp,
               const FoldArgs fa) {
  constexpr bool kResidBuf = ARLO_RESID_TMA && is_resid(EPI);
  constexpr int kColB = col_warp_bytes(EPI);
  using C = TcCfg<BN, true, 0, EW, kResidBuf, kColB>;
  using R = Roles<EW>;
  constexpr int kEpiWarps = R::kEpi, kEpiGroups = R::kGroups, kProducerWarp = R::kProducer, kMmaWarp = R::kMma;
  constexpr int kStagingBytes = C::kStagingBytes;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * C::A_BYTES;
  uint8_t* sStg = sB + C::STAGES * C::B_BYTES;
  uint8_t* rbuf = sStg + kEpiWarps * kColB;  // (kResidBuf) this CTA's 128 x BN residual rows
  uint64_t* full = reinterpret_cast<uint64_t*>(sStg + kStagingBytes);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;
  uint64_t* tempty = tfull + kAccStages;
  uint64_t* rfull = tempty + kAccStages;  // (local to each CTA of the pair)
  uint64_t* rfree = rfull + 1;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(rfree + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = ptx::cluster_ctarank();
  const int pair = blockIdx.x >> 1, npairs = gridDim.x >> 1;
  const int num_m = (M + 2 * BM - 1) / (2 * BM);
  const int num_n = N / BN;
  const int tiles = num_m * num_n;
  const int kblocks = K / BK;

  if (warp == kProducerWarp && lane == 0) {
    ptx::tma_prefetch_desc(&tmA);
    ptx::tma_prefetch_desc(&tmB);
    ptx::tma_prefetch_desc(&tmC);
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < kAccStages; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], 2 * kEpiWarps);  // both CTAs' epilogue warps
    }
    ptx::mbar_init(rfull, 1);
    ptx::mbar_init(rfree, kEpiWarps);
    if (kResidBuf) ptx::tma_prefetch_desc(&tmR);
    ptx::fence_mbar_init();
  }
  if (warp == kMmaWarp) ptx::tmem_alloc_pair(tmem_slot, C::TMEM_COLS);
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  pdl_launch_dependents();  // setup above overlapped the previous kernel's tail

  // W tiles of the first tile are requested before the PDL wait (see gemm_tc_kernel)
  const int pre = pair < tiles ? (kblocks < C::STAGES ? kblocks : C::STAGES) : 0;
  if (warp == kProducerWarp && lane == 0) {
    const int n0 = tile_n(pair, num_m, num_n) * BN + rank * C::B_ROWS;
    for (int kb = 0; kb < pre; ++kb) {
      if (rank == 0) ptx::mbar_arrive_expect_tx(&full[kb], 2 * C::STAGE_BYTES);
      ptx::tma_load_2d_pair(sB + kb * C::B_BYTES, &tmB, ptx::mapa_shared(&full[kb], 0), kb * BK, n0);
    }
  }
  if constexpr (EPI != EPI_BIAS_RESID) {
    if (lnp.y != nullptr) {  // A = LN(y), computed by the whole grid first (layernorm.cuh)
      pdl_wait();
      ln_prologue(lnp);
    }
  }

  if (warp == kProducerWarp) {
    if (lane == 0) {
      pdl_wait();
      if (threadIdx.x == kProducerWarp * 32) trace(0);
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int tile = pair; tile < tiles; tile += npairs, ++it) {
        trace(2 + 6 * it);
#if defined(ARLO_GEMM_SAME_TILE)  // bandwidth experiment only (wrong results): every pair loads tile 0
        const int m0 = rank * BM;
        const int n0 = rank * C::B_ROWS;
#else
        const int m0 = tile_m(tile, num_m, num_n) * 2 * BM + rank * BM;
        const int n0 = tile_n(tile, num_m, num_n) * BN + rank * C::B_ROWS;
#endif
        // this CTA's 128 residual rows of the tile, full BN columns (see gemm_tc_kernel)
        bool r_issued = !kResidBuf;
        auto issue_resid = [&]() {
          const int nr0 = tile_n(tile, num_m, num_n) * BN;
          ptx::mbar_arrive_expect_tx(rfull, (uint32_t)resid_buf_bytes<BN>());
          for (int c = 0; c < BN / CW; ++c)
            ptx::tma_load_2d(rbuf + c * (BM * CW * 2), &tmR, rfull, nr0 + c * CW, m0);
          r_issued = true;
        };
        for (int kb = 0; kb < kblocks; ++kb) {
          const uint32_t fb = ptx::mapa_shared(&full[stage], 0);
          if (it == 0 && kb < pre) {
            ptx::tma_load_2d_pair(sA + stage * C::A_BYTES, &tmA, fb, kb * BK, m0);
          } else {
            ptx::mbar_wait(&empty[stage], phase ^ 1);
            if (rank == 0) ptx::mbar_arrive_expect_tx(&full[stage], 2 * C::STAGE_BYTES);
            ptx::tma_load_2d_pair(sA + stage * C::A_BYTES, &tmA, fb, kb * BK, m0);
            ptx::tma_load_2d_pair(sB + stage * C::B_BYTES, &tmB, fb, kb * BK, n0);
          }
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
          if (!r_issued && (it == 0 || ptx::mbar_test(rfree, (it - 1) & 1))) issue_resid();
        }
        if (!r_issued) {
          ptx::mbar_wait(rfree, (it - 1) & 1);
          issue_resid();
        }
      }
    } else {
      pdl_wait();
    }
  } else if (warp == kMmaWarp) {
    pdl_wait();
    // the whole (converged) MMA warp runs the issue loop and one elected lane issues:
    // a lone lane of a diverged warp pays ~1/3 more per tcgen05.mma (tools/mma_bench.cu),
    // which measured 16.1 -> 12.3 us on the FFN2 mainloop at M = 4096
    if (rank == 0) {
      constexpr uint32_t idesc = ptx::idesc_bf16_f32(2 * BM, BN);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      int it = 0;
      for (int tile = pair; tile < tiles; tile += npairs, ++it) {
        ptx::mbar_wait(&tempty[acc], acc_phase ^ 1);
        ptx::tc_fence_after();
        if (lane == 0) trace(3 + 6 * it);
        const uint32_t d_tmem = tmem_base + acc * BN;
        for (int kb = 0; kb < kblocks; ++kb) {
          ptx::mbar_wait(&full[stage], phase);
          ptx::tc_fence_after();
          if (kb == 0 && lane == 0) trace(4 + 6 * it);
          const uint32_t a_addr = ptx::smem_u32(sA + stage * C::A_BYTES);
          const uint32_t b_addr = ptx::smem_u32(sB + stage * C::B_BYTES);
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            ptx::mma_bf16_ss_pair_w(d_tmem, ptx::desc_k_sw128(a_addr + k * 32),
                                    ptx::desc_k_sw128(b_addr + k * 32), idesc, (kb | k) != 0);
          }
          ptx::mma_commit_pair_w(&empty[stage]);
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
        }
        ptx::mma_commit_pair_w(&tfull[acc]);
        if (lane == 0) trace(5 + 6 * it);
        if (++acc == kAccStages) { acc = 0; acc_phase ^= 1; }
      }
    }
  } else {
    pdl_wait();
    const int q = warp & 3, cg = warp >> 2;
    uint8_t* stg = kResidBuf ? nullptr : sStg + warp * (kStgBufs * kStgBytes + kColB);
    float* sbias = reinterpret_cast<float*>(kResidBuf ? sStg + warp * kColB : stg + kStgBufs * kStgBytes);
    int sc = 0;
    int acc = 0;
    uint32_t acc_phase = 0;
    int it = 0;
    for (int tile = pair; tile < tiles; tile += npairs, ++it) {
      const int m0 = tile_m(tile, num_m, num_n) * 2 * BM + rank * BM, n0 = tile_n(tile, num_m, num_n) * BN;
      uint4 rv0[CW / 8];
      if (!kResidBuf) prefetch_first_resid<BN, EPI>(rv0, resid, m0 + q * 32, lane, n0, cg, M, ldr);
      stage_colv<BN, EPI, kEpiGroups>(sbias, bias, fa, n0, cg, lane);
      // LayerNorm fold: this row's statistics (of A's rows, or of the residual rows)
      float2 rowst = make_float2(0.f, -1.f);
      if constexpr (EPI >= EPI_LNFOLD) {
        const int grow = m0 + q * 32 + lane;
        const int Hs = EPI == EPI_RESID_LN ? N : K;
        if (fa.st_in != nullptr && grow < M) {
          const float2 ms = fold_row_stats(fa.st_in, (size_t)grow * fa.st_in_stride, fa.st_ld, Hs / 32, Hs, fa.eps);
          rowst = EPI == EPI_RESID_LN ? ms : make_float2(-ms.x * ms.y, ms.y);
        } else if (EPI != EPI_RESID_LN) {
          rowst = make_float2(0.f, 1.f);
        }
      }
      ptx::mbar_wait(&tfull[acc], acc_phase);
      if (kResidBuf) ptx::mbar_wait(rfull, it & 1);  // this tile's residual has landed
      ptx::tc_fence_after();
      if (warp == 0 && lane == 0) trace(6 + 6 * it);
      const uint32_t te = ptx::mapa_shared(&tempty[acc], 0);
      epilogue_tile<BN, EPI, kEpiGroups>(tmem_base + acc * BN, q, cg, lane, m0 + q * 32, n0, M, ldr, bias, resid,
                                         &tmC, stg, sc,
                             [te]() {
#if defined(ARLO_ARRIVE_RELEASE_CLUSTER)  // A/B only: the previous fenced arrive
                               ptx::mbar_arrive_cluster(te);
#else
                               ptx::mbar_arrive_remote(te);
#endif
                             }, outp, N, rv0, kResidBuf ? rbuf : nullptr, sbias, rowst, fa.st_out, fa.st_ld);
      if (kResidBuf) {
        if (lane == 0) ptx::bulk_wait_read<0>();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(rfree);
      }
      if (warp == 0 && lane == 0) trace(7 + 6 * it);
      if (++acc == kAccStages) { acc = 0; acc_phase ^= 1; }
    }
    if (lane == 0) ptx::bulk_wait<0>();
  }

  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (threadIdx.x == 0) trace(1);
  if (warp == kMmaWarp) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc_pair(tmem_base, C::TMEM_COLS);
  }
}

// ---------------------------------------------------------------------------------------------
// Skinny GEMM for small M (batch-1/2 runtimes: M = b*L <= a few hundred rows).
// At small M the projections are weight-streaming bound (b*L flop
// per weight byte, below the ridge), so what matters is how many SMs pull W:
// one non-persistent CTA per 128 x BN tile with BN in {16, 32, 64} (N/BN CTAs
// per 128-row block, e.g. 144 CTAs for the BERT-base QKV at BN = 16).  Every
// output element still accumulates the same K = 16 tcgen05.mma steps in the
// same order as the wide kernels (M = 128 instruction, only N differs), so its
// result is bitwise the wide kernels' (tests: tile widths agree bitwise).
// Warps 0-3 epilogue (TMEM lane quarter = warp), warp 4 TMA producer, warp 5
// MMA issuer.  The A box is min(128, M rounded up to 8) rows: TMEM lanes past
// it hold rows that are never stored.  The epilogue stores straight from
// registers (a row's BN*2 bytes per thread).
constexpr int kSkThreads = 192;

template <int BN>
struct SkCfg {
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE = A_BYTES + B_BYTES;
#ifndef ARLO_SKINNY_MAX_STAGES
#define ARLO_SKINNY_MAX_STAGES 12
#endif
  static constexpr int STAGES = (kSmemBudget - 1024) / STAGE > ARLO_SKINNY_MAX_STAGES ? ARLO_SKINNY_MAX_STAGES
                                                                                      : (kSmemBudget - 1024) / STAGE;
  static constexpr int SMEM = 1024 + STAGES * STAGE + 8 * (2 * STAGES + 1) + 16;
  static constexpr int TMEM_COLS = BN <= 32 ? 32 : BN;
  static_assert(SMEM <= 232448, "skinny smem");
};

template <int BN, int EPI>
__global__ void __launch_bounds__(kSkThreads, 1)
gemm_skinny_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, bf16* __restrict__ out,
                   int M, int N, int K, int a_rows, const float* __restrict__ bias, const bf16* __restrict__ resid,
                   int ldr, const FoldArgs fa) {
  using C = SkCfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * C::A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(sB + C::STAGES * C::B_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tfull + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * BN, m0 = blockIdx.y * BM;
  const int kblocks = K / BK;
  const uint32_t stage_tx = (uint32_t)(a_rows * BK * 2 + C::B_BYTES);

  if (warp == 4 && lane == 0) {
    ptx::tma_prefetch_desc(&tmA);
    ptx::tma_prefetch_desc(&tmB);
    for (int i = 0; i < C::STAGES; ++i) {
      ptx::mbar_init(&full[i], 1);
      ptx::mbar_init(&empty[i], 1);
    }
    ptx::mbar_init(tfull, 1);
    ptx::fence_mbar_init();
  }
  if (warp == 5) ptx::tmem_alloc(tmem_slot, C::TMEM_COLS);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 4) {
    if (lane == 0) {
      // weights do not depend on the predecessor kernel: start streaming W before
      // the PDL wait, then A once the producer of A has completed
      const int pre = kblocks < C::STAGES ? kblocks : C::STAGES;
      for (int kb = 0; kb < pre; ++kb) {
        ptx::mbar_arrive_expect_tx(&full[kb], stage_tx);
        ptx::tma_load_2d(sB + kb * C::B_BYTES, &tmB, &full[kb], kb * BK, n0);
      }
      pdl_begin();
      for (int kb = 0; kb < pre; ++kb) ptx::tma_load_2d(sA + kb * C::A_BYTES, &tmA, &full[kb], kb * BK, m0);
      int stage = pre % C::STAGES;
      uint32_t phase = pre == C::STAGES ? 1 : 0;
      for (int kb = pre; kb < kblocks; ++kb) {
        ptx::mbar_wait(&empty[stage], phase ^ 1);
        ptx::mbar_arrive_expect_tx(&full[stage], stage_tx);
        ptx::tma_load_2d(sB + stage * C::B_BYTES, &tmB, &full[stage], kb * BK, n0);
        ptx::tma_load_2d(sA + stage * C::A_BYTES, &tmA, &full[stage], kb * BK, m0);
        if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
      }
    }
  } else if (warp == 5) {
    // the whole (converged) warp runs the issue loop and one elected lane issues each
    // MMA: ~1/3 cheaper per instruction than a lone lane of a diverged warp
    // (tools/mma_bench.cu), which matters here because a BN = 16 MMA is only 8 tensor
    // cycles and the K chain is issue-bound
    pdl_begin();
    constexpr uint32_t idesc = ptx::idesc_bf16_f32(BM, BN);
    int stage = 0;
    uint32_t phase = 0;
#pragma unroll 1
    for (int kb = 0; kb < kblocks; ++kb) {
      ptx::mbar_wait(&full[stage], phase);
      ptx::tc_fence_after();
      const uint32_t a_addr = ptx::smem_u32(sA + stage * C::A_BYTES);
      const uint32_t b_addr = ptx::smem_u32(sB + stage * C::B_BYTES);
#pragma unroll
      for (int k = 0; k < BK / 16; ++k)
        ptx::mma_bf16_ss_w(tmem, ptx::desc_k_sw128(a_addr + k * 32), ptx::desc_k_sw128(b_addr + k * 32), idesc,
                           (kb | k) != 0);
      ptx::mma_commit_w(&empty[stage]);
      if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
    }
    ptx::mma_commit_w(tfull);
  } else {
    pdl_begin();
    // epilogue: thread = row (TMEM lane), BN columns, straight 16-byte stores
    const int row = m0 + warp * 32 + lane;
    const bool row_ok = row < M;
    float2 rowst = make_float2(0.f, -1.f);  // LayerNorm fold (see gemm_tc_kernel)
    if constexpr (EPI >= EPI_LNFOLD) {
      const int Hs = EPI == EPI_RESID_LN ? N : K;
      if (fa.st_in != nullptr && row_ok) {
        const float2 ms = fold_row_stats(fa.st_in, (size_t)row * fa.st_in_stride, fa.st_ld, Hs / 32, Hs, fa.eps);
        rowst = EPI == EPI_RESID_LN ? ms : make_float2(-ms.x * ms.y, ms.y);
      } else if (EPI != EPI_RESID_LN) {
        rowst = make_float2(0.f, 1.f);
      }
    }
    ptx::mbar_wait(tfull, 0);
    ptx::tc_fence_after();
    const uint32_t t_row = tmem + ((uint32_t)(warp * 32) << 16);
    float2 gst = make_float2(0.f, 0.f);
#pragma unroll
    for (int c0 = 0; c0 < BN; c0 += 16) {
      uint32_t r[16];
      ptx::tmem_ld_32x32b_x16(t_row + c0, r);
      ptx::tmem_wait_ld();
      if (row_ok && EPI >= EPI_LNFOLD) {
        uint32_t ru[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        if (EPI == EPI_RESID_LN) {
          const uint4* res4 = reinterpret_cast<const uint4*>(resid + (size_t)row * ldr + n0 + c0);
          const uint4 u0 = ld_dep_v4(res4), u1 = ld_dep_v4(res4 + 1);
          ru[0] = u0.x; ru[1] = u0.y; ru[2] = u0.z; ru[3] = u0.w; ru[4] = u1.x; ru[5] = u1.y; ru[6] = u1.z; ru[7] = u1.w;
        }
        uint32_t pk[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int col = n0 + c0 + 2 * j;
          const float2 a = make_float2(__uint_as_float(r[2 * j]), __uint_as_float(r[2 * j + 1]));
          const float2 v0 = make_float2(__ldg(bias + col), __ldg(bias + col + 1));
          const float2 v1 = fa.v1 ? make_float2(__ldg(fa.v1 + col), __ldg(fa.v1 + col + 1)) : f2(0.f);
          const float2 v2 = EPI == EPI_RESID_LN && fa.v2 ? make_float2(__ldg(fa.v2 + col), __ldg(fa.v2 + col + 1)) : f2(0.f);
          pk[j] = epi_fold_pair<EPI>(a, v0, v1, v2, ru[j], rowst);
        }
        uint4* o4 = reinterpret_cast<uint4*>(out + (size_t)row * N + n0 + c0);
        o4[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
        o4[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
        if (EPI == EPI_RESID_LN && fa.st_out != nullptr) {  // 32-column granules: two 16-column steps
          gst = fold_granule(pk, 8, gst);
          if (c0 & 16) {
            reinterpret_cast<float2*>(fa.st_out)[(size_t)((n0 + c0) / 32) * fa.st_ld + row] = gst;
            gst = make_float2(0.f, 0.f);
          }
        }
      } else if (row_ok) {
        uint4 rv[2];
        if (EPI == EPI_BIAS_RESID) {
          const uint4* res4 = reinterpret_cast<const uint4*>(resid + (size_t)row * ldr + n0 + c0);
          rv[0] = ld_dep_v4(res4);
          rv[1] = ld_dep_v4(res4 + 1);
        }
        uint32_t pk[8];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const float4 b4 = __ldg(reinterpret_cast<const float4*>(bias + n0 + c0) + j);
          uint32_t ua = 0, ub = 0;
          if (EPI == EPI_BIAS_RESID) {
            const uint4 u = rv[j >> 1];
            ua = (j & 1) ? u.z : u.x;
            ub = (j & 1) ? u.w : u.y;
          }
          epi_pack4<EPI>(&r[4 * j], b4, ua, ub, pk[2 * j], pk[2 * j + 1]);
        }
        uint4* o4 = reinterpret_cast<uint4*>(out + (size_t)row * N + n0 + c0);
        o4[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
        o4[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 5) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, C::TMEM_COLS);
  }
}

// ---------------------------------------------------------------------------------------------
// GEMM + bias + residual + LayerNorm over the full row (steps a4+a5 and a7+a8 fused):
//   out[M,N] = LN(A W^T + bias + resid; gamma, beta, eps),  N = hidden (768 / 1024 / 128).
// A cluster of NT = N / BN single-CTA tiles covers whole rows: CTA rank r owns
// columns [r*BN, (r+1)*BN) of the same 128-row block.  The epilogue keeps
// y = acc + bias + resid in TMEM (tcgen05.st back over the accumulator), and
// the per-row sum and sum of squared deviations are combined across the
// cluster through distributed shared memory (each warp publishes its partial
// row sums, arrives on every CTA's stat barrier with release.cluster
// semantics, waits on its own with acquire.cluster, then reads the NT x 2
// partials with ld.shared::cluster).  Two-pass statistics (mean, then
// sum (y-mean)^2) in fp32 as in the unfused LayerNorm; the normalised row is
// written once (TMA store).  Removes the LayerNorm kernels and the y round
// trip through memory.
constexpr int kMaxLnCluster = 8;  // CTAs per row block (N / BN) of the fused LayerNorm kernel

// Sum of one value per (row, column group) over every CTA of the cluster (the full row of
// the fused LayerNorm).  Each epilogue warp pushes its 32 rows' partial sums into the
// exchange buffer of EVERY CTA of the cluster with st.async, which completes transaction
// bytes on that CTA's stat barrier; each CTA arms its own barrier for the bytes of one use
// (nt CTAs x kEpiWarps warps x 32 rows x 4 B) and waits on it locally.  No fence: the
// st.async / complete_tx pair orders the data with the barrier (the previous exchange,
// an arrive.release.cluster per warp and CTA, cost a MEMBAR.ALL.GPU each).  The sum runs
// over CTAs and column groups in a fixed order, so every CTA gets the same bits.  Two
// buffer sets alternate: set s is rewritten only after the exchange between has completed
// cluster-wide, i.e. after every warp has read set s.
template <int BN>
__device__ __forceinline__ float cluster_row_sum(float v, float* red, uint64_t* stat_bar, int& use, int cg,
                                                 int r_local, int lane, uint32_t nt, uint32_t rank, int warp) {
  const int set = use & 1;
  if (warp == 0 && lane == 0) ptx::mbar_arrive_expect_tx(&stat_bar[set], nt * kEpiWarps * 32 * 4);
  float* base = red + (size_t)set * kMaxLnCluster * kEpiGroups * BM;  // red[set][cta][column group][row]
  float* slot = base + ((size_t)rank * kEpiGroups + cg) * BM + r_local;
  for (uint32_t k = 0; k < nt; ++k)
    ptx::st_async_b32(ptx::mapa_shared(slot, k), __float_as_uint(v), ptx::mapa_shared(&stat_bar[set], k));
  ptx::mbar_wait(&stat_bar[set], (use >> 1) & 1);
  float tot = 0.f;
  for (uint32_t k = 0; k < nt; ++k) {
#pragma unroll
    for (int g = 0; g < kEpiGroups; ++g) tot += base[((size_t)k * kEpiGroups + g) * BM + r_local];
  }
  ++use;
  return tot;
}

template <int BN, typename Release>
__device__ __forceinline__ void epilogue_ln_tile(uint32_t t_acc, int q, int cg, int lane, int row0, int n0, int M,
                                                 int N, float eps, const float* __restrict__ bias,
                                                 const bf16* __restrict__ resid, const float* __restrict__ gamma,
                                                 const float* __restrict__ beta, const CUtensorMap* tmC, uint8_t* stg,
                                                 int& sc, float* red, uint64_t* stat_bar, int& use, uint32_t nt,
                                                 uint32_t rank, int warp, Release release) {
  constexpr int COLS = BN / kEpiGroups;
  static_assert(COLS % 32 == 0, "fused LN epilogue: 32-column chunks");
  constexpr int NC = COLS / 32;
  const int r_local = q * 32 + lane;
  const int row = row0 + lane;
  const bool row_ok = row < M;
  const int col0 = n0 + cg * COLS;
  const float4* bias4 = reinterpret_cast<const float4*>(bias + col0);
  const float4* g4 = reinterpret_cast<const float4*>(gamma + col0);
  const float4* be4 = reinterpret_cast<const float4*>(beta + col0);
  const uint4* res4 = reinterpret_cast<const uint4*>(resid + (size_t)(row_ok ? row : 0) * N + col0);
  const uint32_t t_row = t_acc + ((uint32_t)(q * 32) << 16) + cg * COLS;
  // pass 1: y = acc + bias + resid, kept in TMEM; partial row sum
  float s1 = 0.f;
#pragma unroll 1
  for (int c = 0; c < NC; ++c) {
    uint32_t r[32];
    uint4 rv[4];
    if (row_ok) {
#pragma unroll
      for (int j = 0; j < 4; ++j) rv[j] = ld_dep_v4(res4 + c * 4 + j);
    } else {
#pragma unroll
      for (int j = 0; j < 4; ++j) rv[j] = make_uint4(0, 0, 0, 0);
    }
    ptx::tmem_ld_32x32b_x32(t_row + c * 32, r);
    ptx::tmem_wait_ld();
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float4 b4 = __ldg(bias4 + c * 8 + j);
      const uint4 u = rv[j >> 1];
      const float2 fa = unpack_bf16x2((j & 1) ? u.z : u.x), fb = unpack_bf16x2((j & 1) ? u.w : u.y);
      const float y0 = __uint_as_float(r[4 * j + 0]) + b4.x + fa.x;
      const float y1 = __uint_as_float(r[4 * j + 1]) + b4.y + fa.y;
      const float y2 = __uint_as_float(r[4 * j + 2]) + b4.z + fb.x;
      const float y3 = __uint_as_float(r[4 * j + 3]) + b4.w + fb.y;
      s1 += (y0 + y1) + (y2 + y3);
      r[4 * j + 0] = __float_as_uint(y0);
      r[4 * j + 1] = __float_as_uint(y1);
      r[4 * j + 2] = __float_as_uint(y2);
      r[4 * j + 3] = __float_as_uint(y3);
    }
    ptx::tmem_st_32x32b_x32(t_row + c * 32, r);
  }
  ptx::tmem_wait_st();
  const float mean = cluster_row_sum<BN>(s1, red, stat_bar, use, cg, r_local, lane, nt, rank, warp) / (float)N;
  // pass 2: sum of squared deviations
  float s2 = 0.f;
#pragma unroll 1
  for (int c = 0; c < NC; ++c) {
    uint32_t r[32];
    ptx::tmem_ld_32x32b_x32(t_row + c * 32, r);
    ptx::tmem_wait_ld();
#pragma unroll
    for (int j = 0; j < 32; ++j) {
      const float d = __uint_as_float(r[j]) - mean;
      s2 = fmaf(d, d, s2);
    }
  }
  const float var = cluster_row_sum<BN>(s2, red, stat_bar, use, cg, r_local, lane, nt, rank, warp) / (float)N;
  const float rstd = 1.0f / sqrtf(var + eps);
  // pass 3: normalise, affine, bf16, TMA store
#pragma unroll 1
  for (int c = 0; c < NC; ++c) {
    uint32_t r[32];
    ptx::tmem_ld_32x32b_x32(t_row + c * 32, r);
    ptx::tmem_wait_ld();
    if (c == NC - 1) {
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) release();
    }
    uint32_t pk[16];
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const float4 g = __ldg(g4 + c * 8 + j), be = __ldg(be4 + c * 8 + j);
      const float o0 = (__uint_as_float(r[4 * j + 0]) - mean) * rstd * g.x + be.x;
      const float o1 = (__uint_as_float(r[4 * j + 1]) - mean) * rstd * g.y + be.y;
      const float o2 = (__uint_as_float(r[4 * j + 2]) - mean) * rstd * g.z + be.z;
      const float o3 = (__uint_as_float(r[4 * j + 3]) - mean) * rstd * g.w + be.w;
      pk[2 * j] = pack_bf16x2(o0, o1);
      pk[2 * j + 1] = pack_bf16x2(o2, o3);
    }
    uint8_t* buf = stg + (sc & 1) * kStgBytes;
    if (sc >= 2) {
      if (lane == 0) ptx::bulk_wait_read<1>();
      __syncwarp();
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int sw = j ^ ((lane >> 1) & 3);
      *reinterpret_cast<uint4*>(buf + lane * 64 + sw * 16) =
          make_uint4(pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
    }
    ptx::fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) {
      ptx::tma_store_2d(tmC, buf, col0 + c * 32, row0);
      ptx::bulk_commit();
    }
    ++sc;
  }
}

constexpr int kLnReserve = 2 * kMaxLnCluster * kEpiGroups * BM * 4 + 16;  // row-statistics exchange + 2 barriers

template <int BN>
__global__ void __launch_bounds__(kThreads, 1)
gemm_ln_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
               const __grid_constant__ CUtensorMap tmC, int M, int N, int K, const float* __restrict__ bias,
               const bf16* __restrict__ resid, const float* __restrict__ gamma, const float* __restrict__ beta,
               float eps) {
  using C = TcCfg<BN, false, kLnReserve>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * C::A_BYTES;
  uint8_t* sStg = sB + C::STAGES * C::B_BYTES;
  float* red = reinterpret_cast<float*>(sStg + kStagingBytes);  // [2 sets][8 CTAs][column groups][128 rows]
  uint64_t* full = reinterpret_cast<uint64_t*>(red + 2 * kMaxLnCluster * kEpiGroups * BM);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;
  uint64_t* tempty = tfull + kAccStages;
  uint64_t* stat_bar = tempty + kAccStages;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(stat_bar + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint32_t nt;
  asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(nt));
  const uint32_t rank = ptx::cluster_ctarank();
  const int cid = blockIdx.x / nt, ncl = gridDim.x / nt;
  const int num_m = (M + BM - 1) / BM;
  const int n0 = rank * BN;
  const int kblocks = K / BK;

  if (warp == kProducerWarp && lane == 0) {
    ptx::tma_prefetch_desc(&tmA);
    ptx::tma_prefetch_desc(&tmB);
    ptx::tma_prefetch_desc(&tmC);
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < kAccStages; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], kEpiWarps);
    }
    for (int i = 0; i < 2; ++i) ptx::mbar_init(&stat_bar[i], 1);  // one arming arrive + the st.async bytes
    ptx::fence_mbar_init();
  }
  if (warp == kMmaWarp) ptx::tmem_alloc(tmem_slot, C::TMEM_COLS);
  ptx::tc_fence_before();
  ptx::cluster_sync();  // peers' stat barriers are initialised before any remote arrive
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  pdl_launch_dependents();

  if (warp == kProducerWarp) {
    if (lane == 0) {
      // W never depends on the previous kernel: the first row block's first W stages before the
      // PDL wait, its A stages after it (as in gemm_tc_kernel)
      const int pre = cid < num_m ? (kblocks < C::STAGES ? kblocks : C::STAGES) : 0;
      for (int kb = 0; kb < pre; ++kb) {
        ptx::mbar_arrive_expect_tx(&full[kb], C::STAGE_BYTES);
        ptx::tma_load_2d(sB + kb * C::B_BYTES, &tmB, &full[kb], kb * BK, n0);
      }
      pdl_wait();
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int mb = cid; mb < num_m; mb += ncl, ++it) {
        for (int kb = 0; kb < kblocks; ++kb) {
          if (it == 0 && kb < pre) {
            ptx::tma_load_2d(sA + stage * C::A_BYTES, &tmA, &full[stage], kb * BK, mb * BM);
          } else {
            ptx::mbar_wait(&empty[stage], phase ^ 1);
            ptx::mbar_arrive_expect_tx(&full[stage], C::STAGE_BYTES);
            ptx::tma_load_2d(sA + stage * C::A_BYTES, &tmA, &full[stage], kb * BK, mb * BM);
            ptx::tma_load_2d(sB + stage * C::B_BYTES, &tmB, &full[stage], kb * BK, n0);
          }
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
        }
      }
    } else {
      pdl_wait();
    }
  } else if (warp == kMmaWarp) {
    pdl_wait();
    {  // converged warp, elected lane issues
      constexpr uint32_t idesc = ptx::idesc_bf16_f32(BM, BN);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      for (int mb = cid; mb < num_m; mb += ncl) {
        ptx::mbar_wait(&tempty[acc], acc_phase ^ 1);
        ptx::tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BN;
        for (int kb = 0; kb < kblocks; ++kb) {
          ptx::mbar_wait(&full[stage], phase);
          ptx::tc_fence_after();
          const uint32_t a_addr = ptx::smem_u32(sA + stage * C::A_BYTES);
          const uint32_t b_addr = ptx::smem_u32(sB + stage * C::B_BYTES);
#pragma unroll
          for (int k = 0; k < BK / 16; ++k)
            ptx::mma_bf16_ss_w(d_tmem, ptx::desc_k_sw128(a_addr + k * 32), ptx::desc_k_sw128(b_addr + k * 32),
                               idesc, (kb | k) != 0);
          ptx::mma_commit_w(&empty[stage]);
          if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
        }
        ptx::mma_commit_w(&tfull[acc]);
        if (++acc == kAccStages) { acc = 0; acc_phase ^= 1; }
      }
    }
  } else {
    pdl_wait();  // residual rows come from the previous kernels
    const int q = warp & 3, cg = warp >> 2;
    uint8_t* stg = sStg + warp * kWarpStg;
    int sc = 0, use = 0;
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int mb = cid; mb < num_m; mb += ncl) {
      ptx::mbar_wait(&tfull[acc], acc_phase);
      ptx::tc_fence_after();
      uint64_t* te = &tempty[acc];
      epilogue_ln_tile<BN>(tmem_base + acc * BN, q, cg, lane, mb * BM + q * 32, n0, M, N, eps, bias, resid, gamma,
                           beta, &tmC, stg, sc, red, stat_bar, use, nt, rank, warp, [te]() { ptx::mbar_arrive(te); });
      if (++acc == kAccStages) { acc = 0; acc_phase ^= 1; }
    }
    if (lane == 0) ptx::bulk_wait<0>();
  }

  ptx::tc_fence_before();
  ptx::cluster_sync();  // no CTA leaves while a peer may still read its stats or arrive on its barriers
  if (warp == kMmaWarp) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem_base, C::TMEM_COLS);
  }
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// Resolved once, thread-safely (a function-local static is initialised exactly once even when
// runtimes are created from several host threads at the same time).
EncodeTiledFn get_encode_fn() {
  static const EncodeTiledFn fn = []() -> EncodeTiledFn {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      return reinterpret_cast<EncodeTiledFn>(p);
    return nullptr;
  }();
  return fn;
}

template <int BN, int EPI, bool PAIR, int EW>
cudaError_t launch_cfg_ew(const TcGemmPlan& p, cudaStream_t s) {
  using C = TcCfg<BN, PAIR, 0, EW, ARLO_RESID_TMA && is_resid(EPI), col_warp_bytes(EPI)>;
  auto kern = PAIR ? gemm_tc_pair_kernel<BN, EPI, EW> : gemm_tc_kernel<BN, EPI, EW>;
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t e = once_per_device(attr_done, [&] {
    return cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM); });
  if (e != cudaSuccess) return e;
  return launch_k(kern, dim3(p.grid), dim3(Roles<EW>::kThreads), C::SMEM, s, p.tmA, p.tmB, p.tmC, p.tmR, p.M, p.N,
                  p.K, p.bias, (const bf16*)p.resid, p.ldr, (bf16*)p.out, p.lnp, p.fold);
}

template <int BN, int EPI, bool PAIR>
cudaError_t launch_cfg(const TcGemmPlan& p, cudaStream_t s) {
  if constexpr (EPI == EPI_BIAS_GELU || EPI == EPI_LNFOLD_GELU) {
    if (p.ew == 12) return launch_cfg_ew<BN, EPI, PAIR, 12>(p, s);
  }
  return launch_cfg_ew<BN, EPI, PAIR, kEpiWarps>(p, s);
}

template <int BN, bool PAIR>
cudaError_t launch_bn(const TcGemmPlan& p, cudaStream_t s) {
  switch (p.epi) {
    case EPI_BIAS: return launch_cfg<BN, EPI_BIAS, PAIR>(p, s);
    case EPI_BIAS_GELU: return launch_cfg<BN, EPI_BIAS_GELU, PAIR>(p, s);
    case EPI_BIAS_RESID: return launch_cfg<BN, EPI_BIAS_RESID, PAIR>(p, s);
    case EPI_LNFOLD: return launch_cfg<BN, EPI_LNFOLD, PAIR>(p, s);
    case EPI_LNFOLD_GELU: return launch_cfg<BN, EPI_LNFOLD_GELU, PAIR>(p, s);
    case EPI_RESID_LN: return launch_cfg<BN, EPI_RESID_LN, PAIR>(p, s);
  }
  return cudaErrorInvalidValue;
}

template <int BN, int EPI>
cudaError_t launch_skinny_cfg(const TcGemmPlan& p, cudaStream_t s) {
  using C = SkCfg<BN>;
  auto kern = gemm_skinny_kernel<BN, EPI>;
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t e = once_per_device(attr_done, [&] {
    return cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM); });
  if (e != cudaSuccess) return e;
  return launch_k(kern, dim3(p.N / BN, (p.M + BM - 1) / BM), dim3(kSkThreads), C::SMEM, s, p.tmA, p.tmB,
                  (bf16*)p.out, p.M, p.N, p.K, p.a_rows, p.bias, (const bf16*)p.resid, p.ldr, p.fold);
}

template <int BN>
cudaError_t launch_skinny_bn(const TcGemmPlan& p, cudaStream_t s) {
  switch (p.epi) {
    case EPI_BIAS: return launch_skinny_cfg<BN, EPI_BIAS>(p, s);
    case EPI_BIAS_GELU: return launch_skinny_cfg<BN, EPI_BIAS_GELU>(p, s);
    case EPI_BIAS_RESID: return launch_skinny_cfg<BN, EPI_BIAS_RESID>(p, s);
    case EPI_LNFOLD: return launch_skinny_cfg<BN, EPI_LNFOLD>(p, s);
    case EPI_LNFOLD_GELU: return launch_skinny_cfg<BN, EPI_LNFOLD_GELU>(p, s);
    case EPI_RESID_LN: return launch_skinny_cfg<BN, EPI_RESID_LN>(p, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace

int set_gemm_trace(unsigned long long* buf) {
  return (int)cudaMemcpyToSymbol(g_trace, &buf, sizeof(buf));
}

int num_sms() {
  int dev = 0, n = 0;
  if (cudaGetDevice(&dev) != cudaSuccess ||
      cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0)
    n = 148;
  return n;
}

bool encode_tmap_bf16_2d(CUtensorMap* tm, const void* base, uint64_t inner, uint64_t outer,
                         uint32_t box_inner, uint32_t box_outer, int swizzle_bytes, uint64_t row_elems) {
  EncodeTiledFn fn = get_encode_fn();
  if (!fn) return false;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {(row_elems ? row_elems : inner) * 2};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box,
                  estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  swizzle_bytes == 128  ? CU_TENSOR_MAP_SWIZZLE_128B
                  : swizzle_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                  : swizzle_bytes == 32 ? CU_TENSOR_MAP_SWIZZLE_32B
                                        : CU_TENSOR_MAP_SWIZZLE_NONE,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

// 3-D bf16 map {inner, mid, outer} with packed strides (mid stride = inner, outer stride =
// inner * mid elements): tile-contiguous activations [tiles][rows][inner] (encoder_fused.cu).
bool encode_tmap_bf16_3d(CUtensorMap* tm, const void* base, uint64_t inner, uint64_t mid, uint64_t outer,
                         uint32_t box_inner, uint32_t box_mid, int swizzle_bytes) {
  EncodeTiledFn fn = get_encode_fn();
  if (!fn) return false;
  cuuint64_t dims[3] = {inner, mid, outer};
  cuuint64_t strides[2] = {inner * 2, inner * mid * 2};
  cuuint32_t box[3] = {box_inner, box_mid, 1};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = fn(tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE,
                  swizzle_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

// Tile choice: a function of (M, N, K) only (never of the data), minimising a
// wave-quantised time estimate fitted to graph-replayed B200 sweeps
// (tools/gemm_sweep.py --set small/base/large/mid: over 39 shapes the pick is
// the measured best or within 3 % of it on all but two, 11 % and 22 % off):
//   wide kernels:  waves * (2.5 us + kblocks * max(MMA time of one 64-deep
//                  k-block / eff(pair, BN), 0.12 us)),
//   skinny kernel: waves * (2.5 us + kblocks * (0.11 + 0.0005 BN) us).
// eff is the fraction of the tensor pipe a tile shape sustains (operand
// staging per flop: the CTA pair at BN = 256 is best, single-CTA BN = 256 pays
// for its 32 KB W stage).  Returns BN for the single-CTA kernel, -BN for the
// CTA-pair kernel, kSkinnyCode + BN for the skinny kernel.
int tc_choose_bn(int M, int N, int K) {
  const int sms = num_sms();
  const double kblocks = K / BK;
  double best = 1e30;
  int best_bn = 0;
  struct Cand { int code; double eff; };
  const Cand cands[8] = {{-256, 0.75}, {-192, 0.65}, {256, 0.45}, {192, 0.70}, {-128, 0.50}, {128, 0.60}, {96, 0.55},
                         {64, 0.45}};
  for (const Cand& c : cands) {
    const bool pair = c.code < 0;
    const int bn = pair ? -c.code : c.code;
    if (N % bn) continue;
    const int tile_m = pair ? 2 * BM : BM;
    const long tiles = (long)((M + tile_m - 1) / tile_m) * (N / bn);
    const long slots = pair ? sms / 2 : sms;
    const long waves = (tiles + slots - 1) / slots;
    const double mma_kb_us = (double)tile_m * bn * BK * 2 / (pair ? 16384.0 : 8192.0) / 1.9e3;
    const double per_kb = mma_kb_us / c.eff > 0.12 ? mma_kb_us / c.eff : 0.12;
    const double t = waves * (2.5 + kblocks * per_kb);
    if (t < best * 0.999) { best = t; best_bn = c.code; }
  }
  if (M <= 1024 && getenv("ARLO_NO_SKINNY") == nullptr) {
    for (int bn : {16, 32, 64}) {
      if (N % bn) continue;
      const long ctas = (long)((M + BM - 1) / BM) * (N / bn);
      const long waves = (ctas + sms - 1) / sms;
      const double t = waves * (2.5 + kblocks * (0.11 + 0.0005 * bn));
      if (t < best * 0.999) { best = t; best_bn = kSkinnyCode + bn; }
    }
  }
  return best_bn;
}

bool tc_plan_gemm(TcGemmPlan* p, int M, int N, int K, const void* A, const void* W,
                  const float* bias, const void* resid, void* out, int epi, int force_bn) {
  return tc_plan_gemm_strided(p, M, N, K, A, K, W, bias, resid, N, out, epi, force_bn);
}

bool tc_plan_gemm_strided(TcGemmPlan* p, int M, int N, int K, const void* A, int lda, const void* W,
                          const float* bias, const void* resid, int ldr, void* out, int epi, int force_bn) {
  if (M <= 0 || N % 64 || K % 64 || K <= 0 || lda < K || lda % 8 || ldr < N || ldr % 8) return false;
  if (force_bn > kSplitKCode)
    return tc_plan_gemm_splitk(p, M, N, K, A, lda, W, bias, resid, ldr, out, epi, force_bn - kSplitKCode);
  const int choice = force_bn ? force_bn : tc_choose_bn(M, N, K);
  if (choice > kSkinnyCode) {
    int bn = choice - kSkinnyCode;
    if (epi == EPI_RESID_LN && bn == 16) bn = 32;  // statistics granule: 32 columns of one CTA
    if ((bn != 16 && bn != 32 && bn != 64) || N % bn) return false;
    p->M = M; p->N = N; p->K = K; p->BN = bn; p->pair = false; p->skinny = true; p->splitk = false; p->fold = FoldArgs{}; p->lnp = LnPrologue{}; p->epi = epi; p->ln = false; p->ew = 4;
    p->bias = bias; p->resid = resid; p->ldr = ldr; p->out = out;
    p->a_rows = M < BM ? ((M + 7) & ~7) : BM;
    p->grid = (N / bn) * ((M + BM - 1) / BM);
    if (!encode_tmap_bf16_2d(&p->tmA, A, (uint64_t)K, (uint64_t)M, BK, p->a_rows, 128, (uint64_t)lda)) return false;
    if (!encode_tmap_bf16_2d(&p->tmB, W, (uint64_t)K, (uint64_t)N, BK, bn, 128)) return false;
    return true;
  }
  const bool pair = choice < 0;
  const int bn = pair ? -choice : choice;
  if (bn != 64 && bn != 96 && bn != 128 && bn != 192 && bn != 256) return false;
  if (pair && bn < 128) return false;
  if (N % bn) return false;
  p->M = M; p->N = N; p->K = K; p->BN = bn; p->pair = pair; p->skinny = false; p->splitk = false; p->lnp = LnPrologue{}; p->epi = epi; p->ln = false;
  p->bias = bias; p->resid = resid; p->ldr = ldr; p->out = out;
  const int tile_m = pair ? 2 * BM : BM;
  const int tiles = ((M + tile_m - 1) / tile_m) * (N / bn);
  const int slots = pair ? num_sms() / 2 : num_sms();
  p->grid = (tiles < slots ? tiles : slots) * (pair ? 2 : 1);
#ifndef ARLO_GELU_EW12_MAX_M
#define ARLO_GELU_EW12_MAX_M 0  // A/B hook: 8192 = 12 epilogue warps for GELU at M <= 8192 (round 1)
#endif
  p->ew = ((epi == EPI_BIAS_GELU || epi == EPI_LNFOLD_GELU) && M <= ARLO_GELU_EW12_MAX_M) ? 12 : kEpiWarps;
  p->fold = FoldArgs{};
  if (!encode_tmap_bf16_2d(&p->tmA, A, (uint64_t)K, (uint64_t)M, BK, BM, 128, (uint64_t)lda)) return false;
  if (!encode_tmap_bf16_2d(&p->tmB, W, (uint64_t)K, (uint64_t)N, BK, pair ? bn / 2 : bn, 128)) return false;
  if (!encode_tmap_bf16_2d(&p->tmC, out, (uint64_t)N, (uint64_t)M, CW, 32, CW * 2)) return false;
  // residual rows (stride ldr), {32 columns x 128 rows} boxes in the output staging layout
  if ((epi == EPI_BIAS_RESID || epi == EPI_RESID_LN) &&
      !encode_tmap_bf16_2d(&p->tmR, resid, (uint64_t)N, (uint64_t)M, CW, BM, CW * 2, (uint64_t)ldr))
    return false;
  return true;
}

template <int BN>
cudaError_t launch_ln(const TcGemmPlan& p, cudaStream_t s) {
  using C = TcCfg<BN, false, kLnReserve>;
  constexpr int SMEM = C::SMEM;
  static_assert(SMEM <= 232448, "fused LN smem");
  auto kern = gemm_ln_kernel<BN>;
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t e = once_per_device(attr_done, [&] {
    cudaError_t r = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM);
    if (r == cudaSuccess) r = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    return r; });
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(p.grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = SMEM;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = p.N / BN;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, p.tmA, p.tmB, p.tmC, p.M, p.N, p.K, p.bias, (const bf16*)p.resid, p.gamma,
                            p.beta, p.eps);
}

// Fused GEMM + bias + residual + LayerNorm over full rows (N = hidden).
bool tc_plan_gemm_ln(TcGemmPlan* p, int M, int N, int K, const void* A, const void* W, const float* bias,
                     const void* resid, const float* gamma, const float* beta, float eps, void* out) {
  if (M <= 0 || K % 64 || K <= 0) return false;
  int bn = 0;
  // the widest tile that still gives >= 4 CTAs per row block (more CTAs per wave): N = 768 -> 192 x 4,
  // N = 1024 -> 256 x 4
  if (N % 256 == 0 && N / 256 <= 8 && (256 / kEpiGroups) % 32 == 0 && 256 % kEpiGroups == 0) bn = 256;
  if (N % 192 == 0 && N / 192 <= 8 && N / 192 >= 4 && (N % 256 || N / 256 < 4) && (192 / kEpiGroups) % 32 == 0)
    bn = 192;
  if (N == 128 && (128 / kEpiGroups) % 32 == 0 && 128 % kEpiGroups == 0) bn = 128;
  if (!bn) return false;
  const int nt = N / bn;
  p->M = M; p->N = N; p->K = K; p->BN = bn; p->pair = false; p->skinny = false; p->splitk = false; p->lnp = LnPrologue{}; p->epi = EPI_BIAS_RESID; p->ln = true; p->fold = FoldArgs{};
  p->ew = kEpiWarps;
  p->bias = bias; p->resid = resid; p->ldr = N; p->out = out; p->gamma = gamma; p->beta = beta; p->eps = eps;
  const int num_m = (M + BM - 1) / BM;
  const int clusters = num_sms() / nt;
  p->grid = (num_m < clusters ? num_m : clusters) * nt;
  if (!encode_tmap_bf16_2d(&p->tmA, A, (uint64_t)K, (uint64_t)M, BK, BM, 128)) return false;
  if (!encode_tmap_bf16_2d(&p->tmB, W, (uint64_t)K, (uint64_t)N, BK, bn, 128)) return false;
  if (!encode_tmap_bf16_2d(&p->tmC, out, (uint64_t)N, (uint64_t)M, CW, 32, CW * 2)) return false;
  return true;
}

bool tc_plan_attach_ln(TcGemmPlan* p, const LnPrologue& lnp) {
  // persistent tile kernels only (grid <= one CTA per SM: every CTA resident for the grid barrier)
  if (p->skinny || p->splitk || p->ln || p->epi == EPI_BIAS_RESID) return false;
  if (lnp.H % 8 || lnp.H > 1024 || lnp.rows <= 0 || !lnp.y || !lnp.x || !lnp.bar) return false;
  if (p->grid > num_sms()) return false;
  p->lnp = lnp;
  return true;
}

cudaError_t tc_launch_gemm(const TcGemmPlan& p, cudaStream_t s) {
  if (p.splitk) return splitk_launch(p, s);
  if (p.skinny) {
    switch (p.BN) {
      case 16: return launch_skinny_bn<16>(p, s);
      case 32: return launch_skinny_bn<32>(p, s);
      case 64: return launch_skinny_bn<64>(p, s);
    }
    return cudaErrorInvalidValue;
  }
  if (p.ln) {
    switch (p.BN) {
      case 128:
        if constexpr ((128 / kEpiGroups) % 32 == 0 && 128 % kEpiGroups == 0) return launch_ln<128>(p, s);
        return cudaErrorInvalidValue;
      case 192:
        if constexpr ((192 / kEpiGroups) % 32 == 0 && 192 % kEpiGroups == 0) return launch_ln<192>(p, s);
        return cudaErrorInvalidValue;
      case 256:
        if constexpr ((256 / kEpiGroups) % 32 == 0 && 256 % kEpiGroups == 0) return launch_ln<256>(p, s);
        return cudaErrorInvalidValue;
    }
    return cudaErrorInvalidValue;
  }
  if (p.pair) {
    switch (p.BN) {
      case 128: return launch_bn<128, true>(p, s);
      case 192: return launch_bn<192, true>(p, s);
      case 256: return launch_bn<256, true>(p, s);
    }
    return cudaErrorInvalidValue;
  }
  switch (p.BN) {
    case 64: return launch_bn<64, false>(p, s);
    case 96: return launch_bn<96, false>(p, s);
    case 128: return launch_bn<128, false>(p, s);
    case 192: return launch_bn<192, false>(p, s);
    case 256: return launch_bn<256, false>(p, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace arlo
