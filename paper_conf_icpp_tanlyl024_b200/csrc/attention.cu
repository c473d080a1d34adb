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

#include <type_traits>

namespace arlo {
namespace {

constexpr int D = 64;        // head dim (all configs)
constexpr int AQ = 128;      // queries per q-tile (TMEM lanes)
constexpr int AK = 128;      // keys per K/V tile (TMA unit)
constexpr int KC = 64;       // keys per softmax chunk (S MMA N)
constexpr int kTileBytes = 128 * 128;         // 128 rows x 64 bf16 (128 B), SWIZZLE_128B
// Softmax exponentials: of every 16-key piece, the last kPolyPairs key pairs are evaluated by
// ex2_poly2 on the FMA pipe, the rest by MUFU ex2 (16/clk/SM, the softmax's binding unit at
// head dim 64).  A function of the key position only: every runtime computes a key's p alike.
#ifndef ARLO_EXP_POLY_PAIRS
#define ARLO_EXP_POLY_PAIRS 0  // measured: 1-4 pairs no faster at L = 64..512 (the softmax is not MUFU-bound)
#endif
constexpr int kPolyPairs = ARLO_EXP_POLY_PAIRS;

// Launch shape per runtime length: NQ q-tiles per CTA, up to MAXKT 128-key
// K/V tiles (L <= 128 * MAXKT), NS S/P slots per q-tile.  NQ = 1 (L <= 128)
// keeps smem (48 KB) and TMEM (256 columns) small enough for two CTAs per SM.
template <int NQ_, int MAXKT_, int NS_>
struct AttnCfg {
  static constexpr int NQ = NQ_;
  static constexpr int NS = NS_;  // S and P (TMEM) slots per q-tile
  static constexpr int kMaxKT = MAXKT_;
  static constexpr int kKSlots = MAXKT_ < 2 ? MAXKT_ : 2;  // K and V tile rings (2 slots each)
  // softmax warp w: q-tile w/8, key half (w/4)%2 of every chunk, TMEM lane quarter w%4
  static constexpr int kSoftWarps = 8 * NQ;
  static constexpr int kProdWarp = kSoftWarps;
  // MMA issuers of q-tile qi: warp kMmaWarp + 2 qi issues the S = Q K^T MMAs, warp
  // kMmaWarp + 2 qi + 1 the O += P V MMAs (two independent issue chains)
  static constexpr int kMmaWarp = kSoftWarps + 1;
  static constexpr int kThreads = 32 * (kSoftWarps + 1 + 2 * NQ);
  static constexpr int kSmem = 1024 + kTileBytes * (NQ + 2 * kKSlots) + 256;
  // TMEM columns, q-tile qi: S slot sl (64 fp32) at qi*NS*64 + sl*64; O (64 fp32)
  // at kOCol + qi*64; P slot sl (64 bf16 packed in 32 columns) at kPCol + (qi*NS + sl)*32
  static constexpr uint32_t kOCol = NQ * NS * KC;
  static constexpr uint32_t kPCol = kOCol + NQ * D;
  // ALIAS (NS == 1): a warp writes its 32 keys of P (16 packed columns) over the first 16
  // columns of its own 32 S columns, after its S values are in registers.  TMEM per q-tile
  // is then 64 (S/P) + 64 (O) columns: 128 per CTA, so three CTAs share an SM (the b = 32,
  // L <= 128 grids of 384 CTAs run in one wave instead of 1.3).  The next S MMA into the
  // slot waits for the PV MMA that read P from it.
  static constexpr bool ALIAS = NS == 1;
  static constexpr uint32_t kUsedCols = ALIAS ? NQ * (NS * KC + D) : NQ * (NS * KC + D + NS * KC / 2);
  static constexpr uint32_t kTmemCols = kUsedCols <= 128 ? 128 : kUsedCols <= 256 ? 256 : 512;
  static_assert(kUsedCols <= 512, "attention TMEM");
  static constexpr int kMinBlocks = ALIAS ? 3 : 512 / kTmemCols < 2 ? 1 : 2;
  static_assert(kSmem * kMinBlocks <= 232448, "attention smem");
};

// Profiling hook (arlo_debug_attn_trace): the TRACE=true instantiation writes
// Timeline of the first 2048 CTAs into g_atrace[cta * 64 + slot]: slots 0/1 are
// %globaltimer at start/end (cross-SM), 62/63 clock64 at start/end (to convert),
// every other slot is clock64 (cycle resolution within the SM).
__device__ unsigned long long* g_atrace = nullptr;
template <bool TRACE>
__device__ __forceinline__ void atrace(int slot) {
  if (TRACE) {
    const unsigned cta = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
    if (cta < 2048 && slot < 64) {
      unsigned long long t;
      if (slot < 2) {
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        g_atrace[cta * 64 + 62 + slot] = clock64();
      } else {
        t = clock64();
      }
      g_atrace[cta * 64 + slot] = t;
    }
  }
}

// One CTA = (two 128-query tiles, head, sequence).  Keys are processed in
// 64-key chunks: S_qi,c = Q_qi K_c^T (M=128, N=64, K=64) into a double-buffered
// TMEM S slot, O_qi += P_qi,c V_c (M=128, N=64, K=64; V an MN-major B operand)
// into TMEM.  Four softmax warps per q-tile (thread = query row = TMEM lane);
// at head dim 64 the TMEM->RF reads of S and the exp2 (MUFU) work, not the
// tensor pipe, bound attention.  A lazily-rescaled
// running max is kept (O rescaled in TMEM only when a chunk raises a row max
// enough that its p sum passes 2^8); P is written as packed bf16 back into
// TMEM (tcgen05.st) and read from there as the PV MMA's A operand, so P never
// touches shared memory.  S/P slots are double-buffered so S(c+1) is computed
// while chunk c is in the exp stage.  Q, K (2-tile ring) and V (resident, <= 4 tiles) come
// in by TMA once per CTA and are shared by both q-tiles.  Key chunks starting
// at >= len are never loaded or multiplied; keys >= len inside the last chunk
// get p = 0.
//
// PACK = 2 (runtimes with L = 64): one 128-row tile holds two consecutive sequences
// (rows b*64 .. b*64+127 of the QKV buffer are sequences b and b+1), so a CTA serves
// both instead of computing a 128-row tile of which only the first 64 rows are kept.
// Chunk c (keys 64c .. 64c+63 of the tile) is sequence c's keys: the softmax warps of
// lane quarters 2c, 2c+1 (rows of sequence c) treat chunk c as their first and only
// chunk (exactly the arithmetic of an unpacked CTA with len <= 64) and write P = 0 for
// the other chunk, so O_c = P_c V_c + 0 * V_other: bitwise the unpacked rows (the
// cross-L contract), in half the CTAs (b = 32: 192 instead of 384, one wave).
template <int NQ_, int MAXKT_, int NS_, bool TRACE, int PACK>
__global__ void __launch_bounds__(AttnCfg<NQ_, MAXKT_, NS_>::kThreads, AttnCfg<NQ_, MAXKT_, NS_>::kMinBlocks)
attn_tc_kernel(const __grid_constant__ CUtensorMap tm, int B, int L, int heads, const int32_t* __restrict__ lengths,
               bf16* __restrict__ o) {
  static_assert(PACK == 1 || (PACK == 2 && NQ_ == 1 && MAXKT_ == 1 && NS_ == 2), "packed tiles: L = 64 shape");
  using Cfg = AttnCfg<NQ_, MAXKT_, NS_>;
  constexpr int NS = Cfg::NS;
  constexpr int NQ = Cfg::NQ, kMaxKT = Cfg::kMaxKT, kKSlots = Cfg::kKSlots;
  constexpr int kSoftWarps = Cfg::kSoftWarps, kProdWarp = Cfg::kProdWarp, kMmaWarp = Cfg::kMmaWarp;
  constexpr int kAttnThreads = Cfg::kThreads;
  constexpr uint32_t kOCol = Cfg::kOCol, kPCol = Cfg::kPCol, kTmemCols = Cfg::kTmemCols;
  // PDL: barrier init and the TMEM allocation below overlap the previous kernel's tail;
  // nothing the previous kernels write (QKV) or read (O) is touched before pdl_wait().
  // `lengths` is filled by the runtime's input copy, which precedes every kernel of the graph.
  pdl_launch_dependents();
  const int h = blockIdx.y, b = blockIdx.z * PACK;  // (first) sequence of the tile
  const int H = heads * D;
  // lengths come from device memory unvalidated (arlo_enqueue, arlo_op_attention): clamp to
  // [0, L] so a bad length can neither index barriers past kMaxKT nor read the next sequence
  const int len_a = min(max(__ldg(lengths + b), 0), L);
  const int len_b = PACK == 2 && b + 1 < B ? min(max(__ldg(lengths + b + 1), 0), L) : 0;
  const int len = PACK == 2 ? (len_a > len_b ? len_a : len_b) : len_a;  // (PACK: live if either is)
  const int q0 = blockIdx.x * (NQ * AQ);
  const int row_base = b * L;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (q0 >= len) {  // every q-tile wholly padded (or empty slot): zeros
    pdl_wait();
    const int rows = PACK == 2 ? (b + 1 < B ? 2 * L : L) : min(NQ * AQ, L - q0);
    for (int i = threadIdx.x; i < rows * 8; i += kAttnThreads) {
      const int r = i >> 3, c = i & 7;
      *reinterpret_cast<uint4*>(o + (size_t)(row_base + q0 + r) * H + h * D + c * 8) = make_uint4(0, 0, 0, 0);
    }
    return;
  }
  const int n_kt = PACK == 2 ? 1 : (len + AK - 1) / AK;  // K/V tiles
  const int n_ch = PACK == 2 ? 2 : (len + KC - 1) / KC;  // 64-key chunks
  int nq = 1;  // live q-tiles (trailing ones may be wholly padded)
  while (nq < NQ && q0 + nq * AQ < len) ++nq;

  extern __shared__ uint8_t smem_raw[];
  __shared__ float xch[NQ][2][2 * AQ];  // softmax pair exchange: [q-tile][half][chunk parity][row]
  __shared__ float xmax[NQ][2][AQ];     // redo maxima, final partial sums
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + NQ * kTileBytes;
  uint8_t* sV = sK + kKSlots * kTileBytes;
  uint64_t* bar_k = reinterpret_cast<uint64_t*>(sV + kKSlots * kTileBytes);
  uint64_t* bar_v = bar_k + kMaxKT;
  uint64_t* k_free = bar_v + kMaxKT;
  uint64_t* v_free = k_free + kKSlots;
  uint64_t* s_full = v_free + kKSlots;  // [NQ][NS]
  uint64_t* s_free = s_full + NS * NQ;
  uint64_t* p_full = s_free + NS * NQ;
  uint64_t* pv_done = p_full + NS * NQ;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(pv_done + NS * NQ);

  if (warp == kProdWarp && lane == 0) {
    ptx::tma_prefetch_desc(&tm);
    for (int j = 0; j < kMaxKT; ++j) {
      ptx::mbar_init(&bar_k[j], 1);
      ptx::mbar_init(&bar_v[j], 1);
    }
    for (int i = 0; i < kKSlots; ++i) {  // one commit per live q-tile
      ptx::mbar_init(&k_free[i], nq);
      ptx::mbar_init(&v_free[i], nq);
    }
    for (int i = 0; i < NS * NQ; ++i) {
      ptx::mbar_init(&s_full[i], 1);
      ptx::mbar_init(&s_free[i], 8);
      ptx::mbar_init(&p_full[i], 8);
      ptx::mbar_init(&pv_done[i], 1);
    }
    ptx::fence_mbar_init();
  }
  if (warp == kMmaWarp) ptx::tmem_alloc(tmem_slot, kTmemCols);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();
  if (threadIdx.x == 0) atrace<TRACE>(0);

  if (warp == kProdWarp) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0) {
      ptx::mbar_arrive_expect_tx(&bar_k[0], (nq + 1) * kTileBytes);
      for (int qi = 0; qi < nq; ++qi)
        ptx::tma_load_2d(sQ + qi * kTileBytes, &tm, &bar_k[0], h * D, row_base + q0 + qi * AQ);
      ptx::tma_load_2d(sK, &tm, &bar_k[0], H + h * D, row_base);
      // K and V rings: slot j%2 of K (V) frees when the S (PV) MMAs of tile j-2 complete
      for (int j = 0; j < n_kt; ++j) {
        if (j > 0) {
          if (j >= kKSlots) ptx::mbar_wait(&k_free[j & 1], ((j - kKSlots) >> 1) & 1);
          ptx::mbar_arrive_expect_tx(&bar_k[j], kTileBytes);
          ptx::tma_load_2d(sK + (j & 1) * kTileBytes, &tm, &bar_k[j], H + h * D, row_base + j * AK);
        }
        if (j >= kKSlots) ptx::mbar_wait(&v_free[j & 1], ((j - kKSlots) >> 1) & 1);
        ptx::mbar_arrive_expect_tx(&bar_v[j], kTileBytes);
        ptx::tma_load_2d(sV + (j & 1) * kTileBytes, &tm, &bar_v[j], 2 * H + h * D, row_base + j * AK);
      }
    }
  } else if (warp >= kMmaWarp) {
    // ------------------------------------------------------------ MMA issuers
    // Two issuing warps per q-tile.  A tcgen05.mma costs its issuing thread
    // ~50-200 cycles at these shapes (M=128, N=64, K=16; tools/mma_bench.cu),
    // so one thread issuing both S(c+1) and PV(c) (8 MMAs per 64-key chunk) was
    // the per-chunk critical path; with S and PV on separate chains each chunk
    // costs at most 4 MMA issues per chain.  S(c) is issued as soon as its TMEM
    // slot is free and its K tile has landed; PV(c) once P(c) is written.
    const int qi = (warp - kMmaWarp) >> 1;
    const bool pv_role = ((warp - kMmaWarp) & 1) != 0;
    if (qi < nq) {
      if (pv_role) {
        constexpr uint32_t idesc_pv = ptx::idesc_bf16_f32_bmn(AQ, D);
#pragma unroll 1
        for (int c = 0; c < n_ch; ++c) {
          const int t = c >> 1, sl = c % NS;
          ptx::mbar_wait(&p_full[qi * NS + sl], (c / NS) & 1);
          ptx::mbar_wait(&bar_v[t], 0);
          ptx::tc_fence_after();
          // P of keys [16 ks, 16 ks + 16): half ks / 2, 8 packed columns per K = 16 step
          const uint32_t p_tmem = Cfg::ALIAS ? tmem + (qi * NS + sl) * KC : tmem + kPCol + (qi * NS + sl) * (KC / 2);
          const uint32_t v_addr = ptx::smem_u32(sV + (t & 1) * kTileBytes + (c & 1) * (KC * 128));
#pragma unroll
          for (int ks = 0; ks < KC / 16; ++ks)  // 16 keys = 8 packed P columns per step
            ptx::mma_bf16_ts_w(tmem + kOCol + qi * D,
                               p_tmem + (Cfg::ALIAS ? (ks >> 1) * (KC / 2) + (ks & 1) * 8 : ks * 8),
                               ptx::desc_mn_sw128(v_addr + ks * 2048, 0),
                               idesc_pv, (c | ks) != 0);
          ptx::mma_commit_w(&pv_done[qi * NS + sl]);
          if ((c & 1) || c == n_ch - 1) ptx::mma_commit_w(&v_free[t & 1]);  // V tile t done for this q-tile
          if (qi == 0 && c < 14 && lane == 0) atrace<TRACE>(48 + c);  // PV(0, c) issued
        }
      } else {
        constexpr uint32_t idesc_s = ptx::idesc_bf16_f32(AQ, KC);
        const uint32_t q_addr = ptx::smem_u32(sQ + qi * kTileBytes);
#pragma unroll 1
        for (int c = 0; c < n_ch; ++c) {
          const int t = c >> 1, sl = c % NS;
          if (c >= NS) ptx::mbar_wait(&s_free[qi * NS + sl], ((c - NS) / NS) & 1);
          if (Cfg::ALIAS && c >= NS) ptx::mbar_wait(&pv_done[qi * NS + sl], ((c - NS) / NS) & 1);
          ptx::mbar_wait(&bar_k[t], 0);
          ptx::tc_fence_after();
          const uint32_t k_addr = ptx::smem_u32(sK + (t & 1) * kTileBytes + (c & 1) * (KC * 128));
#pragma unroll
          for (int k = 0; k < D / 16; ++k)
            ptx::mma_bf16_ss_w(tmem + qi * NS * KC + sl * KC, ptx::desc_k_sw128(q_addr + k * 32),
                               ptx::desc_k_sw128(k_addr + k * 32), idesc_s, k > 0);
          ptx::mma_commit_w(&s_full[qi * NS + sl]);
          // K tile t is released (for this q-tile) once the S MMAs of both its chunks complete
          if ((c & 1) || c == n_ch - 1) ptx::mma_commit_w(&k_free[t & 1]);
          if (qi == 0 && c < 16 && lane == 0) atrace<TRACE>(32 + c);  // S(0, c) issued
        }
      }
    }
  } else {
    // ----------------------------------------------------------------- softmax
    // Two warps per TMEM lane quarter (same 32 query rows): warp half hf owns
    // keys [32 hf, 32 hf + 32) of every 64-key chunk, O columns [32 hf, 32 hf + 32)
    // and a partial row sum.  The pair shares one running max per row through
    // shared memory (a 64-thread named barrier per chunk), so both halves of a
    // row's P use the same scale.
    const int qi = warp >> 3, hf = (warp >> 2) & 1, quarter = warp & 3;
    const int r = quarter * 32 + lane;  // query row within q-tile qi == TMEM lane
    const int qrow = q0 + qi * AQ + r;
    // PACK: this warp's rows are sequence `seg` of the tile, its only real chunk is chunk seg
    const int seg = PACK == 2 ? quarter >> 1 : 0;
    const int lenw = PACK == 2 ? (seg ? len_b : len_a) : len;
    const bool row_live = PACK == 2 ? (b + seg < B) : (qrow < L);  // row exists in the buffer
    const int bar_id = 1 + qi * 4 + quarter;
    auto pair_sync = [&]() { asm volatile("bar.sync %0, 64;" ::"r"(bar_id) : "memory"); };
    if (qi < nq) {
      const uint32_t t_lane = tmem + ((uint32_t)(quarter * 32) << 16);
      const uint32_t t_s = t_lane + qi * NS * KC + hf * (KC / 2);
      const uint32_t t_o = t_lane + kOCol + qi * D + hf * (D / 2);
      const float c2 = 0.125f * 1.4426950408889634f;  // 1/sqrt(64) * log2(e)
      float m = -INFINITY, l = 0.f;
      // 16 keys: p = 2^(s*c2 - mc) (0 past len when MASK), fp32 partial sums,
      // packed bf16 into the row's 8 TMEM P columns for these keys.  MASK is a
      // compile-time flag: only a chunk straddling len pays for masking.
      auto exp_piece = [&](auto mask_tag, const uint32_t (&v)[16], int key0, float mc, uint32_t t_p,
                           float (&ls)[2]) {
        constexpr bool MASK = decltype(mask_tag)::value;
        uint32_t pk[8];
        float2 acc = make_float2(ls[0], ls[1]);
#pragma unroll
        for (int e = 0; e < 16; e += 2) {
          // paired FFMA2 / FADD2: bitwise the scalar fmaf / += (even keys into ls[0], odd into ls[1])
          const float2 x = __ffma2_rn(make_float2(__uint_as_float(v[e]), __uint_as_float(v[e + 1])),
                                      make_float2(c2, c2), make_float2(-mc, -mc));
          float p0, p1;
          if (e >= 16 - 2 * kPolyPairs) {  // the last kPolyPairs key pairs of a piece on the FMA pipe
            const float2 pp = ex2_poly2(x);
            p0 = pp.x;
            p1 = pp.y;
          } else {
            p0 = ex2_approx(x.x);
            p1 = ex2_approx(x.y);
          }
          if (MASK) {
            if (key0 + e >= lenw) p0 = 0.f;
            if (key0 + e + 1 >= lenw) p1 = 0.f;
          }
          acc = __fadd2_rn(acc, make_float2(p0, p1));
          pk[e >> 1] = pack_bf16x2(p0, p1);
        }
        ls[0] = acc.x;
        ls[1] = acc.y;
        ptx::tmem_st_32x32b_x8(t_p, pk);
      };
      // this warp's 32 keys of a chunk against max mc; returns the partial p sum
      auto exp_half = [&](auto mask_tag, uint32_t t_chunk, float mc, int key0, uint32_t t_p) {
        float ls[2] = {0.f, 0.f};
        uint32_t va[16], vb[16];
        ptx::tmem_ld_32x32b_x16(t_chunk, va);
        ptx::tmem_ld_32x32b_x16(t_chunk + 16, vb);
        ptx::tmem_wait_ld();
        exp_piece(mask_tag, va, key0, mc, t_p, ls);
        exp_piece(mask_tag, vb, key0 + 16, mc, t_p + 8, ls);
        return ls[0] + ls[1];
      };
      auto exp_any = [&](bool full, uint32_t t_chunk, float mc, int key0, uint32_t t_p) {
        return full ? exp_half(std::false_type{}, t_chunk, mc, key0, t_p)
                    : exp_half(std::true_type{}, t_chunk, mc, key0, t_p);
      };
      // row max over this warp's 32 keys of a chunk (first chunk, or the rare redo)
      auto half_max = [&](bool full, uint32_t t_chunk, int key0) {
        float mx[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
        uint32_t va[16], vb[16];
        ptx::tmem_ld_32x32b_x16(t_chunk, va);
        ptx::tmem_ld_32x32b_x16(t_chunk + 16, vb);
        ptx::tmem_wait_ld();
#pragma unroll
        for (int e = 0; e < 16; ++e) {
          if (full || key0 + e < lenw) mx[e & 3] = fmaxf(mx[e & 3], __uint_as_float(va[e]));
          if (full || key0 + 16 + e < lenw) mx[e & 3] = fmaxf(mx[e & 3], __uint_as_float(vb[e]));
        }
        return fmaxf(fmaxf(mx[0], mx[1]), fmaxf(mx[2], mx[3]));
      };
      float* xs = xch[qi][hf];        // this warp's exchange row (chunk-parity double-buffered)
      float* xp = xch[qi][hf ^ 1];    // partner's
#pragma unroll 1
      for (int c = 0; c < n_ch; ++c) {
        const int cur = c % NS, par = c & 1;
        ptx::mbar_wait(&s_full[qi * NS + cur], (c / NS) & 1);
        ptx::tc_fence_after();
        if (warp == 0 && lane == 0) atrace<TRACE>(3 + 3 * (c & 7));
        const int key0 = (c - seg) * KC + hf * (KC / 2);  // key index within the warp's sequence
        const bool full = (c - seg) * KC + KC <= lenw;
        const uint32_t t_chunk = t_s + cur * KC;
        const uint32_t t_p = t_lane + kPCol + (qi * NS + cur) * (KC / 2) + hf * (KC / 4);
        // P slot `cur` was read by PV(c - NS)
        if (c >= NS) {
          ptx::mbar_wait(&pv_done[qi * NS + cur], ((c - NS) / NS) & 1);
          ptx::tc_fence_after();
        }
        float ls;
        if (PACK == 2 && (c != seg || lenw == 0)) {
          // the other sequence's keys (or an empty slot): P = 0, no exp, l unchanged
          const uint32_t z[8] = {0, 0, 0, 0, 0, 0, 0, 0};
          ptx::tmem_st_32x32b_x8(t_p, z);
          ptx::tmem_st_32x32b_x8(t_p + 8, z);
          ls = 0.f;
        } else if constexpr (Cfg::ALIAS) {
          // one TMEM read of the warp's 32 S values; max, exp and (rare) redo from registers;
          // P stored last, over the first 16 of these S columns
          // (S stays intact in TMEM until P is stored at the end, so the rare redo re-reads it:
          // va / vb are not live across the pair barrier, which keeps the kernel under the
          // 56-register budget of three 352-thread CTAs per SM)
          uint32_t va[16], vb[16], pk[16];
          auto load_s = [&]() {
            ptx::tmem_ld_32x32b_x16(t_chunk, va);
            ptx::tmem_ld_32x32b_x16(t_chunk + 16, vb);
            ptx::tmem_wait_ld();
          };
          auto reg_max = [&]() {
            float mx[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
            for (int e = 0; e < 16; ++e) {
              if (full || key0 + e < lenw) mx[e & 3] = fmaxf(mx[e & 3], __uint_as_float(va[e]));
              if (full || key0 + 16 + e < lenw) mx[e & 3] = fmaxf(mx[e & 3], __uint_as_float(vb[e]));
            }
            return fmaxf(fmaxf(mx[0], mx[1]), fmaxf(mx[2], mx[3]));
          };
          auto reg_exp = [&](float mc) {
            float2 acc = make_float2(0.f, 0.f);
#pragma unroll
            for (int e = 0; e < 32; e += 2) {
              const uint32_t* v = e < 16 ? va : vb;
              const int ee = e & 15;
              const float2 x = __ffma2_rn(make_float2(__uint_as_float(v[ee]), __uint_as_float(v[ee + 1])),
                                          make_float2(c2, c2), make_float2(-mc, -mc));
              float p0, p1;
              if (ee >= 16 - 2 * kPolyPairs) {  // same key positions as exp_piece
                const float2 pp = ex2_poly2(x);
                p0 = pp.x;
                p1 = pp.y;
              } else {
                p0 = ex2_approx(x.x);
                p1 = ex2_approx(x.y);
              }
              if (!full) {
                if (key0 + e >= lenw) p0 = 0.f;
                if (key0 + e + 1 >= lenw) p1 = 0.f;
              }
              acc = __fadd2_rn(acc, make_float2(p0, p1));
              pk[e >> 1] = pack_bf16x2(p0, p1);
            }
            return acc.x + acc.y;
          };
          load_s();
          if (c == seg) {
            xs[par * AQ + r] = reg_max();
            pair_sync();
            m = fmaxf(xch[qi][0][par * AQ + r], xch[qi][1][par * AQ + r]);
            ls = reg_exp(m * c2);
          } else {
            ls = reg_exp(m * c2);
            xs[par * AQ + r] = ls;
            pair_sync();
            const bool need = ls > 256.0f || xp[par * AQ + r] > 256.0f;  // same in both warps
            if (__any_sync(0xffffffffu, need)) {
              load_s();
              xmax[qi][hf][r] = reg_max();
              pair_sync();
              const float cmax = fmaxf(m, fmaxf(xmax[qi][0][r], xmax[qi][1][r]));
              float alpha = 1.f;
              if (need) {
                alpha = ex2_approx((m - cmax) * c2);
                l *= alpha;
                m = cmax;
              }
              // O holds PV_0..c-1 (complete: S(c) was issued after PV(c-1) finished); rescaled
              // 16 columns at a time, then S re-read (register budget)
#pragma unroll
              for (int h2 = 0; h2 < 2; ++h2) {
                uint32_t ov[16];
                ptx::tmem_ld_32x32b_x16(t_o + 16 * h2, ov);
                ptx::tmem_wait_ld();
#pragma unroll
                for (int e = 0; e < 16; ++e) ov[e] = __float_as_uint(__uint_as_float(ov[e]) * alpha);
                ptx::tmem_st_32x32b_x16(t_o + 16 * h2, ov);
              }
              ptx::tmem_wait_st();
              load_s();
              ls = reg_exp(m * c2);
            }
          }
          ptx::tmem_st_32x32b_x8(t_chunk, *reinterpret_cast<uint32_t(*)[8]>(&pk[0]));
          ptx::tmem_st_32x32b_x8(t_chunk + 8, *reinterpret_cast<uint32_t(*)[8]>(&pk[8]));
        } else {
#if defined(ARLO_ATTN_C0_TWOPASS)  // A/B only: the previous max pass + exp pass over S
          if (c == seg) {
            xs[par * AQ + r] = half_max(full, t_chunk, key0);
            pair_sync();
            m = fmaxf(xch[qi][0][par * AQ + r], xch[qi][1][par * AQ + r]);
            ls = exp_any(full, t_chunk, m * c2, key0, t_p);
          } else
#endif
          if (c == seg) {
            // first chunk: row max shared by the pair, then exp, from ONE TMEM read of S
            // (values kept in registers across the pair barrier; bitwise the two-pass result)
            uint32_t va[16], vb[16];
            ptx::tmem_ld_32x32b_x16(t_chunk, va);
            ptx::tmem_ld_32x32b_x16(t_chunk + 16, vb);
            ptx::tmem_wait_ld();
            float mx[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
            for (int e = 0; e < 16; ++e) {
              if (full || key0 + e < lenw) mx[e & 3] = fmaxf(mx[e & 3], __uint_as_float(va[e]));
              if (full || key0 + 16 + e < lenw) mx[e & 3] = fmaxf(mx[e & 3], __uint_as_float(vb[e]));
            }
            xs[par * AQ + r] = fmaxf(fmaxf(mx[0], mx[1]), fmaxf(mx[2], mx[3]));
            pair_sync();
            m = fmaxf(xch[qi][0][par * AQ + r], xch[qi][1][par * AQ + r]);
            float l2[2] = {0.f, 0.f};
            if (full) {
              exp_piece(std::false_type{}, va, key0, m * c2, t_p, l2);
              exp_piece(std::false_type{}, vb, key0 + 16, m * c2, t_p + 8, l2);
            } else {
              exp_piece(std::true_type{}, va, key0, m * c2, t_p, l2);
              exp_piece(std::true_type{}, vb, key0 + 16, m * c2, t_p + 8, l2);
            }
            ls = l2[0] + l2[1];
          } else {
            // single streaming pass against the (possibly stale) running max.  A row
            // whose p sum passes 2^8 in either half (necessary if any p > 2^8;
            // impossible while every p <= 4) is redone by both halves against the
            // new row max, O and l rescaled.
            ls = exp_any(full, t_chunk, m * c2, key0, t_p);
            xs[par * AQ + r] = ls;
            pair_sync();
            const bool need = ls > 256.0f || xp[par * AQ + r] > 256.0f;  // same in both warps
            if (__any_sync(0xffffffffu, need)) {
              xmax[qi][hf][r] = half_max(full, t_chunk, key0);
              pair_sync();
              const float cmax = fmaxf(m, fmaxf(xmax[qi][0][r], xmax[qi][1][r]));
              float alpha = 1.f;
              if (need) {
                alpha = ex2_approx((m - cmax) * c2);
                l *= alpha;
                m = cmax;
              }
              // O holds PV_0..c-1 (warp-collective TMEM traffic: every row takes part)
              ptx::mbar_wait(&pv_done[qi * NS + ((c - 1) % NS)], ((c - 1) / NS) & 1);
              ptx::tc_fence_after();
              uint32_t ov[32];
              ptx::tmem_ld_32x32b_x32(t_o, ov);
              ptx::tmem_wait_ld();
#pragma unroll
              for (int e = 0; e < 32; ++e) ov[e] = __float_as_uint(__uint_as_float(ov[e]) * alpha);
              ptx::tmem_st_32x32b_x16(t_o, *reinterpret_cast<uint32_t(*)[16]>(&ov[0]));
              ptx::tmem_st_32x32b_x16(t_o + 16, *reinterpret_cast<uint32_t(*)[16]>(&ov[16]));
              ptx::tmem_wait_st();
              ls = exp_any(full, t_chunk, m * c2, key0, t_p);
            }
          }
        }
        if (warp == 0 && lane == 0) atrace<TRACE>(4 + 3 * (c & 7));
        l += ls;
        // S slot back to the MMA warp, P chunk (TMEM stores complete) to the PV MMA
        ptx::tmem_wait_st();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          ptx::mbar_arrive(&s_free[qi * NS + cur]);
          ptx::mbar_arrive(&p_full[qi * NS + cur]);
        }
        if (warp == 0 && lane == 0) atrace<TRACE>(5 + 3 * (c & 7));
      }
      // l = l_half0 + l_half1 (fixed order); O = (sum_c P_c V_c) / l
      xmax[qi][hf][r] = l;  // (every redo's reads of xmax finished before the last chunk's barrier)
      pair_sync();
      const float inv = 1.f / (xmax[qi][0][r] + xmax[qi][1][r]);
      ptx::mbar_wait(&pv_done[qi * NS + ((n_ch - 1) % NS)], ((n_ch - 1) / NS) & 1);
      ptx::tc_fence_after();
      uint4* orow = reinterpret_cast<uint4*>(o + (size_t)(row_base + qrow) * H + h * D) + hf * 4;
      uint32_t ov[32];
      ptx::tmem_ld_32x32b_x32(t_o, ov);
      ptx::tmem_wait_ld();
      if (row_live && PACK == 2 && lenw == 0) {
#pragma unroll
        for (int i = 0; i < 4; ++i) orow[i] = make_uint4(0, 0, 0, 0);
      } else if (row_live) {
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          uint4 u;
          u.x = pack_bf16x2(__uint_as_float(ov[8 * i + 0]) * inv, __uint_as_float(ov[8 * i + 1]) * inv);
          u.y = pack_bf16x2(__uint_as_float(ov[8 * i + 2]) * inv, __uint_as_float(ov[8 * i + 3]) * inv);
          u.z = pack_bf16x2(__uint_as_float(ov[8 * i + 4]) * inv, __uint_as_float(ov[8 * i + 5]) * inv);
          u.w = pack_bf16x2(__uint_as_float(ov[8 * i + 6]) * inv, __uint_as_float(ov[8 * i + 7]) * inv);
          orow[i] = u;
        }
      }
    } else if (row_live) {
      // q-tile wholly padded: zero rows (each half writes its 32 columns)
      uint4* orow = reinterpret_cast<uint4*>(o + (size_t)(row_base + qrow) * H + h * D) + hf * 4;
#pragma unroll
      for (int i = 0; i < 4; ++i) orow[i] = make_uint4(0, 0, 0, 0);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) atrace<TRACE>(1);
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
  const int len = min(max(__ldg(lengths + b), 0), L);
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

static bool g_attn_trace_on = false;

int set_attn_trace(unsigned long long* buf) {
  g_attn_trace_on = buf != nullptr;
  return (int)cudaMemcpyToSymbol(g_atrace, &buf, sizeof(buf));
}

template <int NQ, int MAXKT, int NS, int PACK = 1>
cudaError_t attn_launch_cfg(const AttnPlan& p, const int32_t* lengths, void* o, cudaStream_t s) {
  using Cfg = AttnCfg<NQ, MAXKT, NS>;
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t e = once_per_device(attr_done, [] {
    cudaError_t r = cudaFuncSetAttribute(attn_tc_kernel<NQ, MAXKT, NS, false, PACK>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::kSmem);
    if (r == cudaSuccess)
      r = cudaFuncSetAttribute(attn_tc_kernel<NQ, MAXKT, NS, true, PACK>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               Cfg::kSmem);
    return r; });
  if (e != cudaSuccess) return e;
  dim3 grid((p.q_rows + NQ * AQ - 1) / (NQ * AQ), p.heads, (p.B + PACK - 1) / PACK);
  if (g_attn_trace_on)
    return launch_k(attn_tc_kernel<NQ, MAXKT, NS, true, PACK>, grid, dim3(Cfg::kThreads), Cfg::kSmem, s, p.tm, p.B,
                    p.L, p.heads, lengths, (bf16*)o);
  return launch_k(attn_tc_kernel<NQ, MAXKT, NS, false, PACK>, grid, dim3(Cfg::kThreads), Cfg::kSmem, s, p.tm, p.B,
                  p.L, p.heads, lengths, (bf16*)o);
}

bool attn_plan(AttnPlan* p, DType dt, int B, int L, int heads, const void* qkv, int q_rows) {
  p->B = B; p->L = L; p->heads = heads; p->dt = dt; p->qkv = qkv;
  p->q_rows = q_rows > 0 && q_rows < L ? q_rows : L;
  if (dt != DT_BF16 && p->q_rows != L) return false;  // fp32 check mode always computes every row
  if (dt != DT_BF16) return true;
  if (L > AK * 4) return false;
  return encode_tmap_bf16_2d(&p->tm, qkv, (uint64_t)3 * heads * D, (uint64_t)B * L, 64, 128, 128);
}

cudaError_t attn_launch(const AttnPlan& p, const int32_t* lengths, void* o, cudaStream_t s) {
  if (p.B <= 0 || p.L <= 0) return cudaSuccess;
  if (p.dt == DT_BF16) {
    // one 128-query tile per CTA, two CTAs per SM (TMEM 256 columns, ~83 KB smem
    // each): one CTA's prologue/epilogue overlaps the other's exp stream
#if defined(ARLO_ATTN_L128_ALIAS)
    // A/B only: P aliased over S (128 TMEM columns), three CTAs per SM.  Correct (tests green)
    // but not faster: at b = 32, 12 heads the 384 CTAs run in one wave (span 8.5 vs 9.5 us in
    // isolation), yet each CTA serialises S(c+1) behind PV(c) and three CTAs share the MUFU /
    // TMEM-read budget: 10.6 vs 10.1 us graph-replayed (round-1 A/B, raw log not kept)
    if (p.L <= 128) return attn_launch_cfg<1, 1, 1>(p, lengths, o, s);
#else
#if !defined(ARLO_ATTN_NO_PACK)
    if (p.L == 64) return attn_launch_cfg<1, 1, 2, 2>(p, lengths, o, s);  // two sequences per 128-row tile
#endif
    if (p.L <= 128) return attn_launch_cfg<1, 1, 2>(p, lengths, o, s);
#endif
    if (p.L <= 256) return attn_launch_cfg<1, 2, 2>(p, lengths, o, s);
    return attn_launch_cfg<1, 4, 2>(p, lengths, o, s);
  } else {
    const long warps = (long)p.B * p.L * p.heads;
    attn_f32_kernel<<<(unsigned)((warps + 3) / 4), 128, 0, s>>>(p.B, p.L, p.heads, (const float*)p.qkv, lengths,
                                                                 (float*)o);
  }
  return cudaGetLastError();
}

}  // namespace arlo
