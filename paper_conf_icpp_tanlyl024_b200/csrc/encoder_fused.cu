// encoder_fused.cu — the whole forward of a small (batch-1) runtime as ONE persistent kernel
// (SURVEY.md §8(f) NEXT-4 "persistent small-b·L megakernel"; steps a1-a9 of §8(a)).
//
// The paper's runtimes serve one request at a time ("we set the batch size for all runtimes
// to 1", §5).  At T = b·L <= 256 tokens a BERT forward is a chain of 7·layers
// dependent steps, each too small to fill a B200: as separate kernels (the tile and split-K
// families) every step costs a launch + prologue + drain, ~4.5 us each, whatever its GEMM
// does (BERT-base b=1 L=64: 87 kernels, 0.39 ms for 171 MB of weights, ~7 % of the HBM
// roofline).  Here one grid of one CTA per SM runs the whole forward as a static task graph:
//
//   embed rows -> per layer: QKV units -> attention (sequence, head) -> out-proj units ->
//   LN1 rows -> FFN1 units -> FFN2 units -> LN2 rows -> ... -> pooler groups -> classifier
//
// * Tasks are assigned to CTAs round-robin in topological order (host, fused_plan); a CTA runs
//   its list in order.  A task waits for the COUNT of finished tasks of the step it consumes
//   (one counter per (layer, step), release-add by the producer task, acquire-poll by the
//   consumer), never for a grid barrier.  Deadlock-free: the earliest unfinished task in the
//   global order has every dependency finished and is at the head of its CTA's list.
// * GEMM units are swap-AB tcgen05 MMAs: D[128 weight rows, T tokens] (M = 128, N = T, K = 16)
//   with the weight tile as the A operand and the activation tile as B, accumulated in TMEM
//   (two accumulators, so the MMA of a CTA's next unit overlaps this unit's epilogue).  At
//   T <= 256 tokens this puts the 128-row MMA dimension on the weights (full tensor rate at
//   N = 64) instead of padding the tokens to 128 rows.
// * Warp roles: warps 0-3 compute (GEMM epilogues from TMEM lane quarters, attention,
//   LayerNorm rows, embedding, head), warp 4 TMA producer, warp 5 MMA issuer.  The producer
//   walks the CTA's GEMM units ahead of the compute warps: it loads each unit's WEIGHT k-blocks
//   into the smem ring as soon as a stage is free and prefetches the next unit's whole weight
//   slice into L2 — weights never depend on activations — and issues the activation k-blocks
//   only when the unit's dependency count is reached.  The weight stream of the whole forward
//   thus runs ahead of the dependency chain instead of inside it.
// * Split-K units (out-proj, FFN2) write fp32 partials; the LayerNorm row task that consumes
//   them adds the partials in the fixed order s = 0, 1, ..., then bias, then the residual
//   (the tile family's epilogue order), rounds to bf16 and normalises (layernorm.cuh).
//   Split factors depend on the weight shape (N, K) only and every other step is per token
//   or per (sequence, head), so a request's logits are bitwise the same on every fused
//   runtime L >= its length and in every batch bucket (tests/test_gpu_fused.py).
// * Attention (L <= 128) runs per (sequence, head) on mma.sync m16n8k16 (warp = 16 queries,
//   64-key chunks, online softmax in exp2, P rounded to bf16 for the PV product as in the
//   tcgen05 attention kernel): a 128-row tcgen05 tile would be mostly padding here.
//   Key chunks past len are skipped, keys >= len masked, query blocks past len zero-filled.
//
// Every activation written inside the kernel is read back with L2-only loads (ld.global.cg)
// or TMA: L1 is not coherent across SMs, and the buffers are reused layer after layer.
#include <cuda.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "common.cuh"
#include "epilogue.cuh"
#include "kernels.h"
#include "layernorm.cuh"
#include "ptx.cuh"

namespace arlo {
namespace {

constexpr int kThreads = 192;   // warps 0-3 compute, 4 producer, 5 MMA
constexpr int kCompute = 128;
constexpr int kProdWarp = 4, kMmaWarp = 5;
constexpr int kRowsPerTask = 4;  // LayerNorm / embedding rows per task (one warp per row)
constexpr int kPoolFeat = 8;     // pooler features per task (2 per compute warp)
constexpr int kAttnRows = 128;   // L <= 128
constexpr int kLnStage = 12288;  // LayerNorm / embedding tasks: output rows staged past bias, gamma, beta (H <= 1024)
constexpr int kWBytes = 128 * 64 * 2;  // one weight k-block: 128 rows x 64 bf16, 128B swizzle
constexpr int kSmemOptIn = 232448;

enum : uint16_t { FT_EMBED = 0, FT_QKV, FT_ATTN, FT_OPROJ, FT_LN1, FT_FFN1, FT_FFN2, FT_LN2, FT_POOL, FT_CLS };
enum : int { CS_X = 0, CS_QKV, CS_ATTN, CS_O, CS_X1, CS_H, CS_F2, kStagesPerLayer = 8 };
enum : int { TM_X = 0, TM_CTX, TM_X1, TM_HB, TM_QKV, kAMaps = 5 };  // activation maps, then 4 weight maps per layer

struct FusedTask {
  uint16_t type, layer, a, b;
};

struct FusedLayer {
  const float *b_qkv, *b_o, *ln1_g, *ln1_b, *b_1, *b_2, *ln2_g, *ln2_b;
};

struct FusedArgs {
  int layers, H, heads, F, C, vocab, B, L, T;
  float eps;
  int s_o, s_f2;              // split factors: out-proj (K = H), FFN2 (K = F)
  int stages, stage_bytes;    // smem ring: stage = weight k-block (16 KB) + activation k-block (T x 128 B)
  int tcols;                  // TMEM columns per accumulator (>= T, power of two)
  int scratch_bytes;          // compute-warp shared scratch: attention Q/K/V/O, epilogue and row staging
  int n_rows, n_pool;         // row tasks (ceil(T / 4)), pooler tasks (ceil(H / 32))
  const CUtensorMap* tm;      // [kAMaps + 4 * layers]
  const FusedLayer* lw;
  const bf16 *word, *pos, *type;
  const float *emb_g, *emb_b;
  const bf16 *w_p, *w_c;
  const float *b_p, *b_c;
  const int32_t *ids, *lengths;
  int32_t* err;
  bf16 *X, *X1, *QKV, *CTX, *HB;
  float *P, *pooled, *logits;
  unsigned* cnt;              // [(layers + 1) * kStagesPerLayer + 1], zero between launches
  const int* task_off;        // [grid + 1]
  const FusedTask* tasks;
};

// Profiling hook (arlo_debug_fused_trace): 16 u64 per task index i of the task array:
// [type | layer << 8 | a << 24 | b << 40 | cta << 52, compute begin, ready (dependency met /
// accumulator full), end (after the completion signal), producer dependency met] in %globaltimer ns;
// slot 5 (task body done) and sub-stamps 6..14 in clock64 cycles, slot 15 = clock64 at begin
// (tools/fused_trace.py converts them with the CTA's measured clock rate).
__device__ unsigned long long* g_ftrace = nullptr;
constexpr int kTr = 16;  // trace slots per task
// sub-stamp k of task i by the calling thread (no-op unless tracing)
#define FT_SUB(i, k)                                              \
  do {                                                            \
    if (unsigned long long* tr_ = g_ftrace) tr_[(size_t)(i) * kTr + (k)] = clock64(); \
  } while (0)
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ bool is_gemm(uint16_t t) {
  return t == FT_QKV || t == FT_OPROJ || t == FT_FFN1 || t == FT_FFN2;
}

__device__ __forceinline__ void compute_sync() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

// Completion signal of a task.  Every task output leaves the SM as a bulk copy from shared
// memory (cp.async.bulk), which thread 0 waits to COMPLETE (bulk_wait<0>) before this relaxed
// add: the data is in L2 before the count moves.  Consumers poll with relaxed loads and read
// only through L2 (TMA, ld.global.cg), so neither side needs a gpu-scope fence.  (A release /
// acquire fence also waits for the SM's in-flight bulk weight prefetches: 0.62 -> 1.67 us per
// hop with a prefetch stream running, tools/signal_bench.cu; relaxed: 0.46 us.)
__device__ __forceinline__ void signal_done(unsigned* p, unsigned n = 1) {
  asm volatile("red.relaxed.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(n) : "memory");
}

__device__ __forceinline__ void wait_count(const unsigned* p, unsigned target) {
  unsigned v;
  do {
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  } while (v < target);
}

// L2-only loads (ld.global.cg) of data other CTAs wrote during this launch.  Ordinary
// (non-volatile) loads so the compiler can keep many in flight; they follow a compute_sync
// (whose asm carries a memory clobber) after the acquire that made the data visible.
__device__ __forceinline__ uint4 ldcg_v4(const void* p) { return __ldcg(reinterpret_cast<const uint4*>(p)); }
__device__ __forceinline__ float4 ldcg_f4(const float* p) { return __ldcg(reinterpret_cast<const float4*>(p)); }

// The counter a task waits for and its target count (nullptr: no dependency).
__device__ __forceinline__ const unsigned* task_dep(const FusedArgs& a, const FusedTask& t, unsigned& target) {
  const unsigned* c = a.cnt + t.layer * kStagesPerLayer;
  switch (t.type) {
    case FT_QKV: target = a.T; return c + CS_X;
    case FT_ATTN: target = 3 * a.H / 128; return c + CS_QKV;
    case FT_OPROJ: target = a.B * a.heads; return c + CS_ATTN;
    case FT_LN1: target = (a.H / 128) * a.s_o; return c + CS_O;
    case FT_FFN1: target = a.n_rows; return c + CS_X1;
    case FT_FFN2: target = a.F / 128; return c + CS_H;
    case FT_LN2: target = (a.H / 128) * a.s_f2; return c + CS_F2;
    case FT_POOL: target = a.T; return a.cnt + a.layers * kStagesPerLayer + CS_X;
    case FT_CLS: target = a.n_pool; return a.cnt + a.layers * kStagesPerLayer + 1;
  }
  return nullptr;
}

// The counter a finished task increments.
__device__ __forceinline__ unsigned* task_done(const FusedArgs& a, const FusedTask& t) {
  unsigned* c = a.cnt + t.layer * kStagesPerLayer;
  switch (t.type) {
    case FT_EMBED: return a.cnt + CS_X;
    case FT_QKV: return c + CS_QKV;
    case FT_ATTN: return c + CS_ATTN;
    case FT_OPROJ: return c + CS_O;
    case FT_LN1: return c + CS_X1;
    case FT_FFN1: return c + CS_H;
    case FT_FFN2: return c + CS_F2;
    case FT_LN2: return c + kStagesPerLayer + CS_X;
    case FT_POOL: return a.cnt + a.layers * kStagesPerLayer + 1;
  }
  return nullptr;
}

// Compute warps: thread 0 waits for the task's dependency, then the four warps sync (every
// non-GEMM task preloads its constants, then calls this, then runs).
__device__ __forceinline__ void dep_wait(const FusedArgs& a, const FusedTask& t, unsigned long long* stamp = nullptr) {
  unsigned target = 0;
  const unsigned* dep = task_dep(a, t, target);
  if (threadIdx.x == 0) {
    if (dep) wait_count(dep, target);
    if (stamp) *stamp = gtimer();
  }
  compute_sync();
}

// Small weights (biases, LayerNorm gamma / beta, position rows, the pooler) are read once per
// forward, each on the critical path of a task: at kernel start every CTA issues bulk L2
// prefetches for its share of them, so those reads hit L2 instead of HBM.
__device__ void prefetch_small(const FusedArgs& a) {
  int item = 0;
  const int me = blockIdx.x, n = gridDim.x;
  auto pf = [&](const void* ptr, uint32_t bytes) {
    if (item++ % n == me && ptr && bytes >= 16)
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(ptr), "r"(bytes & ~15u) : "memory");
  };
  const uint32_t H4 = a.H * 4;
  for (int l = 0; l < a.layers; ++l) {
    const FusedLayer& w = a.lw[l];
    pf(w.b_qkv, 3 * H4); pf(w.b_o, H4); pf(w.ln1_g, H4); pf(w.ln1_b, H4);
    pf(w.b_1, a.F * 4); pf(w.b_2, H4); pf(w.ln2_g, H4); pf(w.ln2_b, H4);
  }
  pf(a.emb_g, H4); pf(a.emb_b, H4); pf(a.type, a.H * 2); pf(a.b_p, H4);
  pf(a.pos, (uint32_t)a.L * a.H * 2);
  pf(a.w_c, (uint32_t)a.C * a.H * 2);
  const size_t wp = (size_t)a.H * a.H * 2;
  for (size_t o = 0; o < wp; o += 16384) pf(reinterpret_cast<const char*>(a.w_p) + o, (uint32_t)(wp - o < 16384 ? wp - o : 16384));
}

struct Gemm {
  int wmap, amap, n0, k0, nkb;
};
__device__ __forceinline__ Gemm gemm_of(const FusedArgs& a, const FusedTask& t) {
  const int wbase = kAMaps + 4 * t.layer;
  switch (t.type) {
    case FT_QKV: return {wbase + 0, TM_X, t.a * 128, 0, a.H / 64};
    case FT_OPROJ: return {wbase + 1, TM_CTX, t.a * 128, t.b * (a.H / a.s_o), a.H / a.s_o / 64};
    case FT_FFN1: return {wbase + 2, TM_X1, t.a * 128, 0, a.H / 64};
    default: return {wbase + 3, TM_HB, t.a * 128, t.b * (a.F / a.s_f2), a.F / a.s_f2 / 64};
  }
}

__device__ __forceinline__ void ring_adv(int& st, uint32_t& ph, int stages) {
  if (++st == stages) {
    st = 0;
    ph ^= 1;
  }
}

// Activation k-block [T x 64] at column k: x / x1 are row-major [T, H] (2-D maps); the context
// is head-major [H/64][T][64] (3-D map: column k = head k/64); the FFN1 output is tile-contiguous
// [F/128][T][128] (3-D map: column k = tile k/128, offset k%128).
__device__ __forceinline__ void load_a(uint8_t* dst, const CUtensorMap* ta, int amap, uint64_t* bar, int k) {
  if (amap == TM_HB)
    ptx::tma_load_3d(dst, ta, bar, k & 127, 0, k >> 7);
  else if (amap == TM_CTX)
    ptx::tma_load_3d(dst, ta, bar, 0, 0, k >> 6);
  else
    ptx::tma_load_2d(dst, ta, bar, k, 0);
}

// Thread 0: copy `bytes` of staged output from shared memory to global (after every compute
// thread's fence.proxy.async.shared::cta + compute_sync), committed; the main loop waits for it.
__device__ __forceinline__ void stage_out(void* gdst, const void* ssrc, uint32_t bytes) {
  ptx::bulk_store(gdst, ssrc, bytes);
  ptx::bulk_commit();
}

// ------------------------------------------------------------------ producer (warp 4, lane 0)
__device__ void producer(const FusedArgs& a, uint8_t* ring, uint64_t* full, uint64_t* empty, int t0, int t1) {
  const int stages = a.stages;
  const uint32_t a_bytes = (uint32_t)a.T * 128;
  const uint32_t stage_tx = kWBytes + a_bytes;
  int st = 0;
  uint32_t ph = 0;
  for (int i = t0; i < t1; ++i) {
    const FusedTask t = a.tasks[i];
    if (!is_gemm(t.type)) continue;
    const Gemm g = gemm_of(a, t);
    const CUtensorMap* tw = a.tm + g.wmap;
    const CUtensorMap* ta = a.tm + g.amap;
    const int npre = g.nkb < stages ? g.nkb : stages;
    int s2 = st;
    uint32_t p2 = ph;
    for (int kb = 0; kb < npre; ++kb) {  // weights first, as far as the ring allows
      ptx::mbar_wait(&empty[s2], p2 ^ 1);
      ptx::mbar_arrive_expect_tx(&full[s2], stage_tx);
      ptx::tma_load_2d(ring + (size_t)s2 * a.stage_bytes, tw, &full[s2], g.k0 + kb * 64, g.n0);
      ring_adv(s2, p2, stages);
    }
    unsigned target = 0;
    const unsigned* dep = task_dep(a, t, target);
    wait_count(dep, target);
    if (unsigned long long* tr = g_ftrace) tr[(size_t)i * kTr + 4] = gtimer();
    for (int kb = 0; kb < npre; ++kb) {
      load_a(ring + (size_t)st * a.stage_bytes + kWBytes, ta, g.amap, &full[st], g.k0 + kb * 64);
      ring_adv(st, ph, stages);
    }
    FT_SUB(i, 12);
    for (int kb = npre; kb < g.nkb; ++kb) {
      ptx::mbar_wait(&empty[st], ph ^ 1);
      ptx::mbar_arrive_expect_tx(&full[st], stage_tx);
      uint8_t* base = ring + (size_t)st * a.stage_bytes;
      ptx::tma_load_2d(base, tw, &full[st], g.k0 + kb * 64, g.n0);
      load_a(base + kWBytes, ta, g.amap, &full[st], g.k0 + kb * 64);
      ring_adv(st, ph, stages);
    }
    // the next unit's weight slice into L2 (weights never depend on activations); issued after
    // this unit's loads so that it does not queue ahead of them in the TMA unit
    for (int j = i + 1; j < t1; ++j) {
      const FusedTask u = a.tasks[j];
      if (!is_gemm(u.type)) continue;
      const Gemm h = gemm_of(a, u);
      for (int kb = 0; kb < h.nkb; ++kb) ptx::tma_prefetch_l2_2d(a.tm + h.wmap, h.k0 + kb * 64, h.n0);
      break;
    }
  }
}

// ------------------------------------------------------------------ MMA issuer (warp 5)
__device__ void mma_issuer(const FusedArgs& a, uint8_t* ring, uint64_t* full, uint64_t* empty, uint64_t* tfull,
                           uint64_t* tempty, uint32_t tmem, int t0, int t1) {
  const int stages = a.stages;
  const uint32_t idesc = ptx::idesc_bf16_f32(128, a.T);
  int st = 0;
  uint32_t ph = 0;
  int acc = 0;
  uint32_t aph = 0;
  for (int i = t0; i < t1; ++i) {
    const FusedTask t = a.tasks[i];
    if (!is_gemm(t.type)) continue;
    const Gemm g = gemm_of(a, t);
    ptx::mbar_wait(&tempty[acc], aph ^ 1);
    ptx::tc_fence_after();
    const uint32_t d = tmem + (uint32_t)(acc * a.tcols);
    for (int kb = 0; kb < g.nkb; ++kb) {
      ptx::mbar_wait(&full[st], ph);
      if (kb == 0 && threadIdx.x == kMmaWarp * 32) FT_SUB(i, 13);
      ptx::tc_fence_after();
      const uint32_t w_addr = ptx::smem_u32(ring + (size_t)st * a.stage_bytes);
      const uint32_t x_addr = w_addr + kWBytes;
#pragma unroll
      for (int k = 0; k < 4; ++k)
        ptx::mma_bf16_ss_w(d, ptx::desc_k_sw128(w_addr + k * 32), ptx::desc_k_sw128(x_addr + k * 32), idesc,
                           (kb | k) != 0);
      ptx::mma_commit_w(&empty[st]);
      ring_adv(st, ph, stages);
    }
    ptx::mma_commit_w(&tfull[acc]);
    if (threadIdx.x == kMmaWarp * 32) FT_SUB(i, 14);
    if (++acc == 2) {
      acc = 0;
      aph ^= 1;
    }
  }
}

// ------------------------------------------------------------------ compute tasks (warps 0-3)
// GEMM epilogue: thread (warp w, lane i) owns TMEM lane 32w + i = output column n0 + 32w + i
// and reads the unit's T token columns 16 at a time into a token-major [64][128] shared tile
// (one 64-token chunk at a time), which thread 0 writes out with ONE bulk copy: every GEMM
// output is tile-contiguous in global memory ([N/128][T][128]: QKV, FFN1 activations; partials
// [S][H/128][T][128]).  A signal after per-thread stores waited for ~16-32 KB of stores to drain
// (~1.1-1.5 us per hop, tools/signal_bench.cu); the bulk copy is waited for once by thread 0.
__device__ void gemm_epilogue(const FusedArgs& a, const FusedTask& t, uint32_t tacc, uint8_t* scratch, float bias,
                              int ti) {
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int n = warp * 32 + lane;
  const uint32_t taddr = tacc + ((uint32_t)(warp * 32) << 16);
  const int T = a.T;
  const bool partial = t.type == FT_OPROJ || t.type == FT_FFN2;
  const bool gelu = t.type == FT_FFN1;
  uint8_t* tile;  // this unit's [T][128] output tile
  if (partial)
    tile = reinterpret_cast<uint8_t*>(a.P + ((size_t)t.b * (a.H / 128) + t.a) * T * 128);
  else
    tile = reinterpret_cast<uint8_t*>((gelu ? a.HB : a.QKV) + (size_t)t.a * T * 128);
  const int esz = partial ? 4 : 2;
  for (int c0 = 0; c0 < T; c0 += 64) {
    const int nt = T - c0 < 64 ? T - c0 : 64;
    if (c0 > 0 && tid == 0) ptx::bulk_wait_read<0>();  // the previous chunk has left the staging tile
    if (c0 > 0) compute_sync();
    for (int t0 = 0; t0 < nt; t0 += 16) {
      uint32_t r[16];
      ptx::tmem_ld_32x32b_x16(taddr + c0 + t0, r);
      ptx::tmem_wait_ld();
      if (partial) {
        float* st = reinterpret_cast<float*>(scratch);
#pragma unroll
        for (int j = 0; j < 16; ++j) st[(t0 + j) * 128 + n] = __uint_as_float(r[j]);
      } else {
        bf16* st = reinterpret_cast<bf16*>(scratch);
#pragma unroll
        for (int j = 0; j < 16; j += 2) {
          // the tile kernels' epilogue arithmetic (epilogue.cuh): acc + bias, then GELU, RNE to bf16
          float2 x = __fadd2_rn(make_float2(__uint_as_float(r[j]), __uint_as_float(r[j + 1])), f2(bias));
          if (gelu) x = gelu2_erf_fast(x);
          st[(t0 + j) * 128 + n] = __float2bfloat16_rn(x.x);
          st[(t0 + j + 1) * 128 + n] = __float2bfloat16_rn(x.y);
        }
      }
    }
    if (tid == 0 && c0 == 0) FT_SUB(ti, 6);
    ptx::fence_proxy_async_smem();  // generic smem writes -> the bulk copy (async proxy)
    compute_sync();
    if (tid == 0 && c0 == 0) FT_SUB(ti, 7);
    if (tid == 0) {
      ptx::bulk_store(tile + (size_t)c0 * 128 * esz, scratch, (uint32_t)(nt * 128 * esz));
      ptx::bulk_commit();
    }
  }
  if (tid == 0) ptx::bulk_wait_read<0>();  // the staging tile is free for the next task (after the caller's sync)
  if (tid == 0) FT_SUB(ti, 8);
}

// Residual + LayerNorm row task (kRowsPerTask rows, one warp per row):
//   y = bf16(((P_0 + P_1 + ... + P_{S-1}) + bias) + resid), then LN(y) -> out
// (reading S3: biased variance, eps inside the root; layernorm.cuh's row arithmetic).  Bias,
// gamma and beta are staged in shared memory before the dependency wait; the output rows are
// staged and leave with one bulk copy.  (Tried: one row per task with the S partial rows
// bulk-loaded to shared memory: slower, ~70 ns per bulk request through the TMA unit.)
template <int MAXV>
__device__ void ln_rows(const FusedArgs& a, const FusedTask& t, uint8_t* scratch, unsigned long long* stamp, int ti) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int row = t.a * kRowsPerTask + warp;
  const FusedLayer& lw = a.lw[t.layer];
  const bool first = t.type == FT_LN1;
  float* sb = reinterpret_cast<float*>(scratch);
  float* sg = sb + a.H;
  float* sbe = sg + a.H;
  {
    const float* bias = first ? lw.b_o : lw.b_2;
    const float* g = first ? lw.ln1_g : lw.ln2_g;
    const float* be = first ? lw.ln1_b : lw.ln2_b;
    for (int i = threadIdx.x * 4; i < a.H; i += kCompute * 4) {
      *reinterpret_cast<float4*>(sb + i) = __ldg(reinterpret_cast<const float4*>(bias + i));
      *reinterpret_cast<float4*>(sg + i) = __ldg(reinterpret_cast<const float4*>(g + i));
      *reinterpret_cast<float4*>(sbe + i) = __ldg(reinterpret_cast<const float4*>(be + i));
    }
  }
  dep_wait(a, t, stamp);
  if (row < a.T) {
    const int S = first ? a.s_o : a.s_f2;
    const bf16* resid = (first ? a.X : a.X1) + (size_t)row * a.H;
    const int nvec = a.H / 8;
    const size_t pstride = (size_t)a.T * a.H;     // one split's partial: [H/128][T][128]
    const float* prow = a.P + (size_t)row * 128;  // column c at prow + (c/128) T 128 + c%128
    float4 s0[MAXV], s1[MAXV];
    uint4 ru[MAXV];
#pragma unroll
    for (int i = 0; i < MAXV; ++i) {  // partial 0 and the residual: all loads in flight at once
      const int c0 = (lane + 32 * i) * 8;
      const int pc = (c0 >> 7) * a.T * 128 + (c0 & 127);
      if (lane + 32 * i < nvec) {
        s0[i] = ldcg_f4(prow + pc);
        s1[i] = ldcg_f4(prow + pc + 4);
        ru[i] = ldcg_v4(resid + c0);
      }
    }
    for (int s = 1; s < S; ++s) {  // partials added in the fixed order s = 1, 2, ...
      float4 q0[MAXV], q1[MAXV];
#pragma unroll
      for (int i = 0; i < MAXV; ++i) {
        const int c0 = (lane + 32 * i) * 8;
        const int pc = (c0 >> 7) * a.T * 128 + (c0 & 127);
        if (lane + 32 * i < nvec) {
          q0[i] = ldcg_f4(prow + s * pstride + pc);
          q1[i] = ldcg_f4(prow + s * pstride + pc + 4);
        }
      }
#pragma unroll
      for (int i = 0; i < MAXV; ++i) {
        if (lane + 32 * i < nvec) {
          s0[i].x += q0[i].x; s0[i].y += q0[i].y; s0[i].z += q0[i].z; s0[i].w += q0[i].w;
          s1[i].x += q1[i].x; s1[i].y += q1[i].y; s1[i].z += q1[i].z; s1[i].w += q1[i].w;
        }
      }
    }
    if (threadIdx.x == 0) FT_SUB(ti, 6);
    float v[MAXV][8];
#pragma unroll
    for (int i = 0; i < MAXV; ++i) {
      if (lane + 32 * i < nvec) {
        const float2 r0 = unpack_bf16x2(ru[i].x), r1 = unpack_bf16x2(ru[i].y), r2 = unpack_bf16x2(ru[i].z),
                     r3 = unpack_bf16x2(ru[i].w);
        const float acc[8] = {s0[i].x, s0[i].y, s0[i].z, s0[i].w, s1[i].x, s1[i].y, s1[i].z, s1[i].w};
        const int c0 = (lane + 32 * i) * 8;
        const float4 b0 = *reinterpret_cast<const float4*>(sb + c0);
        const float4 b1 = *reinterpret_cast<const float4*>(sb + c0 + 4);
        const float bb[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
        const float rr[8] = {r0.x, r0.y, r1.x, r1.y, r2.x, r2.y, r3.x, r3.y};
#pragma unroll
        for (int j = 0; j < 8; ++j)  // the tile kernels' epilogue order (acc + bias) + residual, RNE
          v[i][j] = __bfloat162float(__float2bfloat16_rn(__fadd_rn(__fadd_rn(acc[j], bb[j]), rr[j])));
      }
    }
    ln_finish<bf16, MAXV>(v, nvec, a.H, lane, sg, sbe, a.eps, reinterpret_cast<bf16*>(scratch + kLnStage) + warp * a.H);
    if (threadIdx.x == 0) FT_SUB(ti, 7);
  }
  ptx::fence_proxy_async_smem();
  compute_sync();
  if (threadIdx.x == 0) {  // the task's rows are contiguous in x / x1
    const int r0 = t.a * kRowsPerTask, nr = a.T - r0 < kRowsPerTask ? a.T - r0 : kRowsPerTask;
    stage_out((first ? a.X1 : a.X) + (size_t)r0 * a.H, scratch + kLnStage, (uint32_t)(nr * a.H * 2));
  }
}

// Embedding gather + LayerNorm rows (embed_ln.cu's arithmetic; pad positions t >= len use id 0).
template <int MAXV>
__device__ void embed_rows(const FusedArgs& a, const FusedTask& t, uint8_t* scratch) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int row = t.a * kRowsPerTask + warp;
  const bool live = row < a.T;
  const int nvec = a.H / 8;
  float* sg = reinterpret_cast<float*>(scratch);
  float* sbe = sg + a.H;
  for (int i = threadIdx.x * 4; i < a.H; i += kCompute * 4) {  // gamma / beta -> shared memory
    *reinterpret_cast<float4*>(sg + i) = __ldg(reinterpret_cast<const float4*>(a.emb_g + i));
    *reinterpret_cast<float4*>(sbe + i) = __ldg(reinterpret_cast<const float4*>(a.emb_b + i));
  }
  float v[MAXV][8];
  if (live) {
    const int bi = row / a.L, pos = row - bi * a.L;
    int id = 0;
    if (pos < __ldg(a.lengths + bi)) {
      id = __ldg(a.ids + row);
      if (id < 0 || id >= a.vocab) {
        if (lane == 0 && a.err) *a.err = 1;
        id = 0;
      }
    }
    const bf16* wr = a.word + (size_t)id * a.H;
    const bf16* pr = a.pos + (size_t)pos * a.H;
#pragma unroll
    for (int i = 0; i < MAXV; ++i) {
      const int vi = lane + 32 * i;
      if (vi < nvec) {
        float x[8], p[8], c[8];
        Vec<bf16>::load(wr + vi * 8, x);
        Vec<bf16>::load(pr + vi * 8, p);
        Vec<bf16>::load(a.type + vi * 8, c);
#pragma unroll
        for (int j = 0; j < 8; ++j) v[i][j] = x[j] + p[j] + c[j];
      }
    }
  }
  compute_sync();
  if (live) ln_finish<bf16, MAXV>(v, nvec, a.H, lane, sg, sbe, a.eps, reinterpret_cast<bf16*>(scratch + kLnStage) + warp * a.H);
  ptx::fence_proxy_async_smem();
  compute_sync();
  if (threadIdx.x == 0) {
    const int r0 = t.a * kRowsPerTask, nr = a.T - r0 < kRowsPerTask ? a.T - r0 : kRowsPerTask;
    stage_out(a.X + (size_t)r0 * a.H, scratch + kLnStage, (uint32_t)(nr * a.H * 2));
  }
}

// Masked attention of one (sequence, head): o_t = softmax_j(q_t . k_j / 8, j < len) v_j.
// Warp w takes 16-query blocks w, w + 4, ...; keys in 64-key chunks with an online softmax.
// Q, K, V rows (128 B) sit in shared memory with their 16-byte chunks XOR-swizzled by row
// (conflict-free ldmatrix without padding); the output block [L][64] is staged unswizzled and
// leaves with one bulk copy into the head-major context [H/64][T][64].
__device__ __forceinline__ int swz(int r, int col) { return r * 64 + ((((col >> 3) ^ r) & 7) << 3) + (col & 7); }

__device__ void attention(const FusedArgs& a, const FusedTask& t, uint8_t* scratch, uint64_t* cbar, uint32_t& cph,
                          unsigned long long* stamp, int ti) {
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int L = a.L, H = a.H, b = t.a, h = t.b;
  const int len = min(max(__ldg(a.lengths + b), 0), L);
  const int nq = (len + 15) >> 4;   // live 16-query blocks
  const int nkc = (len + 63) >> 6;  // live 64-key chunks
  const int kvr = (L + 63) & ~63;   // K and V rows: the last 64-key chunk may pass L (zero rows)
  bf16* sQ = reinterpret_cast<bf16*>(scratch);
  bf16* sK = sQ + L * 64;
  bf16* sV = sK + kvr * 64;
  bf16* sO = sV + kvr * 64;
  const int T = a.T;
  dep_wait(a, t, stamp);
  // QKV is tile-contiguous [3H/128][T][128]: head h's q / k / v columns are 64-column halves of
  // tiles h/2, H/128 + h/2, 2H/128 + h/2; one TMA box each ({64, L} rows of the sequence), landing
  // with the 128-byte swizzle that swz() reads
  if (tid == 0) {
    const CUtensorMap* tq = a.tm + TM_QKV;
    ptx::mbar_arrive_expect_tx(cbar, (uint32_t)(3 * L * 128));
    ptx::tma_load_3d(sQ, tq, cbar, (h & 1) * 64, b * L, h >> 1);
    ptx::tma_load_3d(sK, tq, cbar, (h & 1) * 64, b * L, H / 128 + (h >> 1));
    ptx::tma_load_3d(sV, tq, cbar, (h & 1) * 64, b * L, 2 * (H / 128) + (h >> 1));
  }
  for (int idx = L * 8 + tid; idx < kvr * 8; idx += kCompute) {  // key rows L .. kvr-1: zero
    *reinterpret_cast<uint4*>(sK + idx * 8) = make_uint4(0, 0, 0, 0);
    *reinterpret_cast<uint4*>(sV + idx * 8) = make_uint4(0, 0, 0, 0);
  }
  // query rows past the live blocks: zero context
  for (int idx = nq * 16 * 8 + tid; idx < L * 8; idx += kCompute)
    *reinterpret_cast<uint4*>(sO + idx * 8) = make_uint4(0, 0, 0, 0);
  ptx::mbar_wait(cbar, cph);
  cph ^= 1;
  compute_sync();
  if (tid == 0) FT_SUB(ti, 6);
  const float sc = 0.125f * 1.4426950408889634f;  // 1/sqrt(64), in log2 units
  const int g = lane >> 2, c2 = (lane & 3) * 2;
  for (int qb = warp; qb < nq; qb += 4) {
    uint32_t qf[4][4];
#pragma unroll
    for (int ks = 0; ks < 4; ++ks)
      ptx::ldmatrix_x4(qf[ks], sQ + swz(qb * 16 + (lane & 15), ks * 16 + (lane >> 4) * 8));
    float o[8][4];
#pragma unroll
    for (int i = 0; i < 8; ++i) o[i][0] = o[i][1] = o[i][2] = o[i][3] = 0.f;
    float m0 = -INFINITY, m1 = -INFINITY, l0 = 0.f, l1 = 0.f;
    for (int kc = 0; kc < nkc; ++kc) {
      float s[8][4];
#pragma unroll
      for (int i = 0; i < 8; ++i) s[i][0] = s[i][1] = s[i][2] = s[i][3] = 0.f;
#pragma unroll
      for (int ks = 0; ks < 4; ++ks) {
#pragma unroll
        for (int np = 0; np < 4; ++np) {
          uint32_t kb[4];
          ptx::ldmatrix_x4(kb, sK + swz(kc * 64 + np * 16 + (lane & 7) + ((lane >> 4) << 3),
                                        ks * 16 + ((lane >> 3) & 1) * 8));
          ptx::mma_m16n8k16_bf16(s[2 * np], qf[ks], kb[0], kb[1]);
          ptx::mma_m16n8k16_bf16(s[2 * np + 1], qf[ks], kb[2], kb[3]);
        }
      }
      float mx0 = -INFINITY, mx1 = -INFINITY;
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        const int key = kc * 64 + nt * 8 + c2;
        s[nt][0] = key < len ? s[nt][0] * sc : -INFINITY;
        s[nt][1] = key + 1 < len ? s[nt][1] * sc : -INFINITY;
        s[nt][2] = key < len ? s[nt][2] * sc : -INFINITY;
        s[nt][3] = key + 1 < len ? s[nt][3] * sc : -INFINITY;
        mx0 = fmaxf(mx0, fmaxf(s[nt][0], s[nt][1]));
        mx1 = fmaxf(mx1, fmaxf(s[nt][2], s[nt][3]));
      }
      mx0 = fmaxf(mx0, __shfl_xor_sync(0xffffffffu, mx0, 1));
      mx0 = fmaxf(mx0, __shfl_xor_sync(0xffffffffu, mx0, 2));
      mx1 = fmaxf(mx1, __shfl_xor_sync(0xffffffffu, mx1, 1));
      mx1 = fmaxf(mx1, __shfl_xor_sync(0xffffffffu, mx1, 2));
      const float mn0 = fmaxf(m0, mx0), mn1 = fmaxf(m1, mx1);  // finite: key 0 is live in chunk 0
      const float f0 = ex2_approx(m0 - mn0), f1 = ex2_approx(m1 - mn1);
      m0 = mn0;
      m1 = mn1;
      l0 *= f0;
      l1 *= f1;
#pragma unroll
      for (int dt = 0; dt < 8; ++dt) {
        o[dt][0] *= f0; o[dt][1] *= f0; o[dt][2] *= f1; o[dt][3] *= f1;
      }
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        s[nt][0] = ex2_approx(s[nt][0] - mn0);
        s[nt][1] = ex2_approx(s[nt][1] - mn0);
        s[nt][2] = ex2_approx(s[nt][2] - mn1);
        s[nt][3] = ex2_approx(s[nt][3] - mn1);
        l0 += s[nt][0] + s[nt][1];
        l1 += s[nt][2] + s[nt][3];
      }
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        uint32_t pa[4];
        pa[0] = pack_bf16x2(s[2 * kk][0], s[2 * kk][1]);
        pa[1] = pack_bf16x2(s[2 * kk][2], s[2 * kk][3]);
        pa[2] = pack_bf16x2(s[2 * kk + 1][0], s[2 * kk + 1][1]);
        pa[3] = pack_bf16x2(s[2 * kk + 1][2], s[2 * kk + 1][3]);
#pragma unroll
        for (int dp = 0; dp < 4; ++dp) {
          uint32_t vb[4];
          ptx::ldmatrix_x4_trans(vb, sV + swz(kc * 64 + kk * 16 + (lane & 7) + ((lane >> 3) & 1) * 8,
                                              dp * 16 + (lane >> 4) * 8));
          ptx::mma_m16n8k16_bf16(o[2 * dp], pa, vb[0], vb[1]);
          ptx::mma_m16n8k16_bf16(o[2 * dp + 1], pa, vb[2], vb[3]);
        }
      }
    }
    l0 += __shfl_xor_sync(0xffffffffu, l0, 1);
    l0 += __shfl_xor_sync(0xffffffffu, l0, 2);
    l1 += __shfl_xor_sync(0xffffffffu, l1, 1);
    l1 += __shfl_xor_sync(0xffffffffu, l1, 2);
    const float i0 = 1.0f / l0, i1 = 1.0f / l1;
    bf16* r0 = sO + (qb * 16 + g) * 64 + c2;
    bf16* r1 = r0 + 8 * 64;
#pragma unroll
    for (int dt = 0; dt < 8; ++dt) {
      *reinterpret_cast<uint32_t*>(r0 + dt * 8) = pack_bf16x2(o[dt][0] * i0, o[dt][1] * i0);
      *reinterpret_cast<uint32_t*>(r1 + dt * 8) = pack_bf16x2(o[dt][2] * i1, o[dt][3] * i1);
    }
  }
  ptx::fence_proxy_async_smem();
  compute_sync();
  if (tid == 0) stage_out(a.CTX + ((size_t)h * T + (size_t)b * L) * 64, sO, (uint32_t)(L * 128));
}

// Pooler features [8 a, 8 a + 8): pooled[b, j] = tanh(W_p[j] . x[b, 0] + b_p[j]) (head.cu's
// reading S8); warp w owns features 8 a + 2 w, 8 a + 2 w + 1, whose W_p rows it loads into
// registers before the dependency wait; lane-strided 16-byte vectors, then a warp sum.
template <int MAXV>
__device__ void pool_task(const FusedArgs& a, const FusedTask& t, uint8_t* scratch, unsigned long long* stamp) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nvec = a.H / 8;
  const int j0 = t.a * kPoolFeat + warp * 2;
  uint4 w[2][MAXV];
#pragma unroll
  for (int f = 0; f < 2; ++f)
#pragma unroll
    for (int i = 0; i < MAXV; ++i)
      if (j0 + f < a.H && lane + 32 * i < nvec)
        w[f][i] = __ldg(reinterpret_cast<const uint4*>(a.w_p + (size_t)(j0 + f) * a.H) + lane + 32 * i);
  dep_wait(a, t, stamp);
  for (int b = 0; b < a.B; ++b) {
    uint4 xq[MAXV];
    const bf16* xr = a.X + (size_t)b * a.L * a.H;
#pragma unroll
    for (int i = 0; i < MAXV; ++i)
      if (lane + 32 * i < nvec) xq[i] = ldcg_v4(xr + (lane + 32 * i) * 8);
#pragma unroll
    for (int f = 0; f < 2; ++f) {
      const int j = j0 + f;
      if (j >= a.H) break;
      float s = 0.f;
#pragma unroll
      for (int i = 0; i < MAXV; ++i) {
        if (lane + 32 * i < nvec) {
          const uint32_t wu[4] = {w[f][i].x, w[f][i].y, w[f][i].z, w[f][i].w};
          const uint32_t xu[4] = {xq[i].x, xq[i].y, xq[i].z, xq[i].w};
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const float2 wv = unpack_bf16x2(wu[e]), xv = unpack_bf16x2(xu[e]);
            s = fmaf(wv.x, xv.x, s);
            s = fmaf(wv.y, xv.y, s);
          }
        }
      }
      s = warp_sum(s);
      if (lane == 0) reinterpret_cast<float*>(scratch)[b * kPoolFeat + warp * 2 + f] = tanhf(s + __ldg(a.b_p + j));
    }
  }
  ptx::fence_proxy_async_smem();
  compute_sync();
  if (threadIdx.x == 0 && t.a * kPoolFeat + kPoolFeat <= a.H)
    for (int b = 0; b < a.B; ++b)
      stage_out(a.pooled + (size_t)b * a.H + t.a * kPoolFeat, scratch + b * kPoolFeat * 4, kPoolFeat * 4);
}

// Classifier: logits[b, c] = W_c[c] . pooled[b] + b_c[c], one warp per (b, c).
__device__ void cls_task(const FusedArgs& a, const FusedTask& t, unsigned long long* stamp) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  dep_wait(a, t, stamp);
  for (int p = warp; p < a.B * a.C; p += 4) {
    const int b = p / a.C, c = p - b * a.C;
    const bf16* wr = a.w_c + (size_t)c * a.H;
    const float* pr = a.pooled + (size_t)b * a.H;
    float s = 0.f;
    for (int vi = lane; vi < a.H / 8; vi += 32) {
      float w[8];
      Vec<bf16>::load(wr + vi * 8, w);
      const float4 q0 = ldcg_f4(pr + vi * 8), q1 = ldcg_f4(pr + vi * 8 + 4);
      s = fmaf(w[0], q0.x, s); s = fmaf(w[1], q0.y, s); s = fmaf(w[2], q0.z, s); s = fmaf(w[3], q0.w, s);
      s = fmaf(w[4], q1.x, s); s = fmaf(w[5], q1.y, s); s = fmaf(w[6], q1.z, s); s = fmaf(w[7], q1.w, s);
    }
    s = warp_sum(s);
    if (lane == 0) a.logits[(size_t)b * a.C + c] = s + __ldg(a.b_c + c);
  }
}

template <int MAXV>
__global__ void __launch_bounds__(kThreads, 1) fused_forward_kernel(const __grid_constant__ FusedArgs a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* ring = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* scratch = ring + (size_t)a.stages * a.stage_bytes;
  uint64_t* full = reinterpret_cast<uint64_t*>(scratch + a.scratch_bytes);
  uint64_t* empty = full + a.stages;
  uint64_t* tfull = empty + a.stages;
  uint64_t* tempty = tfull + 2;
  uint64_t* cbar = tempty + 2;  // compute warps' bulk / TMA loads (LayerNorm rows, attention Q K V)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(cbar + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int t0 = a.task_off[blockIdx.x], t1 = a.task_off[blockIdx.x + 1];

  if (threadIdx.x == 0) {
    for (int i = 0; i < a.stages; ++i) {
      ptx::mbar_init(&full[i], 1);
      ptx::mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&tfull[i], 1);
      ptx::mbar_init(&tempty[i], 1);
    }
    ptx::mbar_init(cbar, 1);
    ptx::fence_mbar_init();
  }
  if (warp == kMmaWarp) ptx::tmem_alloc(tmem_slot, 2 * a.tcols);
  if (warp == kProdWarp && lane == 0)
    for (int i = 0; i < kAMaps + 4 * a.layers && i < 64; ++i) ptx::tma_prefetch_desc(a.tm + i);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == kProdWarp) {
    if (lane == 0) producer(a, ring, full, empty, t0, t1);
    if (lane == 1) prefetch_small(a);
  } else if (warp == kMmaWarp) {
    mma_issuer(a, ring, full, empty, tfull, tempty, tmem, t0, t1);
  } else {
    int acc = 0;
    uint32_t aph = 0, cph = 0;
    unsigned long long* const tr = g_ftrace;
    for (int i = t0; i < t1; ++i) {
      const FusedTask t = a.tasks[i];
      if (tr && threadIdx.x == 0) {
        tr[(size_t)i * kTr] = (unsigned long long)t.type | ((unsigned long long)t.layer << 8) |
                            ((unsigned long long)t.a << 24) | ((unsigned long long)t.b << 40) |
                            ((unsigned long long)blockIdx.x << 52);
        tr[(size_t)i * kTr + 1] = gtimer();
        tr[(size_t)i * kTr + 15] = clock64();
      }
      if (is_gemm(t.type)) {
        float bias = 0.f;  // before the accumulator wait (weights: never produced in the kernel)
        if (t.type == FT_QKV || t.type == FT_FFN1)
          bias = __ldg((t.type == FT_FFN1 ? a.lw[t.layer].b_1 : a.lw[t.layer].b_qkv) + t.a * 128 + threadIdx.x);
        ptx::mbar_wait(&tfull[acc], aph);
        if (tr && threadIdx.x == 0) tr[(size_t)i * kTr + 2] = gtimer();
        ptx::tc_fence_after();
        gemm_epilogue(a, t, tmem + (uint32_t)(acc * a.tcols), scratch, bias, i);
        ptx::tc_fence_before();
        if (++acc == 2) {
          acc = 0;
          aph ^= 1;
        }
      } else {
        unsigned long long* stamp = tr ? tr + (size_t)i * kTr + 2 : nullptr;  // ready: dependency met
        if (stamp && threadIdx.x == 0) *stamp = gtimer();
        switch (t.type) {
#ifndef OFF_EMBED
          case FT_EMBED: embed_rows<MAXV>(a, t, scratch); break;
#endif
#ifndef OFF_ATTN
          case FT_ATTN: attention(a, t, scratch, cbar, cph, stamp, i); break;
#endif
#ifndef OFF_LN
          case FT_LN1:
          case FT_LN2: ln_rows<MAXV>(a, t, scratch, stamp, i); break;
#endif
#ifndef OFF_POOL
          case FT_POOL: pool_task<MAXV>(a, t, scratch, stamp); break;
#endif
          case FT_CLS: cls_task(a, t, stamp); break;
        }
      }
      if (tr && threadIdx.x == 0) tr[(size_t)i * kTr + 5] = clock64();
      compute_sync();
      if (threadIdx.x == 0) {
        if (is_gemm(t.type)) {
          ptx::mbar_arrive(&tempty[(acc + 1) & 1]);  // the accumulator just drained
          FT_SUB(i, 9);
        }
        ptx::bulk_wait<0>();  // the task's output copies are complete (in L2)
        FT_SUB(i, 10);
        unsigned* done = task_done(a, t);
        // (an embedding task counts its rows: the layer-0 QKV waits for T rows like later layers)
        // row tasks count their rows, so the QKV of every layer (and the pooler) waits for T rows
        const bool rows = t.type == FT_EMBED || t.type == FT_LN2;
        if (done) signal_done(done, rows ? (unsigned)min(kRowsPerTask, a.T - t.a * kRowsPerTask) : 1u);
        if (tr) tr[(size_t)i * kTr + 3] = gtimer();
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == kMmaWarp) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, 2 * a.tcols);
  }
  // the last CTA out resets the counters for the next launch (graph replays)
  if (threadIdx.x == 0) {
    unsigned* fin = a.cnt + (a.layers + 1) * kStagesPerLayer;
    __threadfence();
    if (atomicAdd(fin, 1u) == gridDim.x - 1) {
      for (int i = 0; i < (a.layers + 1) * kStagesPerLayer; ++i) a.cnt[i] = 0;
      *fin = 0;
      __threadfence();
    }
  }
}

}  // namespace

// ------------------------------------------------------------------ host side
cudaError_t set_fused_trace(unsigned long long* buf) { return cudaMemcpyToSymbol(g_ftrace, &buf, sizeof(buf)); }

int fused_split(int N, int K) {
  // smallest S dividing K/64 with at most `kb_max` k-blocks per unit; kb_max = 4 for K <= 1024
  // (out-proj: 768 -> 3, 1024 -> 4), 6..8 above (FFN2: 3072 -> 8, 4096 -> 8)
  (void)N;
  const int nkb = K / 64;
  const int kb_max = K <= 1024 ? 4 : 8;
  if (const char* e = getenv(K <= 1024 ? "ARLO_FUSED_KB_O" : "ARLO_FUSED_KB_F2")) {
    const int v = atoi(e);
    if (v > 0) {
      for (int s = 1; s <= nkb; ++s)
        if (nkb % s == 0 && nkb / s <= v) return s;
    }
  }
  for (int s = 1; s <= nkb; ++s)
    if (nkb % s == 0 && nkb / s <= kb_max) return s;
  return nkb;
}

struct FusedPlanImpl {
  FusedArgs args;
  void* dev = nullptr;
  int grid = 0, smem = 0, maxv = 0;
};

bool fused_supported(int B, int L, int H, int heads, int F) {
  const int T = B * L;
  return T >= 16 && T <= 256 && T % 16 == 0 && L <= kAttnRows && H % 128 == 0 && F % 128 == 0 &&
         heads * 64 == H && H <= 1024;
}

void fused_destroy(FusedPlanImpl* p) {
  if (!p) return;
  if (p->dev) cudaFree(p->dev);
  delete p;
}

// t = the canonical weight tensors (arlo.h), buffers from the runtime arena.
FusedPlanImpl* fused_create(int B, int L, int layers, int H, int heads, int F, int C, int vocab, float eps,
                            const void* const* t, const int32_t* ids, const int32_t* lengths, int32_t* err, void* X,
                            void* X1, void* QKV, void* CTX, void* HB, float* pooled, float* logits) {
  if (!fused_supported(B, L, H, heads, F)) return nullptr;
  const int T = B * L;
  FusedPlanImpl* p = new FusedPlanImpl;
  FusedArgs& a = p->args;
  memset(&a, 0, sizeof a);
  a.layers = layers; a.H = H; a.heads = heads; a.F = F; a.C = C; a.vocab = vocab; a.B = B; a.L = L; a.T = T;
  a.eps = eps;
  a.s_o = fused_split(H, H);
  a.s_f2 = fused_split(H, F);
  a.stage_bytes = kWBytes + T * 128;
  // compute scratch: attention Q (L rows of 128 B), K, V (L rounded up to 64 rows each), O (L rows);
  // GEMM epilogue staging [64][128] fp32 = 32 KB; LayerNorm constants + row staging
  const int kvr = (L + 63) & ~63;
  a.scratch_bytes = std::max({(2 * L + 2 * kvr) * 128, 32768, kLnStage + kRowsPerTask * H * 2,
                                                        0});
  a.scratch_bytes = (a.scratch_bytes + 1023) & ~1023;
  a.stages = (kSmemOptIn - 1024 - a.scratch_bytes - 256) / a.stage_bytes;
  if (a.stages > 8) a.stages = 8;
  a.tcols = 32;
  while (a.tcols < T) a.tcols <<= 1;
  a.n_rows = (T + kRowsPerTask - 1) / kRowsPerTask;
  a.n_pool = (H + kPoolFeat - 1) / kPoolFeat;
  p->grid = num_sms();
  p->smem = 1024 + a.stages * a.stage_bytes + a.scratch_bytes + 256;
  p->maxv = (H / 8 + 31) / 32;

  // ---- static task graph, topological order, round-robin over the CTAs
  std::vector<FusedTask> order;
  auto push = [&](uint16_t type, int layer, int x, int y) {
    order.push_back(FusedTask{type, (uint16_t)layer, (uint16_t)x, (uint16_t)y});
  };
  for (int r = 0; r < a.n_rows; ++r) push(FT_EMBED, 0, r, 0);
  for (int l = 0; l < layers; ++l) {
    for (int n = 0; n < 3 * H / 128; ++n) push(FT_QKV, l, n, 0);
    for (int b = 0; b < B; ++b)
      for (int h = 0; h < heads; ++h) push(FT_ATTN, l, b, h);
    for (int s = 0; s < a.s_o; ++s)
      for (int n = 0; n < H / 128; ++n) push(FT_OPROJ, l, n, s);
    for (int r = 0; r < a.n_rows; ++r) push(FT_LN1, l, r, 0);
    for (int n = 0; n < F / 128; ++n) push(FT_FFN1, l, n, 0);
    for (int s = 0; s < a.s_f2; ++s)
      for (int n = 0; n < H / 128; ++n) push(FT_FFN2, l, n, s);
    for (int r = 0; r < a.n_rows; ++r) push(FT_LN2, l, r, 0);
  }
  for (int j = 0; j < a.n_pool; ++j) push(FT_POOL, layers, j, 0);
  push(FT_CLS, layers, 0, 0);
  std::vector<std::vector<FusedTask>> per(p->grid);
  for (size_t i = 0; i < order.size(); ++i) per[i % p->grid].push_back(order[i]);
  std::vector<int> off(p->grid + 1, 0);
  std::vector<FusedTask> tasks;
  for (int c = 0; c < p->grid; ++c) {
    off[c] = (int)tasks.size();
    tasks.insert(tasks.end(), per[c].begin(), per[c].end());
  }
  off[p->grid] = (int)tasks.size();

  // ---- tensor maps: A operands (box {64, T}) and per-layer weights (box {64, 128})
  std::vector<CUtensorMap> tm(kAMaps + 4 * layers);
  bool ok = encode_tmap_bf16_2d(&tm[TM_X], X, H, T, 64, T, 128) &&
            encode_tmap_bf16_3d(&tm[TM_CTX], CTX, 64, T, H / 64, 64, T, 128) &&
            encode_tmap_bf16_2d(&tm[TM_X1], X1, H, T, 64, T, 128) &&
            encode_tmap_bf16_3d(&tm[TM_HB], HB, 128, T, F / 128, 64, T, 128) &&
            encode_tmap_bf16_3d(&tm[TM_QKV], QKV, 128, T, 3 * H / 128, 64, L, 128);
  std::vector<FusedLayer> lw(layers);
  for (int l = 0; l < layers && ok; ++l) {
    const void* const* lt = t + 5 + 12 * l;
    ok = encode_tmap_bf16_2d(&tm[kAMaps + 4 * l + 0], lt[0], H, 3 * H, 64, 128, 128) &&
         encode_tmap_bf16_2d(&tm[kAMaps + 4 * l + 1], lt[2], H, H, 64, 128, 128) &&
         encode_tmap_bf16_2d(&tm[kAMaps + 4 * l + 2], lt[6], H, F, 64, 128, 128) &&
         encode_tmap_bf16_2d(&tm[kAMaps + 4 * l + 3], lt[8], F, H, 64, 128, 128);
    lw[l] = FusedLayer{(const float*)lt[1], (const float*)lt[3], (const float*)lt[4], (const float*)lt[5],
                       (const float*)lt[7], (const float*)lt[9], (const float*)lt[10], (const float*)lt[11]};
  }
  if (!ok) {
    fused_destroy(p);
    return nullptr;
  }

  // ---- one device allocation: tensor maps | layer pointers | task offsets | tasks | counters | partials
  auto al = [](size_t x) { return (x + 255) & ~size_t(255); };
  const size_t n_cnt = (size_t)(layers + 1) * kStagesPerLayer + 1;
  const int smax = a.s_o > a.s_f2 ? a.s_o : a.s_f2;
  size_t o = 0;
  const size_t o_tm = o; o = al(o + tm.size() * sizeof(CUtensorMap));
  const size_t o_lw = o; o = al(o + lw.size() * sizeof(FusedLayer));
  const size_t o_off = o; o = al(o + off.size() * sizeof(int));
  const size_t o_tasks = o; o = al(o + tasks.size() * sizeof(FusedTask));
  const size_t o_cnt = o; o = al(o + n_cnt * sizeof(unsigned));
  const size_t o_P = o; o = al(o + (size_t)smax * T * H * sizeof(float));
  if (cudaMalloc(&p->dev, o) != cudaSuccess) {
    p->dev = nullptr;
    fused_destroy(p);
    return nullptr;
  }
  char* d = (char*)p->dev;
  bool cp = cudaMemset(d, 0, o) == cudaSuccess &&
            cudaMemcpy(d + o_tm, tm.data(), tm.size() * sizeof(CUtensorMap), cudaMemcpyHostToDevice) == cudaSuccess &&
            cudaMemcpy(d + o_lw, lw.data(), lw.size() * sizeof(FusedLayer), cudaMemcpyHostToDevice) == cudaSuccess &&
            cudaMemcpy(d + o_off, off.data(), off.size() * sizeof(int), cudaMemcpyHostToDevice) == cudaSuccess &&
            cudaMemcpy(d + o_tasks, tasks.data(), tasks.size() * sizeof(FusedTask), cudaMemcpyHostToDevice) == cudaSuccess;
  if (!cp) {
    fused_destroy(p);
    return nullptr;
  }
  a.tm = (const CUtensorMap*)(d + o_tm);
  a.lw = (const FusedLayer*)(d + o_lw);
  a.task_off = (const int*)(d + o_off);
  a.tasks = (const FusedTask*)(d + o_tasks);
  a.cnt = (unsigned*)(d + o_cnt);
  a.P = (float*)(d + o_P);
  a.word = (const bf16*)t[0]; a.pos = (const bf16*)t[1]; a.type = (const bf16*)t[2];
  a.emb_g = (const float*)t[3]; a.emb_b = (const float*)t[4];
  const void* const* hd = t + 5 + 12 * layers;
  a.w_p = (const bf16*)hd[0]; a.b_p = (const float*)hd[1]; a.w_c = (const bf16*)hd[2]; a.b_c = (const float*)hd[3];
  a.ids = ids; a.lengths = lengths; a.err = err;
  a.X = (bf16*)X; a.X1 = (bf16*)X1; a.QKV = (bf16*)QKV; a.CTX = (bf16*)CTX; a.HB = (bf16*)HB;
  a.pooled = pooled; a.logits = logits;
  return p;
}

template <int MAXV>
static cudaError_t fused_launch_t(const FusedPlanImpl& p, cudaStream_t s) {
  auto kern = fused_forward_kernel<MAXV>;
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t e = once_per_device(attr_done, [&] {
    return cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemOptIn); });
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(p.grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = p.smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;  // every CTA resident: tasks wait on each other
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, p.args);
}

cudaError_t fused_launch(const FusedPlanImpl* p, cudaStream_t s) {
  switch (p->maxv) {
    case 1: return fused_launch_t<1>(*p, s);
    case 2: return fused_launch_t<2>(*p, s);
    case 3: return fused_launch_t<3>(*p, s);
    case 4: return fused_launch_t<4>(*p, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace arlo
