// kernels.h — host-side launchers of the hot-path kernels.
// Every launcher is asynchronous on `stream`, takes raw device pointers and
// returns cudaSuccess or the launch error.  No torch types anywhere.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <cuda.h>  // CUtensorMap (header only; the driver entry point is resolved at run time)

namespace arlo {

enum DType { DT_BF16 = 0, DT_FP32 = 1 };
enum Epi {
  EPI_BIAS = 0, EPI_BIAS_GELU = 1, EPI_BIAS_RESID = 2,
  // LayerNorm folded into the GEMMs (runtime.cu, ARLO_NO_LN_FOLD=1 disables):
  //  EPI_LNFOLD / _GELU: A = y (a residual sum, NOT normalised), W' = W * gamma (column scaled),
  //    out = rstd_r * acc - rstd_r * mu_r * s_n + c_n (s = W' row sums, c = W beta + b), mu_r and
  //    rstd_r from the per-row statistics of y (FoldArgs::st_in), then GELU for _GELU;
  //  EPI_RESID_LN: out = (acc + b_n) + LN(r) with LN(r) = (r - mu_r) * rstd_r * gamma_n + beta_n
  //    computed on the fly from the residual rows r and their statistics (plain r when st_in is
  //    null), and the statistics of the bf16 output written to FoldArgs::st_out.
  EPI_LNFOLD = 3, EPI_LNFOLD_GELU = 4, EPI_RESID_LN = 5
};

// Row statistics of an activation y[M, H] for the LayerNorm fold: per row, per 32-column granule
// g, the fp32 sums (sum_j y, sum_j y^2) over its 32 bf16 values in column order, stored
// granule-major st[g][row][2] with a fixed row capacity `st_ld` (a warp's 32 rows are contiguous:
// coalesced stores by the producing epilogue and loads by the consumer).  A consumer adds the
// H/32 granules in order: every kernel and tile shape produces the same bits.
struct FoldArgs {
  const float* v1;    // EPI_LNFOLD*: c [N];  EPI_RESID_LN: gamma [N] of the residual's LayerNorm
  const float* v2;    // EPI_RESID_LN: beta [N]
  const float* st_in; // EPI_LNFOLD*: statistics of A's rows (K/32 granules); EPI_RESID_LN: of the residual rows
  int st_in_stride;   // row stride of st_in in rows (1, or L for the CLS rows of a full layer)
  float* st_out;      // EPI_RESID_LN: statistics of the output rows (N/32 granules)
  float eps;
  int st_ld;          // rows per granule plane of st_in and st_out (their allocated row count)
};

int num_sms();
int set_gemm_trace(unsigned long long* buf);  // profiling hook, nullptr = off
int set_attn_trace(unsigned long long* buf);  // profiling hook, nullptr = off

// ---- a1: embedding + LN;  a5/a8: LN ------------------------------------------------------
cudaError_t launch_embed_ln(DType dt, int B, int L, int H, int vocab, const int32_t* ids,
                            const int32_t* lengths, const void* word, const void* pos,
                            const void* type, const float* g, const float* b, float eps, void* out,
                            int32_t* err_flag, cudaStream_t s);
cudaError_t launch_layernorm(DType dt, int M, int H, const void* in, const float* g,
                             const float* b, float eps, void* out, cudaStream_t s);
// LayerNorm fold: W' = bf16(W * gamma) (column scale), s = row sums of W', c = W beta + b (see EPI_LNFOLD)
cudaError_t launch_fold_weights(int N, int K, const void* W, const float* gamma, const float* beta, const float* b,
                                void* Wf, float* s, float* c, cudaStream_t st);

// ---- a2/a4/a6/a7: GEMM + fused epilogue ----------------------------------------------------
// LayerNorm run as the prologue of a persistent GEMM (layernorm.cuh): x = LN(y) over `rows`
// rows of H, then a grid barrier, then the GEMM on x.  y == nullptr: no prologue.
struct LnPrologue {
  const void* y;   // [rows, H] bf16 input (the previous residual GEMM's output)
  const float* g;  // gamma [H]
  const float* b;  // beta [H]
  void* x;         // [rows, H] bf16 output (this GEMM's A operand)
  unsigned* bar;   // grid barrier {count, generation}: zero-initialised device memory
  float eps;
  int rows, H;
};

// tcgen05 plan: tensor maps are encoded once (at runtime create) and the
// launch is then a plain kernel launch that CUDA graphs can capture.
struct TcGemmPlan {
  CUtensorMap tmA;  // activations [M, K] bf16, box {64, 128}, 128B swizzle
  CUtensorMap tmB;  // weights     [N, K] bf16, box {64, BN (BN/2 for a pair)}, 128B swizzle
  CUtensorMap tmC;  // output      [M, N] bf16, box {32, 32}, 64B swizzle (epilogue TMA stores)
  CUtensorMap tmR;  // residual    [M, N] bf16 (row stride ldr), box {32, 128}, 64B swizzle (EPI_BIAS_RESID)
  int M, N, K, BN, epi, grid;
  int ew;       // epilogue warps of the persistent kernels (8, or 12 for GELU at M <= 8192)
  bool pair;    // CTA-pair (cta_group::2) kernel, 256-row tiles
  bool skinny;  // small-M kernel: one CTA per 128 x BN tile (BN 16/32/64), direct stores
  int a_rows;   // skinny / split-K: A box rows (min(128, M rounded up to 8))
  // split-K weight-streaming kernel (latency runtimes): a cluster of `splits` CTAs per
  // (n-tile, 128-row block), CTA s accumulates K range [s*kc, (s+1)*kc); the partials are
  // summed in the fixed order s = 0, 1, ... over distributed shared memory
  bool splitk;
  int splits, kc, stages, a_stage, smem;
  bool ln;    // fused residual + LayerNorm epilogue over full rows (cluster of N/BN CTAs)
  const float* gamma;
  const float* beta;
  float eps;
  const float* bias;
  const void* resid;
  int ldr;  // residual row stride (elements)
  void* out;
  LnPrologue lnp;  // (bias / GELU epilogues of the persistent tile kernels only)
  FoldArgs fold;   // EPI_LNFOLD, EPI_LNFOLD_GELU, EPI_RESID_LN
};
// Attach a LayerNorm prologue to a planned GEMM whose A operand is lnp.x; false if the plan's
// kernel cannot run it (skinny / split-K / residual epilogue / H > 1024).
bool tc_plan_attach_ln(TcGemmPlan* p, const LnPrologue& lnp);
bool tc_plan_gemm(TcGemmPlan* p, int M, int N, int K, const void* A, const void* W,
                  const float* bias, const void* resid, void* out, int epi, int force_bn);
// Row-strided variant: A row i at A + i*lda, residual row i at resid + i*ldr (elements).
// The runtime's CLS-only last layer reads row 0 of every sequence (lda = ldr = L*H).
bool tc_plan_gemm_strided(TcGemmPlan* p, int M, int N, int K, const void* A, int lda, const void* W,
                          const float* bias, const void* resid, int ldr, void* out, int epi, int force_bn);
cudaError_t tc_launch_gemm(const TcGemmPlan& p, cudaStream_t s);
// Tile choice codes: BN (single CTA), -BN (CTA pair), kSkinnyCode + BN (skinny kernel).
constexpr int kSkinnyCode = 1000;
constexpr int kSplitKCode = 2000;  // kSplitKCode + BN: split-K kernel (splitk_factor(N, K) splits)
constexpr int kFusedCode = 3000;   // kFusedCode + split factor: unit of the fused persistent forward
int tc_choose_bn(int M, int N, int K);
// out = LN(A W^T + bias + resid; gamma, beta, eps), N = hidden size (128 / 768 / 1024 ...).
// `out` may alias `resid` (each tile reads its residual before storing the same region).
bool tc_plan_gemm_ln(TcGemmPlan* p, int M, int N, int K, const void* A, const void* W, const float* bias,
                     const void* resid, const float* gamma, const float* beta, float eps, void* out);

// Split-K plan (the weight-streaming GEMM of latency runtimes, M = b*L small).  The split
// factor is splitk_factor(N, K): a function of the weight shape only, so every runtime of
// the latency family reduces each output element in the same order (cross-L bitwise).
// bn = 0 lets splitk_bn(M, N, S) choose the tile width (any width gives the same bits).
int splitk_factor(int N, int K);
cudaError_t splitk_launch(const TcGemmPlan& p, cudaStream_t s);  // (tc_launch_gemm dispatches here)
int splitk_bn(int M, int N, int S);
bool tc_plan_gemm_splitk(TcGemmPlan* p, int M, int N, int K, const void* A, int lda, const void* W,
                         const float* bias, const void* resid, int ldr, void* out, int epi, int bn = 0);

cudaError_t launch_gemm_simt(DType dt, int M, int N, int K, const void* A, const void* W,
                             const float* bias, const void* resid, void* out, int epi,
                             cudaStream_t s);

// ---- a3: masked attention -----------------------------------------------------------------
// bf16: tcgen05 flash attention, QKV read through a TMA map encoded once per
// (buffer, B, L) at plan time; fp32 check mode: FFMA kernel.  L <= 512 (bf16).
struct AttnPlan {
  CUtensorMap tm;  // QKV [B*L, 3H] bf16, box {64, 128}, 128B swizzle
  int B, L, heads;
  int q_rows;  // queries computed per sequence: L, or 1 for the CLS-only last layer (one 128-row q-tile)
  DType dt;
  const void* qkv;
};
bool attn_plan(AttnPlan* p, DType dt, int B, int L, int heads, const void* qkv, int q_rows = 0);
cudaError_t attn_launch(const AttnPlan& p, const int32_t* lengths, void* o, cudaStream_t s);

// ---- a9: CLS pooler + classifier ----------------------------------------------------------
// ln: optional LayerNorm applied to the CLS rows on the fly (the LN fold leaves the last layer's
// output un-normalised): x = bf16((y - mu) rstd * gamma + beta), mu / rstd from the row statistics
struct HeadLn {
  const float* st;  // granule statistics [H/32][st_ld][2] of y (row of sequence i: i * L), or nullptr
  const float* gamma;
  const float* beta;
  float eps;
  int st_ld;
};
cudaError_t launch_head(DType dt, int B, int L, int H, int C, const void* x, const void* w_p,
                        const float* b_p, const void* w_c, const float* b_c, float* pooled,
                        float* logits, cudaStream_t s, HeadLn ln = HeadLn{}, unsigned* cnt = nullptr);
// (cnt: [ceil(B / 8)] zero-initialised counters -> the classifier runs in the pooler's last CTA of
//  each 8-sequence group instead of a second kernel; the runtimes pass their arena's counters)

// ---- fused persistent forward (encoder_fused.cu): the whole batch-1 forward as one kernel ----
struct FusedPlanImpl;
bool fused_supported(int B, int L, int H, int heads, int F);
int fused_split(int N, int K);  // split-K factor of the fused family's GEMM units (weight shape only)
// t = the canonical weight tensors of arlo_weights_create; nullptr if unsupported / allocation failed
FusedPlanImpl* fused_create(int B, int L, int layers, int H, int heads, int F, int C, int vocab, float eps,
                            const void* const* t, const int32_t* ids, const int32_t* lengths, int32_t* err, void* X,
                            void* X1, void* QKV, void* CTX, void* HB, float* pooled, float* logits);
cudaError_t fused_launch(const FusedPlanImpl* p, cudaStream_t s);
void fused_destroy(FusedPlanImpl* p);
cudaError_t set_fused_trace(unsigned long long* buf);  // profiling hook, nullptr = off

// Resolve cuTensorMapEncodeTiled through the runtime (no link-time libcuda dependency).
// row_elems = row stride in elements (0: rows are contiguous, stride = inner).
bool encode_tmap_bf16_2d(CUtensorMap* tm, const void* base, uint64_t inner, uint64_t outer,
                         uint32_t box_inner, uint32_t box_outer, int swizzle_bytes, uint64_t row_elems = 0);
bool encode_tmap_bf16_3d(CUtensorMap* tm, const void* base, uint64_t inner, uint64_t mid, uint64_t outer,
                         uint32_t box_inner, uint32_t box_mid, int swizzle_bytes);

}  // namespace arlo
