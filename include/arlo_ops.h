/*
 * arlo_ops.h — per-kernel entry points of libarlo.so, one per hot-path step of
 * SURVEY.md §8(a).  They launch exactly the kernels the runtime graphs launch
 * (same code, same launch configuration chooser) on plain DEVICE buffers, so
 * tests can check each step against the oracle in isolation and bench can
 * time one kernel.  All pointers are DEVICE pointers; `stream` is a
 * cudaStream_t (NULL = legacy default stream); calls are asynchronous.
 * dtype is ARLO_BF16 or ARLO_FP32 (arlo.h); in ARLO_BF16 activations and
 * matrices are bf16 and vectors (bias, gamma, beta) fp32; in ARLO_FP32 all
 * are fp32.  Errors: ARLO_EINVAL for bad shapes/null pointers, ARLO_ECUDA for
 * launch failures.
 */
#ifndef ARLO_OPS_H_
#define ARLO_OPS_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { ARLO_EPI_BIAS = 0, ARLO_EPI_BIAS_GELU = 1, ARLO_EPI_BIAS_RESIDUAL = 2 };

/*
 * Step a2/a4/a6/a7: out[M,N] = epi(A[M,K] * W[N,K]^T + bias[N]) with
 * epi = identity | GELU_erf | (+ residual[M,N]).  Row-major, K-major operands
 * (PyTorch Linear layout).  Requires N % 64 == 0, K % 64 == 0, 1 <= M.
 * ARLO_BF16 runs the tcgen05/TMEM/TMA kernel; ARLO_FP32 the FFMA kernel.
 * force_bn: 0 = automatic tile choice; 64/128/192/256 = single-CTA kernel with that tile
 * width; -128/-192/-256 = CTA-pair (cta_group::2, 256-row tiles) kernel; 1016/1032/1064 =
 * skinny small-M kernel (one CTA per 128 x BN tile, BN = 16/32/64) (tests, sweeps).
 * Every choice gives bitwise the same rows (same K order per output element).
 */
int arlo_op_gemm(int32_t dtype, int32_t M, int32_t N, int32_t K, const void* A, const void* W,
                 const float* bias, const void* residual, void* out, int32_t epi,
                 int32_t force_bn, void* stream);

/*
 * Steps a4+a5 / a7+a8 fused (bf16): out[M,N] = LN(A W^T + bias + residual; gamma, beta, eps)
 * over full rows, N = hidden size (multiple of 192 or 256 with <= 8 column tiles, or 128).
 * A cluster of N/BN CTAs shares per-row statistics through distributed shared memory.
 * `out` may alias `residual`.  Errors: ARLO_EINVAL for unsupported N / bad pointers.
 */
int arlo_op_gemm_ln(int32_t M, int32_t N, int32_t K, const void* A, const void* W, const float* bias,
                    const void* residual, const float* gamma, const float* beta, float eps, void* out,
                    void* stream);

/* Step a5/a8: out[M,H] = LN(in[M,H]; gamma, beta, eps) per row (biased variance). */
int arlo_op_layernorm(int32_t dtype, int32_t M, int32_t H, const void* in, const float* gamma,
                      const float* beta, float eps, void* out, void* stream);

/*
 * Step a1: out[b*L + t] = LN(word[id] + pos[t] + type[0]) with id = ids[b,t]
 * for t < lengths[b] and id = 0 otherwise; ids outside [0, vocab) are replaced
 * by 0 and set *err_flag (device int32, may be NULL) to 1.
 */
int arlo_op_embed(int32_t dtype, int32_t B, int32_t L, int32_t H, int32_t vocab,
                  const int32_t* ids, const int32_t* lengths, const void* word, const void* pos,
                  const void* type, const float* gamma, const float* beta, float eps, void* out,
                  int32_t* err_flag, void* stream);

/*
 * Step a3: padding-masked multi-head attention over a static [B, L] batch.
 * qkv [B*L, 3H] (Q | K | V, head j at columns j*64), o [B*L, H].  Query row t
 * of sequence b attends keys 0..lengths[b]-1 with scale 1/8; key tiles past
 * lengths[b] are skipped; rows of a query tile lying wholly at t >=
 * lengths[b] are written as 0 (never read by a real token).  Query tiles are
 * 128 rows (bf16: tcgen05 kernel, requires L <= 512).
 */
int arlo_op_attention(int32_t dtype, int32_t B, int32_t L, int32_t heads, const void* qkv,
                      const int32_t* lengths, void* o, void* stream);

/*
 * Step a9: pooled[b] = tanh(W_p x[b*L] + b_p) (fp32 [B, H], caller-provided
 * scratch), logits[b] = W_c pooled[b] + b_c for b < B, fp32 out [B, C].  H <= 2048.
 */
int arlo_op_head(int32_t dtype, int32_t B, int32_t L, int32_t H, int32_t C, const void* x,
                 const void* w_p, const float* b_p, const void* w_c, const float* b_c,
                 float* pooled, float* logits, void* stream);

/*
 * Steps a5/a8 + a6 (or the next layer's a2) in one launch, as the runtime graphs run them:
 * x = LN(y; gamma, beta, eps) over M rows of K = hidden (LayerNorm of the residual GEMM's
 * output, reading S3), then out = epi(x W^T + bias), epi = ARLO_EPI_BIAS or ARLO_EPI_BIAS_GELU.
 * y, x: [M, K] bf16 DEVICE (x is written: the next residual); W [N, K] bf16; out [M, N] bf16.
 * The whole persistent grid normalises the rows, meets at a grid barrier (`barrier`: 8 bytes of
 * zero-initialised DEVICE memory, reusable by later calls on the same stream), then runs the GEMM.
 * force_bn: a persistent tile code (BN / -BN, see arlo_gemm_tile_choice), 0 = chooser; EINVAL if
 * that kernel is the skinny one (its grid is not persistent).  Launches with a grid barrier must
 * not run concurrently with one another on the same device (one runtime stream per device).
 */
int arlo_op_ln_gemm(int32_t M, int32_t N, int32_t K, const void* y, const float* gamma, const float* beta, float eps,
                    void* x, const void* W, const float* bias, void* out, int32_t epi, int32_t force_bn,
                    void* barrier, void* stream);

/*
 * LayerNorm fold epilogues of the tcgen05 GEMM (the throughput runtimes fold every LayerNorm into
 * the GEMMs around it instead of launching it; BERT post-LN, PAPER.md:L422 [17]).
 * Row statistics st[g][row][2] = (sum, sum of squares) of the 32 bf16 values of granule g of a row
 * (fp32, column order), granule-major with st_ld >= M rows per granule plane; a consumer adds the
 * granules in order and uses var = E[y^2] - mean^2.
 *   epi ARLO_EPI_LNFOLD (3) / ARLO_EPI_LNFOLD_GELU (4): A = y [M, K] (not normalised), W = W' [N, K]
 *     (= bf16(W * gamma)), v0 = s [N] (row sums of W'), v1 = c [N] (= W beta + b), st_in = statistics
 *     of A's rows (K / 32 granules; row i's statistics are those of row i * st_in_stride):
 *     out = bf16(rstd_i * acc - rstd_i * mean_i * s_n + c_n) (then GELU, erf form).
 *   epi ARLO_EPI_RESID_LN (5): out = bf16((acc + v0_n) + LN(r)) with LN(r) = ((r - mean) * rstd) *
 *     v1_n + v2_n from the residual rows r and their statistics st_in (N / 32 granules; st_in = NULL:
 *     plain residual r); st_out (optional) receives the statistics of the bf16 output rows.
 * Device pointers; M >= 1, N and K multiples of 64; force_bn as for arlo_op_gemm.  Split-K codes
 * (2000 + BN, BN in {32, 64, 128}: splitk_factor(N, K) partial sums in a fixed order) are accepted
 * for epi 5 only (the LATENCY runtimes' FFN2); there each granule's statistics are the column-order
 * sums of its 8 four-column quads, added by an xor tree (the same at every M and tile width).
 * Errors: EINVAL, ECUDA.
 */
enum { ARLO_EPI_LNFOLD = 3, ARLO_EPI_LNFOLD_GELU = 4, ARLO_EPI_RESID_LN = 5 };
int arlo_op_gemm_fold(int32_t M, int32_t N, int32_t K, const void* A, const void* W, const float* v0,
                      const float* v1, const float* v2, const float* st_in, int32_t st_in_stride,
                      float* st_out, int32_t st_ld, float eps, const void* residual, void* out, int32_t epi,
                      int32_t force_bn, void* stream);

/* The tile configuration arlo_op_gemm / the runtime graphs use for (M, N, K):
 * BN for the single-CTA kernel, -BN for the CTA-pair kernel, 1000 + BN for the
 * skinny small-M kernel, 0 if unsupported. */
int32_t arlo_gemm_tile_choice(int32_t M, int32_t N, int32_t K);

/*
 * Profiling hook (tools/gemm_trace.py): when `buf` is a DEVICE buffer of
 * >= 64 * grid uint64 entries, later single-CTA GEMM launches write
 * %globaltimer stamps of their pipeline events into it; NULL turns it off.
 */
int arlo_debug_gemm_trace(void* buf);
/* Same for the bf16 attention kernel: >= 64 * 2048 uint64 entries. */
int arlo_debug_attn_trace(void* buf);
/* Same for the fused persistent forward (ARLO_RUNTIME_FUSED): >= 6 uint64 per task of the
 * plan (the task array in CTA order); stamps per task: [type | layer << 8 | a << 24 | b << 40 |
 * cta << 52, compute begin, ready (dependency met / accumulator full), end (after its completion
 * signal), producer dependency met (GEMM units), 0] in %globaltimer ns (tools/fused_trace.py). */
int arlo_debug_fused_trace(void* buf);

#ifdef __cplusplus
}
#endif
#endif /* ARLO_OPS_H_ */
