/*
 * arlo.h — C ABI of the B200-native per-length encoder runtimes behind Arlo's
 * polymorphing (Tan et al., "Arlo: Serving Transformer-based Language Models
 * with Dynamic Input Lengths", ICPP '24; text in PAPER.md).
 *
 * Polymorphing = several statically shaped runtimes of one model, each
 * compiled for a fixed max_length L; a request of length len may run only on
 * runtimes with max_length >= len, zero-padded to L (§1,
 * L101 §2.2, L111 §2.3, L135 §3.2).  This library implements one such runtime
 * on one B200 (arlo_runtime_*) and the two host-side schedulers around them:
 * the Runtime Scheduler's allocation program (arlo_allocate, Eqs. 1-7,
 * PAPER.md:L181-203 §3.3) and the Request Scheduler's multi-level queue
 * (arlo_sched_* / arlo_dispatch, Algorithm 1, §3.4).
 *
 * Conventions
 *  - Every call returning int returns ARLO_OK (0) or a negative ARLO_E* code;
 *    no C++ exception crosses this boundary.  arlo_last_error() returns a
 *    thread-local message describing the last failure on the calling thread.
 *  - Pointers documented as "host or device" are classified with
 *    cudaPointerGetAttributes; all other device pointers must be CUDA device
 *    (or managed) memory on the runtime's device.
 *  - Ownership: the caller owns every buffer it passes.  Weights are BORROWED
 *    (the caller keeps them alive and unchanged until every runtime built on
 *    them is destroyed); a runtime OWNS its activation arena and CUDA graphs.
 *  - Thread safety: a runtime or a scheduler is used by one host thread at a
 *    time.  Different runtimes may be driven concurrently from different
 *    threads.
 */
#ifndef ARLO_H_
#define ARLO_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
  ARLO_OK = 0,
  ARLO_EINVAL = -1,       /* bad argument (shape, null pointer, id out of range) */
  ARLO_ETOOLONG = -2,     /* a request longer than the runtime's L */
  ARLO_ENOMEM = -3,       /* device or host allocation failed */
  ARLO_ECUDA = -4,        /* a CUDA runtime/driver call failed (message says which) */
  ARLO_EINFEASIBLE = -5,  /* Eqs. 2, 3, 7 cannot all hold */
  ARLO_ENOCAND = -6,      /* no deployed runtime with max_length >= len */
  ARLO_ENODEV = -7        /* no sm_100 CUDA device available */
};

enum { ARLO_BF16 = 0, ARLO_FP32 = 1 };

/* Thread-local message of the last failing call on this thread ("" if none). */
const char* arlo_last_error(void);
/* Library version string. */
const char* arlo_version(void);

/* ------------------------------------------------------------------ model */
/*
 * BERT encoder dimensions (Devlin et al. [17]; the evaluated
 * "Bert-Base and Bert-Large").  heads must divide hidden with
 * hidden/heads == 64; hidden % 64 == 0; ffn % 64 == 0; num_labels in [1, 64].
 * dtype ARLO_BF16: bf16 storage, tcgen05 tensor-core GEMMs, fp32 accumulation,
 * softmax and LayerNorm statistics.  dtype ARLO_FP32 ("check mode"): every
 * tensor fp32 and every product an fp32 FFMA (no TF32).
 */
typedef struct {
  int32_t layers, hidden, heads, ffn, vocab, max_pos, type_vocab, num_labels;
  float ln_eps;
  int32_t dtype;
} arlo_model_config;

typedef struct arlo_weights arlo_weights;

/* Number of tensors arlo_weights_create expects: 5 + 12*layers + 4. */
int32_t arlo_weights_count(const arlo_model_config* cfg);

/*
 * Wrap a weight set that already lives on `device`.  tensors[] are DEVICE
 * pointers in canonical order:
 *   word_emb[vocab,H], pos_emb[max_pos,H], type_emb[type_vocab,H], emb_ln_g[H], emb_ln_b[H],
 *   per layer: W_qkv[3H,H], b_qkv[3H], W_o[H,H], b_o[H], ln1_g[H], ln1_b[H],
 *              W_1[F,H], b_1[F], W_2[H,F], b_2[H], ln2_g[H], ln2_b[H],
 *   W_p[H,H], b_p[H], W_c[C,H], b_c[C].
 * Matrices and embedding tables are row-major [out,in] in cfg->dtype (bf16 or
 * fp32); all vectors (biases, LayerNorm gamma/beta) are fp32.  W_qkv stacks
 * the query, key and value projections (rows 0..H-1 = Q).  Every pointer must
 * be 16-byte aligned.  BORROWED: not copied, not freed.
 * Errors: EINVAL (bad config / null / misaligned pointer), ENODEV, ECUDA.
 */
int arlo_weights_create(int32_t device, const arlo_model_config* cfg,
                        const void* const* tensors, int32_t n_tensors,
                        arlo_weights** out);
void arlo_weights_destroy(arlo_weights* w);

/* ---------------------------------------------------------------- runtime */
typedef struct arlo_runtime arlo_runtime;

/*
 * One statically shaped runtime with max_length L (PAPER.md:L123 step 2
 * "compiled into multiple runtimes, each with a different max_length"; the
 * static (batch, length) shape, L77 §2.1).  Requires 16 <= L <= max_pos,
 * L % 16 == 0, 1 <= max_batch <= 64.  Allocates the activation arena for
 * (max_batch, L) and captures one CUDA graph per batch bucket: embedding+LN,
 * layers x {QKV GEMM, masked attention, out-proj GEMM+residual, LN, FFN1
 * GEMM+GELU, FFN2 GEMM+residual, LN}, CLS pooler + classifier.  Buckets are
 * b in {1, 2, 4} then every multiple of 8 below max_batch, plus max_batch.
 * The runtime uses its own non-blocking stream until arlo_runtime_set_stream.
 * Errors: EINVAL, ENOMEM, ECUDA, ENODEV.
 */
int arlo_runtime_create(int32_t L, int32_t max_batch, const arlo_weights* w, arlo_runtime** out);

/*
 * Runtime families (bf16; fp32 check mode ignores the family: SIMT GEMMs + LayerNorm kernels).
 * Within a family a request's logits are bitwise equal on every runtime L >= its length and in
 * every batch bucket; across families they agree to bf16 rounding (all within 2e-2 of the oracle).
 *  THROUGHPUT (DEFAULT): tcgen05 tile GEMMs (each output element's K chain in one accumulator),
 *    attention, LayerNorm kernels: 3 + 7 * layers kernels per forward.
 *  LATENCY: the paper's batch-1 runtimes (§5).  The same tile GEMMs with every
 *    LayerNorm folded into the GEMMs around it (include/arlo_ops.h arlo_op_gemm_fold): residual
 *    GEMMs emit row statistics, the consuming GEMMs run on gamma-scaled weights and normalise in
 *    their epilogue, no LayerNorm kernel (3 + 5 * layers kernels).  Measured on B200: batch-1
 *    forwards 6-9 % faster than THROUGHPUT; at batch 32 the heavier epilogues cost more than the
 *    LayerNorm launches they replace, hence not the default.
 *  FUSED: see below.
 *  SPLITK: every GEMM a split-K weight-streaming kernel (a cluster of S CTAs per column tile,
 *    S a function of (N, K) only, partials added in a fixed order over distributed shared memory)
 *    + LayerNorm kernels; measured no faster than THROUGHPUT at batch 1.
 */
enum { ARLO_RUNTIME_DEFAULT = 0, ARLO_RUNTIME_LATENCY = 1, ARLO_RUNTIME_THROUGHPUT = 2, ARLO_RUNTIME_FUSED = 3,
       ARLO_RUNTIME_SPLITK = 4 };
/*
 * ARLO_RUNTIME_FUSED: the whole forward (embedding .. logits) as ONE persistent kernel of one
 * CTA per SM running a static task graph (GEMM units, attention per (sequence, head),
 * LayerNorm row groups, head), tasks waiting on per-step completion counters instead of
 * kernel boundaries; weights stream ahead of the dependency chain (the
 * batch-1 setting of PAPER.md:L282 §5).  Needs bf16, max_batch*L <= 256, L <= 128, hidden and
 * ffn multiples of 128, hidden <= 1024 (EINVAL otherwise).  GEMM units split K by a factor of
 * the weight shape only, so within the family a request's logits are bitwise equal on every
 * runtime L >= its length and in every bucket; against the other families they agree to
 * bf16 rounding.  arlo_runtime_gemm_tiles reports 3000 + the split factor of each GEMM.
 */
int arlo_runtime_create_ex(int32_t L, int32_t max_batch, const arlo_weights* w, int32_t family,
                           arlo_runtime** out);
/* The family the runtime was built as (never ARLO_RUNTIME_DEFAULT). */
int32_t arlo_runtime_family(const arlo_runtime* rt);
void arlo_runtime_destroy(arlo_runtime* rt);
/* Launch stream for every later call (a cudaStream_t; NULL = legacy default stream). */
int arlo_runtime_set_stream(arlo_runtime* rt, void* cuda_stream);
int32_t arlo_runtime_length(const arlo_runtime* rt);
int32_t arlo_runtime_max_batch(const arlo_runtime* rt);

/*
 * Run one batch synchronously (returns after the logits are written).
 *   token_ids [max_batch][L] int32, row-major, host or device.
 *   lengths   [max_batch] int32, host or device; n = number of leading
 *             entries > 0; entries from the first 0 on are empty slots.
 *   logits    [max_batch][num_labels] fp32, host or device; rows 0..n-1 are
 *             written (fp32 logits of each request over its real tokens),
 *             later rows are untouched.
 * Ids at positions t >= lengths[i] are ignored (treated as pad id 0), so
 * callers need not zero the padding.  Validation: 1 <= lengths[i] <= L
 * (ETOOLONG if > L), ids at t < lengths[i] in [0, vocab) (EINVAL; device ids
 * are checked by the embedding kernel and reported after the run).
 * Picks the smallest captured bucket b >= n and replays its graph.
 */
int arlo_infer(arlo_runtime* rt, const int32_t* token_ids, const int32_t* lengths, float* logits);

/*
 * Asynchronous form for callers that keep everything on the device (bench,
 * trace replay): enqueue one forward of n requests on the runtime's stream
 * and return without synchronising.  All three pointers are DEVICE memory:
 * token_ids [n][L], lengths [n] (all >= 1 and <= L; NOT validated here),
 * logits [n][num_labels].  Errors: EINVAL, ECUDA.
 */
int arlo_enqueue(arlo_runtime* rt, int32_t n, const int32_t* token_ids, const int32_t* lengths,
                 float* logits);

/* Batch bucket (captured graph size) that serves n requests: the smallest of
 * 1, 2, 4, 6, 8, ..., 32 (every 2), 40, 48, ... (every 8), max_batch that is >= n.
 * EINVAL unless 1 <= n <= max_batch. */
int32_t arlo_runtime_bucket(const arlo_runtime* rt, int32_t n);

/* Number of kernels one forward at bucket b launches (graph node count). */
int32_t arlo_runtime_kernel_count(const arlo_runtime* rt, int32_t n);

/* Tile codes of the four GEMMs (QKV, out-proj, FFN1, FFN2; 0 = not a tensor-core GEMM, e.g.
 * fp32 check mode) captured in the graph serving n requests.  Codes: BN single CTA, -BN CTA
 * pair, 1000 + BN skinny.  bf16 runtimes pick them at create time by timing every valid tile on
 * the device (ARLO_NO_AUTOTUNE=1: the analytic chooser); results are bitwise independent of the
 * tile.  Writes codes[4].  Errors: EINVAL. */
int arlo_runtime_gemm_tiles(const arlo_runtime* rt, int32_t n, int32_t* codes);

/* ------------------------------------------- Runtime Scheduler (host, C++) */
/*
 * Allocation program of PAPER.md:L181-203 (§3.3, Eqs. 1-7):
 *   min  sum_i L_i(B_i) * C_i                                  (Eq. 1)
 *   s.t. sum_i N_i = G                                          (Eq. 2)
 *        N_i >= floor(Q_i / M_i)                                (Eq. 3)
 *        R_0 = 0, R_i = max(R_{i-1} + Q_i - N_i M_i, 0)          (Eq. 4)
 *        C_i = min(R_{i-1} + Q_i, N_i M_i) (i < I), R_{I-1} + Q_I (Eq. 5)
 *        B_i = C_i / N_i                                        (Eq. 6)
 *        N_I >= 1                                               (Eq. 7)
 * G GPUs, I runtimes sorted by ascending max_length; Q[i] mean requests per
 * SLO window in bin i; M[i] max capacity per instance within the SLO;
 * lat[i*nb + (b-1)] profiled mean latency of runtime i at batch b = 1..nb.
 * L_i(B) interpolates lat linearly with B clamped to [1, nb]; a runtime with
 * N_i = 0 contributes 0.  Exact: enumerates every composition of G into I
 * parts (ties: first in lexicographic order).  Writes N_out[I] and
 * *objective_out (may be NULL).  Errors: EINVAL (G < 1, I < 1, nb < 1,
 * M[i] <= 0, or more than 5e7 compositions), EINFEASIBLE.
 */
int arlo_allocate(int32_t G, int32_t I, const double* Q, const double* M, const double* lat,
                  int32_t nb, int32_t* N_out, double* objective_out);

/*
 * Instance replacement (§4): "each time Runtime Scheduler resolves
 * a new allocation, it makes a replacement plan that replaces the minimum number
 * of current runtime instances".  cur[g] = runtime index of GPU g's instance
 * (-1 = none), g < G; N_new[I] = the new allocation (sum <= G).  Writes next[G]
 * (-1 where sum N_new < G) and, if non-NULL, *n_replaced = #{g : next[g] != cur[g]},
 * which is minimal: GPU g keeps cur[g] while that runtime still needs instances
 * (lowest GPU indices first); the missing runtimes, in ascending order, go first
 * to GPUs freed from an oversubscribed runtime, then to idle GPUs.  On B200 a replacement swaps which pre-captured CUDA graphs a
 * GPU replays (the paper's "hot instances pre-loaded in GPU RAM").  Errors:
 * EINVAL (G < 1, I < 1, N_new[i] < 0, sum N_new > G, cur[g] out of range).
 */
int arlo_replace_plan(int32_t G, int32_t I, const int32_t* cur, const int32_t* N_new, int32_t* next,
                      int32_t* n_replaced);

/* ------------------------------------------- Request Scheduler (host, C++) */
typedef struct arlo_sched arlo_sched;

/*
 * Multi-level queue of Fig. 5 / Algorithm 1:
 * K levels (runtimes) sorted by ascending max_len[k]; level k has n_inst[k]
 * instances (may be 0), each with max capacity capacity[k] (> 0) within the
 * SLO.  lambda = initial threshold, alpha = decay, peek = maximum peeking
 * level L (paper defaults 0.85, 0.9, 6).
 * Errors: EINVAL (K < 1, unsorted max_len, capacity <= 0, peek < 1).
 */
int arlo_sched_create(int32_t K, const int32_t* max_len, const int32_t* n_inst,
                      const double* capacity, double lambda, double alpha, int32_t peek,
                      arlo_sched** out);
void arlo_sched_destroy(arlo_sched* s);

/*
 * Algorithm 1 for one arriving request of `length`: candidates = levels with
 * max_len >= length and >= 1 instance (line 2), first `peek` of them (3-5);
 * congestion P = N/M of each candidate's head instance (7-9); choose the first
 * with P < lambda, else lambda *= alpha (10-15); fall back to the first
 * candidate (18-19); dispatch to that level's head instance and update its
 * priority queue (21-22).  Head = least outstanding, lowest id on ties.
 * Writes the chosen level and instance index.  O(peek + log n_inst).
 * Errors: EINVAL (length < 1), ENOCAND.
 */
int arlo_dispatch(arlo_sched* s, int32_t length, int32_t* runtime_out, int32_t* instance_out);

/* Dispatch policy (the Table 4 ablation): ARLO_DISPATCH_RS =
 * Algorithm 1 (default); ARLO_DISPATCH_ILB = Intra-group Load Balance: the
 * runtime requiring the least padding, its least-loaded instance;
 * ARLO_DISPATCH_IG = Inter-groups Greedy: the least busy head instance among
 * ALL candidate runtimes (fewest outstanding requests, ties to the smaller
 * max_length; peek is ignored).  Errors: EINVAL. */
enum { ARLO_DISPATCH_RS = 0, ARLO_DISPATCH_ILB = 1, ARLO_DISPATCH_IG = 2 };
int arlo_sched_set_policy(arlo_sched* s, int32_t policy);

/* Replace lambda, alpha and peek of an existing scheduler (state is kept).
 * Errors: EINVAL (peek < 1). */
int arlo_sched_set_params(arlo_sched* s, double lambda, double alpha, int32_t peek);

/* A request finished on (runtime, instance): outstanding -= 1, heap fix-up.
 * Errors: EINVAL (bad index or outstanding already 0). */
int arlo_complete(arlo_sched* s, int32_t runtime, int32_t instance);

/* Outstanding requests of one instance (>= 0), or a negative error code. */
int32_t arlo_sched_outstanding(const arlo_sched* s, int32_t runtime, int32_t instance);

#ifdef __cplusplus
}
#endif
#endif /* ARLO_H_ */
