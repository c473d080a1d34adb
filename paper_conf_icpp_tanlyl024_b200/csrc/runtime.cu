// runtime.cu — per-length runtime (K9: CUDA-graph runtime builder) and the C ABI.
//
// A runtime is the B200 counterpart of one statically compiled engine of
// Arlo's polymorphing: the model "compiled into multiple runtimes, each with a
// different max_length" (PAPER.md:L123 step 2), one static (batch, length)
// shape each (L77 §2.1).  Here "compile" = allocate a graph-stable activation
// arena for (max_batch, L), encode the TMA descriptors of every GEMM once, and
// capture one CUDA graph per batch bucket b in {1, 2, 4, ..., max_batch}.  A
// request batch is served by copying ids/lengths into the arena and replaying
// the graph of the smallest bucket b >= n (one launch instead of 2 + 7*layers).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "../../include/arlo.h"
#include "../../include/arlo_ops.h"
#include "errors.h"
#include "kernels.h"

namespace arlo {

namespace {
thread_local std::string g_err;
}

int set_error(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}
void clear_error() { g_err.clear(); }

bool pdl_enabled() {
  static const bool on = getenv("ARLO_NO_PDL") == nullptr;
  return on;
}

static int cuda_fail(cudaError_t e, const char* what) {
  return set_error(ARLO_ECUDA, "%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
}

#define ARLO_CUDA(call, what)                    \
  do {                                           \
    cudaError_t e_ = (call);                     \
    if (e_ != cudaSuccess) return cuda_fail(e_, what); \
  } while (0)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

static int check_device(int device) {
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || n <= 0) return set_error(ARLO_ENODEV, "no CUDA device");
  if (device < 0 || device >= n) return set_error(ARLO_ENODEV, "device %d out of range (%d devices)", device, n);
  cudaDeviceProp p;
  if (cudaGetDeviceProperties(&p, device) != cudaSuccess) return set_error(ARLO_ENODEV, "cudaGetDeviceProperties failed");
  if (p.major != 10 || p.minor != 0)
    return set_error(ARLO_ENODEV, "device %d is sm_%d%d; libarlo is built for sm_100a (B200) only", device, p.major,
                     p.minor);
  return ARLO_OK;
}

}  // namespace arlo

using namespace arlo;

// ------------------------------------------------------------------------ weights
// LayerNorm-folded copies of the weights that consume a LayerNorm output (launch_fold_weights):
// per layer l, the QKV projection folded with layer l-1's LN2 (l >= 1) and FFN1 with layer l's LN1.
struct FoldLayer {
  void* wq = nullptr;  // [3H, H] bf16 = W_qkv * gamma2(l-1)
  float* sq = nullptr;  // [3H] row sums of wq
  float* cq = nullptr;  // [3H] W_qkv beta2(l-1) + b_qkv
  void* w1 = nullptr;   // [F, H] bf16 = W_1 * gamma1(l)
  float* s1 = nullptr;
  float* c1 = nullptr;
};

struct arlo_weights {
  int device;
  arlo_model_config cfg;
  std::vector<const void*> t;  // canonical order
  std::mutex fold_mu;          // the fold cache is built once, by the first runtime that needs it
  void* fold_buf = nullptr;
  std::vector<FoldLayer> fold;
  const void* word() const { return t[0]; }
  const void* pos() const { return t[1]; }
  const void* type() const { return t[2]; }
  const float* emb_g() const { return (const float*)t[3]; }
  const float* emb_b() const { return (const float*)t[4]; }
  const void* lt(int layer, int k) const { return t[5 + 12 * layer + k]; }
  const void* hd(int k) const { return t[5 + 12 * cfg.layers + k]; }
};

enum { LW_QKV = 0, LB_QKV, LW_O, LB_O, LN1_G, LN1_B, LW_1, LB_1, LW_2, LB_2, LN2_G, LN2_B };

extern "C" const char* arlo_last_error(void) { return g_err.c_str(); }
extern "C" const char* arlo_version(void) { return "arlo-b200 0.1 (sm_100a)"; }

extern "C" int32_t arlo_weights_count(const arlo_model_config* cfg) {
  return cfg ? 5 + 12 * cfg->layers + 4 : ARLO_EINVAL;
}

static int validate_cfg(const arlo_model_config* c) {
  if (!c) return set_error(ARLO_EINVAL, "null config");
  if (c->layers < 1 || c->hidden < 64 || c->heads < 1 || c->hidden != 64 * c->heads)
    return set_error(ARLO_EINVAL, "config: need hidden == 64 * heads (head dim 64), layers >= 1");
  if (c->hidden % 64 || c->ffn % 64 || c->ffn < 64)
    return set_error(ARLO_EINVAL, "config: hidden and ffn must be multiples of 64");
  if (c->hidden > 2048) return set_error(ARLO_EINVAL, "config: hidden > 2048 unsupported");
  if (c->vocab < 1 || c->max_pos < 16 || c->type_vocab < 1 || c->num_labels < 1 || c->num_labels > 64)
    return set_error(ARLO_EINVAL, "config: bad vocab/max_pos/type_vocab/num_labels");
  if (c->dtype != ARLO_BF16 && c->dtype != ARLO_FP32) return set_error(ARLO_EINVAL, "config: bad dtype");
  if (!(c->ln_eps > 0)) return set_error(ARLO_EINVAL, "config: ln_eps must be > 0");
  return ARLO_OK;
}

extern "C" int arlo_weights_create(int32_t device, const arlo_model_config* cfg, const void* const* tensors,
                                   int32_t n_tensors, arlo_weights** out) {
  clear_error();
  if (!out || !tensors) return set_error(ARLO_EINVAL, "arlo_weights_create: null argument");
  int rc = validate_cfg(cfg);
  if (rc) return rc;
  if (n_tensors != arlo_weights_count(cfg))
    return set_error(ARLO_EINVAL, "arlo_weights_create: expected %d tensors, got %d", arlo_weights_count(cfg), n_tensors);
  if ((rc = check_device(device))) return rc;
  for (int i = 0; i < n_tensors; ++i) {
    if (!tensors[i] || (reinterpret_cast<uintptr_t>(tensors[i]) & 15))
      return set_error(ARLO_EINVAL, "arlo_weights_create: tensor %d is null or not 16-byte aligned", i);
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, tensors[i]) != cudaSuccess || (a.type != cudaMemoryTypeDevice && a.type != cudaMemoryTypeManaged)) {
      cudaGetLastError();
      return set_error(ARLO_EINVAL, "arlo_weights_create: tensor %d is not device memory", i);
    }
  }
  arlo_weights* w = new (std::nothrow) arlo_weights;
  if (!w) return set_error(ARLO_ENOMEM, "out of host memory");
  w->device = device;
  w->cfg = *cfg;
  w->t.assign(tensors, tensors + n_tensors);
  *out = w;
  return ARLO_OK;
}

extern "C" void arlo_weights_destroy(arlo_weights* w) {
  if (w && w->fold_buf) {
    DeviceGuard g(w->device);
    cudaFree(w->fold_buf);
  }
  delete w;
}

// Build the LayerNorm-folded weight copies (once per weight set).  bf16 only.
static int ensure_fold(arlo_weights* w, cudaStream_t s) {
  std::lock_guard<std::mutex> lk(w->fold_mu);
  if (w->fold_buf) return ARLO_OK;
  const arlo_model_config& c = w->cfg;
  const size_t H = c.hidden, F = c.ffn, nl = c.layers;
  auto al = [](size_t x) { return (x + 255) & ~size_t(255); };
  const size_t per = al(6 * H * H) + 3 * al(4 * 3 * H) + al(2 * F * H) + 2 * al(4 * F);
  void* buf = nullptr;
  cudaError_t e = cudaMalloc(&buf, per * nl);
  if (e != cudaSuccess) return set_error(ARLO_ENOMEM, "LayerNorm-fold weights (%zu bytes): %s", per * nl, cudaGetErrorString(e));
  std::vector<FoldLayer> fl(nl);
  for (size_t l = 0; l < nl; ++l) {
    char* p = (char*)buf + per * l;
    FoldLayer& f = fl[l];
    f.wq = p; p += al(6 * H * H);
    f.sq = (float*)p; p += al(4 * 3 * H);
    f.cq = (float*)p; p += al(4 * 3 * H);
    p += al(4 * 3 * H);
    f.w1 = p; p += al(2 * F * H);
    f.s1 = (float*)p; p += al(4 * F);
    f.c1 = (float*)p;
    if (l >= 1)
      e = launch_fold_weights(3 * H, H, w->lt(l, LW_QKV), (const float*)w->lt(l - 1, LN2_G), (const float*)w->lt(l - 1, LN2_B),
                              (const float*)w->lt(l, LB_QKV), f.wq, f.sq, f.cq, s);
    if (e == cudaSuccess)
      e = launch_fold_weights(F, H, w->lt(l, LW_1), (const float*)w->lt(l, LN1_G), (const float*)w->lt(l, LN1_B),
                              (const float*)w->lt(l, LB_1), f.w1, f.s1, f.c1, s);
    if (e != cudaSuccess) break;
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) {
    cudaFree(buf);
    return cuda_fail(e, "LayerNorm-fold weights");
  }
  w->fold_buf = buf;
  w->fold = std::move(fl);
  return ARLO_OK;
}

// ------------------------------------------------------------------------ runtime
struct LayerPlans {
  TcGemmPlan qkv, o, f1, f2;
};

struct Bucket {
  int b = 0;
  std::vector<LayerPlans> plans;  // bf16 only
  // LayerNorm run as the prologue of the GEMM that consumes it (layernorm.cuh): ln1_in_f1[l] =
  // layer l's LN1 runs inside its FFN1 GEMM, ln2_in_qkv[l] = layer l's LN2 inside layer l+1's QKV
  std::vector<char> ln1_in_f1, ln2_in_qkv;
  bool fused_ln = false;          // o / f2 plans carry residual + LayerNorm (no separate LN kernels)
  int tiles[4] = {0, 0, 0, 0};    // measured tile codes of the qkv, o, f1, f2 GEMMs (pick_tile)
  AttnPlan attn;
  // CLS-only last layer (bf16): only position 0 of each sequence feeds the pooler
  // (reading S8), so after the last layer's QKV projection and the attention of
  // q-tile 0, the out-projection, LayerNorms and FFN run on the b CLS rows
  // (A and residual read with row stride L*H, outputs compact [b, H]).  Same
  // K order per row => bitwise the rows the full layer would produce.
  bool cls_prune = false;
  LayerPlans cls;
  AttnPlan attn_cls;
  FusedPlanImpl* fused = nullptr;  // fused family: the whole forward as one persistent kernel
  cudaGraphExec_t exec = nullptr;
  size_t nodes = 0;
};

struct arlo_runtime {
  int L = 0, max_batch = 0, device = 0;
  // split-K family (ARLO_RUNTIME_SPLITK): every GEMM is the split-K weight-streaming kernel
  // (gemm_splitk.cu); the other families use the tile kernels chosen per bucket
  bool latency = false;
  // fused family (ARLO_RUNTIME_FUSED): one persistent kernel per forward (encoder_fused.cu)
  bool fused = false;
  // LayerNorm fold (throughput family, bf16; ARLO_NO_LN_FOLD=1 disables): no LayerNorm kernels;
  // the residual GEMMs emit row statistics (S1 after the out-projection, S2 after FFN2), the
  // consuming GEMMs run on folded weights, the next residual GEMM and the pooler normalise on the fly
  bool ln_fold = false;
  float *S1 = nullptr, *S2 = nullptr;  // [max_batch * L][H/32][2] granule statistics
  arlo_weights* w = nullptr;
  DType dt = DT_BF16;
  cudaStream_t own_stream = nullptr, stream = nullptr;
  // arena (one allocation)
  void* arena = nullptr;
  int32_t* err = nullptr;      // [1]
  int32_t* lengths = nullptr;  // [max_batch]  (err, lengths, ids are contiguous: one staging copy)
  int32_t* ids = nullptr;      // [max_batch * L]
  float* logits = nullptr;     // [max_batch * C]
  float* pooled = nullptr;     // [max_batch * H] fp32 pooler output
  unsigned* gbar = nullptr;    // grid barrier of the LayerNorm-prologue GEMMs (zero-initialised)
  unsigned* head_cnt = nullptr;  // pooler -> classifier arrival counters, one per 8 sequences (zero-initialised)
  void *X = nullptr, *QKV = nullptr, *O = nullptr, *Y = nullptr, *F = nullptr;
  // pinned host staging
  void* h_stage = nullptr;
  size_t h_stage_bytes = 0;
  std::vector<Bucket> buckets;
};

static int bucket_index(const arlo_runtime* rt, int n) {
  for (size_t i = 0; i < rt->buckets.size(); ++i)
    if (rt->buckets[i].b >= n) return (int)i;
  return -1;
}

// Timing experiments only (tools/forward_costs.py): ARLO_DEBUG_SKIP=ln,attn drops those kernels
// from the captured forward (wrong results) so that the forward-time difference is their cost
// inside the graph, where every kernel's prologue overlaps its predecessor (PDL).
static bool debug_skip(const char* what) {
  const char* e = getenv("ARLO_DEBUG_SKIP");
  return e != nullptr && strstr(e, what) != nullptr;
}

// Enqueue one forward at bucket size b (the body every graph captures).
static int enqueue_forward(arlo_runtime* rt, Bucket& bk, cudaStream_t s) {
  const arlo_weights* w = rt->w;
  const arlo_model_config& c = w->cfg;
  const int b = bk.b, L = rt->L, H = c.hidden, F = c.ffn, M = b * L;
  const DType dt = rt->dt;
  if (rt->fused) {
    ARLO_CUDA(fused_launch(bk.fused, s), "fused forward launch");
    return ARLO_OK;
  }
  ARLO_CUDA(launch_embed_ln(dt, b, L, H, c.vocab, rt->ids, rt->lengths, w->word(), w->pos(), w->type(), w->emb_g(),
                            w->emb_b(), c.ln_eps, rt->X, rt->err, s),
            "embed_ln launch");
  if (rt->ln_fold) {
    // LayerNorm fold: 4 GEMMs + attention per layer, no LayerNorm kernel (plans carry the fold)
    for (int l = 0; l < c.layers; ++l) {
      const bool cls = bk.cls_prune && l == c.layers - 1;
      ARLO_CUDA(tc_launch_gemm(bk.plans[l].qkv, s), "qkv gemm launch");
      if (!debug_skip("attn")) ARLO_CUDA(attn_launch(cls ? bk.attn_cls : bk.attn, rt->lengths, rt->O, s), "attention launch");
      const LayerPlans& p = cls ? bk.cls : bk.plans[l];
      ARLO_CUDA(tc_launch_gemm(p.o, s), "out-proj gemm launch");
      ARLO_CUDA(tc_launch_gemm(p.f1, s), "ffn1 gemm launch");
      ARLO_CUDA(tc_launch_gemm(p.f2, s), "ffn2 gemm launch");
    }
    const int l = c.layers - 1;
    HeadLn hl{rt->S2, (const float*)w->lt(l, LN2_G), (const float*)w->lt(l, LN2_B), c.ln_eps, rt->max_batch * L};
    ARLO_CUDA(launch_head(dt, b, bk.cls_prune ? 1 : L, H, c.num_labels, rt->X, w->hd(0), (const float*)w->hd(1),
                          w->hd(2), (const float*)w->hd(3), rt->pooled, rt->logits, s, hl, rt->head_cnt),
              "head launch");
    return ARLO_OK;
  }
  for (int l = 0; l < c.layers; ++l) {
    if (bk.cls_prune && l == c.layers - 1) {
      // last layer on the b CLS rows only (see Bucket::cls_prune)
      ARLO_CUDA(tc_launch_gemm(bk.plans[l].qkv, s), "qkv gemm launch");
      ARLO_CUDA(attn_launch(bk.attn_cls, rt->lengths, rt->O, s), "attention launch (CLS q-tile)");
      ARLO_CUDA(tc_launch_gemm(bk.cls.o, s), "out-proj gemm launch (CLS rows)");
      ARLO_CUDA(launch_layernorm(dt, b, H, rt->Y, (const float*)w->lt(l, LN1_G), (const float*)w->lt(l, LN1_B),
                                 c.ln_eps, rt->X, s),
                "ln1 launch (CLS rows)");
      ARLO_CUDA(tc_launch_gemm(bk.cls.f1, s), "ffn1 gemm launch (CLS rows)");
      ARLO_CUDA(tc_launch_gemm(bk.cls.f2, s), "ffn2 gemm launch (CLS rows)");
      ARLO_CUDA(launch_layernorm(dt, b, H, rt->Y, (const float*)w->lt(l, LN2_G), (const float*)w->lt(l, LN2_B),
                                 c.ln_eps, rt->X, s),
                "ln2 launch (CLS rows)");
      continue;
    }
    if (dt == DT_BF16) {
      ARLO_CUDA(tc_launch_gemm(bk.plans[l].qkv, s), "qkv gemm launch");
    } else {
      ARLO_CUDA(launch_gemm_simt(dt, M, 3 * H, H, rt->X, w->lt(l, LW_QKV), (const float*)w->lt(l, LB_QKV), nullptr,
                                 rt->QKV, EPI_BIAS, s),
                "qkv gemm launch");
    }
    if (!debug_skip("attn")) ARLO_CUDA(attn_launch(bk.attn, rt->lengths, rt->O, s), "attention launch");
    if (dt == DT_BF16) {
      ARLO_CUDA(tc_launch_gemm(bk.plans[l].o, s), "out-proj gemm launch");
    } else {
      ARLO_CUDA(launch_gemm_simt(dt, M, H, H, rt->O, w->lt(l, LW_O), (const float*)w->lt(l, LB_O), rt->X, rt->Y,
                                 EPI_BIAS_RESID, s),
                "out-proj gemm launch");
    }
    if (!bk.fused_ln && !(l < (int)bk.ln1_in_f1.size() && bk.ln1_in_f1[l]) && !debug_skip("ln"))
      ARLO_CUDA(launch_layernorm(dt, M, H, rt->Y, (const float*)w->lt(l, LN1_G), (const float*)w->lt(l, LN1_B),
                                 c.ln_eps, rt->X, s),
                "ln1 launch");
    if (dt == DT_BF16) {
      ARLO_CUDA(tc_launch_gemm(bk.plans[l].f1, s), "ffn1 gemm launch");
      ARLO_CUDA(tc_launch_gemm(bk.plans[l].f2, s), "ffn2 gemm launch");
    } else {
      ARLO_CUDA(launch_gemm_simt(dt, M, F, H, rt->X, w->lt(l, LW_1), (const float*)w->lt(l, LB_1), nullptr, rt->F,
                                 EPI_BIAS_GELU, s),
                "ffn1 gemm launch");
      ARLO_CUDA(launch_gemm_simt(dt, M, H, F, rt->F, w->lt(l, LW_2), (const float*)w->lt(l, LB_2), rt->X, rt->Y,
                                 EPI_BIAS_RESID, s),
                "ffn2 gemm launch");
    }
    if (!bk.fused_ln && !(l < (int)bk.ln2_in_qkv.size() && bk.ln2_in_qkv[l]) && !debug_skip("ln"))
      ARLO_CUDA(launch_layernorm(dt, M, H, rt->Y, (const float*)w->lt(l, LN2_G), (const float*)w->lt(l, LN2_B),
                                 c.ln_eps, rt->X, s),
                "ln2 launch");
  }
  // the pooler reads position 0 of sequence i at row i*L of X, or row i after a CLS-only last layer
  ARLO_CUDA(launch_head(dt, b, bk.cls_prune ? 1 : L, H, c.num_labels, rt->X, w->hd(0), (const float*)w->hd(1), w->hd(2),
                        (const float*)w->hd(3), rt->pooled, rt->logits, s, HeadLn{}, rt->head_cnt),
            "head launch");
  return ARLO_OK;
}

// Build-time tile selection ("tactics", as a TensorRT engine build times its kernels): for one
// GEMM shape of the runtime, time every valid tile code on the runtime's stream (layer-0 buffers,
// 2 warm-up launches, best of 3 rounds of 4) and keep the fastest; the analytic chooser's pick is one of
// the candidates and wins ties.  Every tile code computes each output element with the same K
// chain, so the choice changes time only, never a bit of the result (tile-width bitwise tests).
// ARLO_NO_AUTOTUNE=1 keeps the analytic chooser.
// `only` (optional): time these codes instead, the first one the incumbent (the split-K tile widths
// of the fold family's FFN2, which share one arithmetic whatever the width).
template <typename PlanFn>
static int pick_tile(int M, int N, int K, cudaStream_t s, PlanFn plan, const std::vector<int>* only = nullptr) {
  const int base = only ? (*only)[0] : tc_choose_bn(M, N, K);
  if (getenv("ARLO_NO_AUTOTUNE") != nullptr) return base;
  std::vector<int> cands = {base};
  if (only) {
    cands = *only;
  } else {
    for (int code : {-256, -192, -128, 256, 192, 128, 96, 64})
      if (code != base && N % (code < 0 ? -code : code) == 0) cands.push_back(code);
    if (M <= 1024)
      for (int bn : {16, 32, 64})
        if (kSkinnyCode + bn != base && N % bn == 0) cands.push_back(kSkinnyCode + bn);
  }
  cudaEvent_t e0, e1;
  if (cudaEventCreate(&e0) != cudaSuccess) return base;
  if (cudaEventCreate(&e1) != cudaSuccess) { cudaEventDestroy(e0); return base; }
  int best = base;
  float best_ms = 1e30f;
  // Each candidate: 2 warm-up launches, then the best of 3 rounds of 4 back-to-back launches (the
  // minimum filters out clock ramps and other noise, so the choice repeats from run to run).
  for (int code : cands) {
    TcGemmPlan p;
    if (!plan(&p, code)) continue;
    bool ok = tc_launch_gemm(p, s) == cudaSuccess && tc_launch_gemm(p, s) == cudaSuccess;
    if (!ok) { cudaGetLastError(); continue; }
    float ms = 1e30f;
    for (int round = 0; round < 3 && ok; ++round) {
      cudaEventRecord(e0, s);
      for (int r = 0; r < 4 && ok; ++r) ok = tc_launch_gemm(p, s) == cudaSuccess;
      cudaEventRecord(e1, s);
      if (!ok || cudaEventSynchronize(e1) != cudaSuccess) { ok = false; break; }
      float t = 0.f;
      cudaEventElapsedTime(&t, e0, e1);
      ms = t < ms ? t : ms;
    }
    if (!ok) { cudaGetLastError(); continue; }
    if (ms < best_ms * 0.98f) { best_ms = ms; best = code; }  // a candidate must beat the incumbent by 2 %
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return best;
}

// Latency family: the four GEMMs of every layer (and of the CLS-only last layer) as split-K
// weight-streaming GEMMs; the split factor depends on (N, K) only (cross-L bitwise within
// the family), the tile width on M.
static int plan_bucket_latency(arlo_runtime* rt, Bucket& bk) {
  const arlo_weights* w = rt->w;
  const arlo_model_config& c = w->cfg;
  const int b = bk.b, L = rt->L, M = b * L, H = c.hidden, F = c.ffn;
  bk.plans.resize(c.layers);
  bk.fused_ln = false;
  for (int l = 0; l < c.layers; ++l) {
    LayerPlans& p = bk.plans[l];
    const bool ok =
        tc_plan_gemm_splitk(&p.qkv, M, 3 * H, H, rt->X, H, w->lt(l, LW_QKV), (const float*)w->lt(l, LB_QKV), nullptr,
                            3 * H, rt->QKV, EPI_BIAS) &&
        tc_plan_gemm_splitk(&p.o, M, H, H, rt->O, H, w->lt(l, LW_O), (const float*)w->lt(l, LB_O), rt->X, H, rt->Y,
                            EPI_BIAS_RESID) &&
        tc_plan_gemm_splitk(&p.f1, M, F, H, rt->X, H, w->lt(l, LW_1), (const float*)w->lt(l, LB_1), nullptr, F,
                            rt->F, EPI_BIAS_GELU) &&
        tc_plan_gemm_splitk(&p.f2, M, H, F, rt->F, F, w->lt(l, LW_2), (const float*)w->lt(l, LB_2), rt->X, H, rt->Y,
                            EPI_BIAS_RESID);
    if (!ok) return set_error(ARLO_ECUDA, "split-K plan: tensor-map encoding failed");
  }
  const LayerPlans& p0 = bk.plans[0];
  bk.tiles[0] = kSplitKCode + p0.qkv.BN; bk.tiles[1] = kSplitKCode + p0.o.BN;
  bk.tiles[2] = kSplitKCode + p0.f1.BN; bk.tiles[3] = kSplitKCode + p0.f2.BN;
  bk.cls_prune = getenv("ARLO_NO_CLS_PRUNE") == nullptr;
  if (bk.cls_prune) {
    const int l = c.layers - 1;
    const bool ok =
        attn_plan(&bk.attn_cls, rt->dt, b, L, c.heads, rt->QKV, 1) &&
        tc_plan_gemm_splitk(&bk.cls.o, b, H, H, rt->O, L * H, w->lt(l, LW_O), (const float*)w->lt(l, LB_O), rt->X,
                            L * H, rt->Y, EPI_BIAS_RESID) &&
        tc_plan_gemm_splitk(&bk.cls.f1, b, F, H, rt->X, H, w->lt(l, LW_1), (const float*)w->lt(l, LB_1), nullptr, F,
                            rt->F, EPI_BIAS_GELU) &&
        tc_plan_gemm_splitk(&bk.cls.f2, b, H, F, rt->F, F, w->lt(l, LW_2), (const float*)w->lt(l, LB_2), rt->X, H,
                            rt->Y, EPI_BIAS_RESID);
    if (!ok) return set_error(ARLO_ECUDA, "CLS-row split-K plan: tensor-map encoding failed");
  }
  return ARLO_OK;
}

// LayerNorm-fold plans (see arlo_runtime::ln_fold).  Per layer l:
//   QKV:  l = 0 plain on x (the embedding LayerNorm's output); l >= 1 EPI_LNFOLD on y2(l-1) (X) with the
//         folded weights of LN2(l-1) and statistics S2
//   out:  EPI_RESID_LN, residual X = y2(l-1) normalised on the fly with LN2(l-1) and S2 (plain x for
//         l = 0) -> y1 (Y) and its statistics S1
//   FFN1: EPI_LNFOLD_GELU on y1 with the folded weights of LN1(l) and S1 -> F
//   FFN2: EPI_RESID_LN, residual y1 normalised with LN1(l) and S1 -> y2(l) (X) and S2
// The pooler normalises the CLS rows of y2(last) with LN2(last) and S2.
static int plan_bucket_fold(arlo_runtime* rt, Bucket& bk) {
  arlo_weights* w = rt->w;
  const arlo_model_config& c = w->cfg;
  const int b = bk.b, L = rt->L, M = b * L, H = c.hidden, F = c.ffn;
  const float eps = c.ln_eps;
  bk.plans.resize(c.layers);
  bk.fused_ln = false;
  const FoldLayer& f0 = w->fold[c.layers > 1 ? 1 : 0];
  cudaStream_t ts = rt->own_stream;
  // tile codes timed on layer 0's shapes (the folded epilogues' costs)
  const int t_qkv = pick_tile(M, 3 * H, H, ts, [&](TcGemmPlan* p, int code) {
    return tc_plan_gemm(p, M, 3 * H, H, rt->X, c.layers > 1 ? f0.wq : w->lt(0, LW_QKV),
                        c.layers > 1 ? f0.sq : (const float*)w->lt(0, LB_QKV), nullptr, rt->QKV,
                        c.layers > 1 ? EPI_LNFOLD : EPI_BIAS, code); });
  const int t_f1 = pick_tile(M, F, H, ts, [&](TcGemmPlan* p, int code) {
    return tc_plan_gemm(p, M, F, H, rt->Y, w->fold[0].w1, w->fold[0].s1, nullptr, rt->F, EPI_LNFOLD_GELU, code); });
  const int t_o = pick_tile(M, H, H, ts, [&](TcGemmPlan* p, int code) {
    return tc_plan_gemm(p, M, H, H, rt->O, w->lt(0, LW_O), (const float*)w->lt(0, LB_O), rt->X, rt->Y, EPI_RESID_LN,
                        code); });
  // FFN2 (K = 4H: the longest K chain, 4H/16 MMAs per output tile) runs split-K: S = f(N, K)
  // CTAs per column tile, partials reduced in a fixed order; its arithmetic is the same at every M,
  // so it holds for every runtime and bucket of the family, the CLS rows included.
  // ARLO_FOLD_FFN2_TILE=1 keeps the tile kernels (A/B).
  std::vector<int> sk_codes;
  if (getenv("ARLO_FOLD_FFN2_TILE") == nullptr)
    for (int bn : {64, 32, 128, 192})  // (BN = 192: M = 512 in 16 clusters, within one wave of 6-CTA clusters)
      if (H % bn == 0) sk_codes.push_back(kSplitKCode + bn);
  const bool f2_splitk = !sk_codes.empty();
  const int t_f2 = pick_tile(M, H, F, ts, [&](TcGemmPlan* p, int code) {
    return tc_plan_gemm(p, M, H, F, rt->F, w->lt(0, LW_2), (const float*)w->lt(0, LB_2), rt->Y, rt->X, EPI_RESID_LN,
                        code); }, f2_splitk ? &sk_codes : nullptr);
  if (cudaStreamSynchronize(ts) != cudaSuccess) return set_error(ARLO_ECUDA, "tile selection failed");
  bk.tiles[0] = t_qkv; bk.tiles[1] = t_o; bk.tiles[2] = t_f1; bk.tiles[3] = t_f2;
  auto ln_g = [&](int l, int k) { return (const float*)w->lt(l, k); };
  for (int l = 0; l < c.layers; ++l) {
    LayerPlans& p = bk.plans[l];
    const FoldLayer& f = w->fold[l];
    bool ok = l == 0 ? tc_plan_gemm(&p.qkv, M, 3 * H, H, rt->X, w->lt(0, LW_QKV), (const float*)w->lt(0, LB_QKV),
                                    nullptr, rt->QKV, EPI_BIAS, t_qkv)
                     : tc_plan_gemm(&p.qkv, M, 3 * H, H, rt->X, f.wq, f.sq, nullptr, rt->QKV, EPI_LNFOLD, t_qkv);
    ok = ok &&
         tc_plan_gemm(&p.o, M, H, H, rt->O, w->lt(l, LW_O), (const float*)w->lt(l, LB_O), rt->X, rt->Y, EPI_RESID_LN, t_o) &&
         tc_plan_gemm(&p.f1, M, F, H, rt->Y, f.w1, f.s1, nullptr, rt->F, EPI_LNFOLD_GELU, t_f1) &&
         tc_plan_gemm(&p.f2, M, H, F, rt->F, w->lt(l, LW_2), (const float*)w->lt(l, LB_2), rt->Y, rt->X, EPI_RESID_LN, t_f2);
    if (!ok) return set_error(ARLO_ECUDA, "LayerNorm-fold plan: tensor-map encoding failed");
    if (l >= 1) p.qkv.fold = FoldArgs{f.cq, nullptr, rt->S2, 1, nullptr, eps, rt->max_batch * rt->L};
    p.o.fold = FoldArgs{l >= 1 ? ln_g(l - 1, LN2_G) : nullptr, l >= 1 ? ln_g(l - 1, LN2_B) : nullptr,
                        l >= 1 ? rt->S2 : nullptr, 1, rt->S1, eps, rt->max_batch * rt->L};
    p.f1.fold = FoldArgs{f.c1, nullptr, rt->S1, 1, nullptr, eps, rt->max_batch * rt->L};
    p.f2.fold = FoldArgs{ln_g(l, LN1_G), ln_g(l, LN1_B), rt->S1, 1, rt->S2, eps, rt->max_batch * rt->L};
  }
  bk.cls_prune = getenv("ARLO_NO_CLS_PRUNE") == nullptr;
  if (bk.cls_prune) {
    // last layer on the b CLS rows: out-projection reads rows i*L of the context and of X (and of
    // S2); everything after it is compact [b, .]
    const int l = c.layers - 1;
    const FoldLayer& f = w->fold[l];
    const bool ok =
        attn_plan(&bk.attn_cls, rt->dt, b, L, c.heads, rt->QKV, 1) &&
        tc_plan_gemm_strided(&bk.cls.o, b, H, H, rt->O, L * H, w->lt(l, LW_O), (const float*)w->lt(l, LB_O), rt->X,
                             L * H, rt->Y, EPI_RESID_LN, 0) &&
        tc_plan_gemm(&bk.cls.f1, b, F, H, rt->Y, f.w1, f.s1, nullptr, rt->F, EPI_LNFOLD_GELU, 0) &&
        tc_plan_gemm(&bk.cls.f2, b, H, F, rt->F, w->lt(l, LW_2), (const float*)w->lt(l, LB_2), rt->Y, rt->X,
                     EPI_RESID_LN, f2_splitk ? kSplitKCode + (H % 64 == 0 ? 64 : 32) : 0);
    if (!ok) return set_error(ARLO_ECUDA, "CLS-row LayerNorm-fold plan: tensor-map encoding failed");
    bk.cls.o.fold = FoldArgs{l >= 1 ? ln_g(l - 1, LN2_G) : nullptr, l >= 1 ? ln_g(l - 1, LN2_B) : nullptr,
                             l >= 1 ? rt->S2 : nullptr, L, rt->S1, eps, rt->max_batch * rt->L};
    bk.cls.f1.fold = FoldArgs{f.c1, nullptr, rt->S1, 1, nullptr, eps, rt->max_batch * rt->L};
    bk.cls.f2.fold = FoldArgs{ln_g(l, LN1_G), ln_g(l, LN1_B), rt->S1, 1, rt->S2, eps, rt->max_batch * rt->L};
  }
  return ARLO_OK;
}

static int plan_bucket(arlo_runtime* rt, Bucket& bk) {
  if (rt->latency) return plan_bucket_latency(rt, bk);
  if (rt->ln_fold) return plan_bucket_fold(rt, bk);
  const arlo_weights* w = rt->w;
  const arlo_model_config& c = w->cfg;
  const int M = bk.b * rt->L, H = c.hidden, F = c.ffn;
  bk.plans.resize(c.layers);
  // Residual + LayerNorm fused into the out-proj / FFN2 GEMM epilogues (cluster
  // row statistics).  Opt-in (ARLO_FUSED_LN=1): measured slower than GEMM + LN
  // kernel on B200 in round 1 (one tile per CTA leaves its three-pass epilogue
  // exposed; small M runs on N/BN CTAs only), see DESIGN.md.
  TcGemmPlan probe;
  bk.fused_ln = getenv("ARLO_FUSED_LN") != nullptr &&
                tc_plan_gemm_ln(&probe, M, H, H, rt->O, w->lt(0, LW_O), (const float*)w->lt(0, LB_O), rt->X,
                                (const float*)w->lt(0, LN1_G), (const float*)w->lt(0, LN1_B), c.ln_eps, rt->X);
  // one tile code per GEMM shape of this bucket, measured on layer 0's buffers
  cudaStream_t ts = rt->own_stream;
  const int t_qkv = pick_tile(M, 3 * H, H, ts, [&](TcGemmPlan* p, int code) {
    return tc_plan_gemm(p, M, 3 * H, H, rt->X, w->lt(0, LW_QKV), (const float*)w->lt(0, LB_QKV), nullptr, rt->QKV,
                        EPI_BIAS, code); });
  const int t_f1 = pick_tile(M, F, H, ts, [&](TcGemmPlan* p, int code) {
    return tc_plan_gemm(p, M, F, H, rt->X, w->lt(0, LW_1), (const float*)w->lt(0, LB_1), nullptr, rt->F,
                        EPI_BIAS_GELU, code); });
  const int t_o = bk.fused_ln ? 0 : pick_tile(M, H, H, ts, [&](TcGemmPlan* p, int code) {
    return tc_plan_gemm(p, M, H, H, rt->O, w->lt(0, LW_O), (const float*)w->lt(0, LB_O), rt->X, rt->Y,
                        EPI_BIAS_RESID, code); });
  const int t_f2 = bk.fused_ln ? 0 : pick_tile(M, H, F, ts, [&](TcGemmPlan* p, int code) {
    return tc_plan_gemm(p, M, H, F, rt->F, w->lt(0, LW_2), (const float*)w->lt(0, LB_2), rt->X, rt->Y,
                        EPI_BIAS_RESID, code); });
  if (cudaStreamSynchronize(ts) != cudaSuccess) return set_error(ARLO_ECUDA, "tile selection failed");
  bk.tiles[0] = t_qkv; bk.tiles[1] = t_o; bk.tiles[2] = t_f1; bk.tiles[3] = t_f2;
  for (int l = 0; l < c.layers; ++l) {
    LayerPlans& p = bk.plans[l];
    bool ok = tc_plan_gemm(&p.qkv, M, 3 * H, H, rt->X, w->lt(l, LW_QKV), (const float*)w->lt(l, LB_QKV), nullptr,
                           rt->QKV, EPI_BIAS, t_qkv) &&
              tc_plan_gemm(&p.f1, M, F, H, rt->X, w->lt(l, LW_1), (const float*)w->lt(l, LB_1), nullptr, rt->F,
                           EPI_BIAS_GELU, t_f1);
    if (bk.fused_ln) {
      ok = ok &&
           tc_plan_gemm_ln(&p.o, M, H, H, rt->O, w->lt(l, LW_O), (const float*)w->lt(l, LB_O), rt->X,
                           (const float*)w->lt(l, LN1_G), (const float*)w->lt(l, LN1_B), c.ln_eps, rt->X) &&
           tc_plan_gemm_ln(&p.f2, M, H, F, rt->F, w->lt(l, LW_2), (const float*)w->lt(l, LB_2), rt->X,
                           (const float*)w->lt(l, LN2_G), (const float*)w->lt(l, LN2_B), c.ln_eps, rt->X);
    } else {
      ok = ok &&
           tc_plan_gemm(&p.o, M, H, H, rt->O, w->lt(l, LW_O), (const float*)w->lt(l, LB_O), rt->X, rt->Y,
                        EPI_BIAS_RESID, t_o) &&
           tc_plan_gemm(&p.f2, M, H, F, rt->F, w->lt(l, LW_2), (const float*)w->lt(l, LB_2), rt->X, rt->Y,
                        EPI_BIAS_RESID, t_f2);
    }
    if (!ok) return set_error(ARLO_ECUDA, "tensor-map encoding failed (cuTensorMapEncodeTiled unavailable?)");
  }
  // LayerNorm prologues: LN1 of layer l into its FFN1, LN2 of layer l into layer l+1's QKV, where
  // that GEMM is a persistent tile kernel (every CTA resident: its grid barrier needs it)
  bk.ln1_in_f1.assign(c.layers, 0);
  bk.ln2_in_qkv.assign(c.layers, 0);
  // Opt-in (ARLO_LN_PROLOGUE=1): bitwise the LN kernel + GEMM, but measured slower on B200 (BERT-base
  // L=128 b=32 0.975 -> 1.063 ms, L=64 b=32 0.683 -> 0.736 ms): the grid barrier and
  // the grid's 1,500-2,000 warps normalising 2-3 rows each cost more than the LN kernel, whose
  // 4,096 warps run one row each and overlap the GEMMs on either side through PDL.
  if (!bk.fused_ln && getenv("ARLO_LN_PROLOGUE") != nullptr) {
    for (int l = 0; l < c.layers; ++l) {
      const bool cls_last = getenv("ARLO_NO_CLS_PRUNE") == nullptr && l == c.layers - 1;  // (CLS rows: LN kernel)
      LnPrologue ln1{rt->Y, (const float*)w->lt(l, LN1_G), (const float*)w->lt(l, LN1_B), rt->X, rt->gbar,
                     c.ln_eps, M, H};
      if (!cls_last) bk.ln1_in_f1[l] = tc_plan_attach_ln(&bk.plans[l].f1, ln1);
      if (l + 1 < c.layers) {
        LnPrologue ln2{rt->Y, (const float*)w->lt(l, LN2_G), (const float*)w->lt(l, LN2_B), rt->X, rt->gbar,
                       c.ln_eps, M, H};
        bk.ln2_in_qkv[l] = tc_plan_attach_ln(&bk.plans[l + 1].qkv, ln2);
      }
    }
  }
  bk.cls_prune = !bk.fused_ln && getenv("ARLO_NO_CLS_PRUNE") == nullptr;
  if (bk.cls_prune) {
    const int l = c.layers - 1, b = bk.b, L = rt->L;
    // out-proj: A = O rows {i*L}, residual = X rows {i*L}, y -> Y[0:b]; LN1 -> X[0:b];
    // FFN1: X[0:b] -> F[0:b]; FFN2: F[0:b], residual X[0:b] -> Y[0:b]; LN2 -> X[0:b]
    const bool ok =
        attn_plan(&bk.attn_cls, rt->dt, b, L, c.heads, rt->QKV, 1) &&
        tc_plan_gemm_strided(&bk.cls.o, b, H, H, rt->O, L * H, w->lt(l, LW_O), (const float*)w->lt(l, LB_O), rt->X,
                             L * H, rt->Y, EPI_BIAS_RESID, 0) &&
        tc_plan_gemm(&bk.cls.f1, b, F, H, rt->X, w->lt(l, LW_1), (const float*)w->lt(l, LB_1), nullptr, rt->F,
                     EPI_BIAS_GELU, 0) &&
        tc_plan_gemm(&bk.cls.f2, b, H, F, rt->F, w->lt(l, LW_2), (const float*)w->lt(l, LB_2), rt->X, rt->Y,
                     EPI_BIAS_RESID, 0);
    if (!ok) return set_error(ARLO_ECUDA, "CLS-row plan: tensor-map encoding failed");
  }
  return ARLO_OK;
}

static void destroy_runtime(arlo_runtime* rt) {
  if (!rt) return;
  for (auto& bk : rt->buckets) {
    if (bk.exec) cudaGraphExecDestroy(bk.exec);
    fused_destroy(bk.fused);
  }
  if (rt->arena) cudaFree(rt->arena);
  if (rt->h_stage) cudaFreeHost(rt->h_stage);
  if (rt->own_stream) cudaStreamDestroy(rt->own_stream);
  delete rt;
}

extern "C" int arlo_runtime_gemm_tiles(const arlo_runtime* rt, int32_t n, int32_t* codes) {
  if (!rt || !codes) return set_error(ARLO_EINVAL, "arlo_runtime_gemm_tiles: null argument");
  const int k = bucket_index(rt, n);
  if (k < 0) return set_error(ARLO_EINVAL, "arlo_runtime_gemm_tiles: n = %d exceeds max_batch", n);
  for (int i = 0; i < 4; ++i) codes[i] = rt->buckets[k].tiles[i];
  return ARLO_OK;
}

extern "C" int arlo_runtime_create(int32_t L, int32_t max_batch, const arlo_weights* w, arlo_runtime** out) {
  return arlo_runtime_create_ex(L, max_batch, w, ARLO_RUNTIME_DEFAULT, out);
}

extern "C" int32_t arlo_runtime_family(const arlo_runtime* rt) {
  return rt ? (rt->fused ? (int32_t)ARLO_RUNTIME_FUSED : rt->latency ? (int32_t)ARLO_RUNTIME_SPLITK
                : rt->ln_fold ? (int32_t)ARLO_RUNTIME_LATENCY : (int32_t)ARLO_RUNTIME_THROUGHPUT)
            : ARLO_EINVAL;
}

extern "C" int arlo_runtime_create_ex(int32_t L, int32_t max_batch, const arlo_weights* w, int32_t family,
                                      arlo_runtime** out) {
  clear_error();
  if (!w || !out) return set_error(ARLO_EINVAL, "arlo_runtime_create: null argument");
  if (family != ARLO_RUNTIME_DEFAULT && family != ARLO_RUNTIME_LATENCY && family != ARLO_RUNTIME_THROUGHPUT &&
      family != ARLO_RUNTIME_FUSED && family != ARLO_RUNTIME_SPLITK)
    return set_error(ARLO_EINVAL, "arlo_runtime_create_ex: unknown runtime family %d", family);
  const arlo_model_config& c = w->cfg;
  if (L < 16 || L % 16 || L > c.max_pos)
    return set_error(ARLO_EINVAL, "arlo_runtime_create: need 16 <= L <= max_pos (%d) and L %% 16 == 0, got %d", c.max_pos, L);
  if (max_batch < 1 || max_batch > 64) return set_error(ARLO_EINVAL, "arlo_runtime_create: need 1 <= max_batch <= 64");
  if (family == ARLO_RUNTIME_FUSED &&
      (c.dtype != ARLO_BF16 || !fused_supported(max_batch, L, c.hidden, c.heads, c.ffn)))
    return set_error(ARLO_EINVAL,
                     "arlo_runtime_create_ex: the fused family needs bf16, max_batch*L <= 256, L <= 128, "
                     "hidden and ffn multiples of 128, hidden <= 1024 (got L=%d max_batch=%d H=%d F=%d)",
                     L, max_batch, c.hidden, c.ffn);
  DeviceGuard g(w->device);
  arlo_runtime* rt = new (std::nothrow) arlo_runtime;
  if (!rt) return set_error(ARLO_ENOMEM, "out of host memory");
  rt->L = L;
  rt->max_batch = max_batch;
  rt->w = const_cast<arlo_weights*>(w);  // (the LayerNorm-fold cache is built lazily inside it)
  rt->device = w->device;
  rt->dt = c.dtype == ARLO_BF16 ? DT_BF16 : DT_FP32;
  // batch-1 runtimes (the paper's setting) stream weights with split-K GEMMs
  // (DEFAULT = THROUGHPUT: measured on B200, the split-K family does not shorten a batch-1 forward;
  // its 87 dependent kernels cost ~4.5 us each whatever the GEMM kernel)
  rt->latency = rt->dt == DT_BF16 && family == ARLO_RUNTIME_SPLITK;
  rt->fused = family == ARLO_RUNTIME_FUSED;
  // LATENCY family = the LayerNorm fold (ARLO_LN_FOLD=1 applies it to the THROUGHPUT family too, A/B)
  rt->ln_fold = rt->dt == DT_BF16 && (family == ARLO_RUNTIME_LATENCY || getenv("ARLO_LN_FOLD") != nullptr) &&
                !rt->latency && !rt->fused && c.hidden % 32 == 0;
  auto fail = [&](int code) { destroy_runtime(rt); return code; };
  cudaError_t e = cudaStreamCreateWithFlags(&rt->own_stream, cudaStreamNonBlocking);
  if (e != cudaSuccess) return fail(cuda_fail(e, "cudaStreamCreate"));
  rt->stream = rt->own_stream;

  const size_t es = rt->dt == DT_BF16 ? 2 : 4;
  const size_t Mmax = (size_t)max_batch * L, H = c.hidden, F = c.ffn;
  auto al = [](size_t x) { return (x + 255) & ~size_t(255); };
  const size_t off_err = 0;
  const size_t off_len = 16;  // err (int32) then lengths then ids, contiguous
  const size_t off_ids = off_len + 4 * (size_t)max_batch;
  size_t off = al(off_ids + 4 * Mmax);
  const size_t off_logits = off; off = al(off + 4 * (size_t)max_batch * c.num_labels);
  const size_t off_pooled = off; off = al(off + 4 * (size_t)max_batch * H);
  const size_t off_gbar = off; off = al(off + 64);
  const size_t off_hcnt = off; off = al(off + 4 * (size_t)((max_batch + 7) / 8));
  const size_t off_X = off; off = al(off + es * Mmax * H);
  const size_t off_QKV = off; off = al(off + es * Mmax * 3 * H);
  const size_t off_O = off; off = al(off + es * Mmax * H);
  const size_t off_Y = off; off = al(off + es * Mmax * H);
  const size_t off_F = off; off = al(off + es * Mmax * F);
  const size_t st_bytes = rt->ln_fold ? 4 * Mmax * (H / 32) * 2 : 0;
  const size_t off_S1 = off; off = al(off + st_bytes);
  const size_t off_S2 = off; off = al(off + st_bytes);
  e = cudaMalloc(&rt->arena, off);
  if (e != cudaSuccess) return fail(set_error(ARLO_ENOMEM, "arena of %zu bytes: %s", off, cudaGetErrorString(e)));
  e = cudaMemset(rt->arena, 0, off);
  if (e != cudaSuccess) return fail(cuda_fail(e, "arena memset"));
  char* a = (char*)rt->arena;
  rt->err = (int32_t*)(a + off_err);
  rt->lengths = (int32_t*)(a + off_len);
  rt->ids = (int32_t*)(a + off_ids);
  rt->logits = (float*)(a + off_logits);
  rt->pooled = (float*)(a + off_pooled);
  rt->gbar = (unsigned*)(a + off_gbar);
  // classifier in the pooler's last CTA (ARLO_HEAD_IN_POOLER=1): bitwise the same logits, one launch
  // less, but measured no faster (the last CTA's serial classifier costs what the hop saved)
  rt->head_cnt = getenv("ARLO_HEAD_IN_POOLER") ? (unsigned*)(a + off_hcnt) : nullptr;
  rt->X = a + off_X; rt->QKV = a + off_QKV; rt->O = a + off_O; rt->Y = a + off_Y; rt->F = a + off_F;
  if (rt->ln_fold) {
    rt->S1 = (float*)(a + off_S1);
    rt->S2 = (float*)(a + off_S2);
    const int rc = ensure_fold(rt->w, rt->own_stream);
    if (rc) return fail(rc);
  }
  rt->h_stage_bytes = off_ids + 4 * Mmax + 4 * (size_t)max_batch * c.num_labels + 64;
  e = cudaMallocHost(&rt->h_stage, rt->h_stage_bytes);
  if (e != cudaSuccess) return fail(set_error(ARLO_ENOMEM, "pinned staging: %s", cudaGetErrorString(e)));

  // batch buckets 1, 2, 4, then every multiple of `step` (2) up to 32 and of 8 beyond, and max_batch:
  // a partly filled batch pads to at most step - 1 empty slots below 32 (7 above).  The padded slots
  // are computed for nothing (the batch dimension's padding waste); round 1's
  // multiples of 8 left up to 7 (e.g. 17 requests in a 24 bucket).  ARLO_BUCKET_STEP=4 / 8: coarser.
  std::vector<int> bs;
  int step = 2;
  if (const char* e = getenv("ARLO_BUCKET_STEP")) step = atoi(e) >= 1 ? atoi(e) : 2;
  if (getenv("ARLO_BUCKET_STEP8")) step = 8;
  for (int b = 1; b < max_batch && b <= 4; b *= 2) bs.push_back(b);
  for (int b = step < 4 ? 4 + step : 8; b < max_batch; b += (b < 32 ? step : 8)) bs.push_back(b);
  bs.push_back(max_batch);
  rt->buckets.resize(bs.size());
  for (size_t i = 0; i < bs.size(); ++i) {
    Bucket& bk = rt->buckets[i];
    bk.b = bs[i];
    if (!attn_plan(&bk.attn, rt->dt, bk.b, L, c.heads, rt->QKV))
      return fail(set_error(ARLO_EINVAL, "attention plan failed (bf16 attention needs L <= 512)"));
    if (rt->fused) {
      bk.fused = fused_create(bk.b, L, c.layers, c.hidden, c.heads, c.ffn, c.num_labels, c.vocab, c.ln_eps,
                              w->t.data(), rt->ids, rt->lengths, rt->err, rt->X, rt->Y, rt->QKV, rt->O, rt->F,
                              rt->pooled, rt->logits);
      if (!bk.fused) return fail(set_error(ARLO_ECUDA, "fused forward plan failed (tensor maps / device memory)"));
      bk.tiles[0] = kFusedCode + 1; bk.tiles[1] = kFusedCode + fused_split(c.hidden, c.hidden);
      bk.tiles[2] = kFusedCode + 1; bk.tiles[3] = kFusedCode + fused_split(c.hidden, c.ffn);
    } else if (rt->dt == DT_BF16) {
      int rc = plan_bucket(rt, bk);
      if (rc) return fail(rc);
    }
    cudaGraph_t graph = nullptr;
    e = cudaStreamBeginCapture(rt->own_stream, cudaStreamCaptureModeThreadLocal);
    if (e != cudaSuccess) return fail(cuda_fail(e, "cudaStreamBeginCapture"));
    int rc = enqueue_forward(rt, bk, rt->own_stream);
    cudaError_t e2 = cudaStreamEndCapture(rt->own_stream, &graph);
    if (rc) { if (graph) cudaGraphDestroy(graph); return fail(rc); }
    if (e2 != cudaSuccess) return fail(cuda_fail(e2, "cudaStreamEndCapture"));
    cudaGraphGetNodes(graph, nullptr, &bk.nodes);
    e = cudaGraphInstantiate(&bk.exec, graph, 0);
    cudaGraphDestroy(graph);
    if (e != cudaSuccess) return fail(cuda_fail(e, "cudaGraphInstantiate"));
    e = cudaGraphUpload(bk.exec, rt->own_stream);
    if (e != cudaSuccess) return fail(cuda_fail(e, "cudaGraphUpload"));
  }
  e = cudaStreamSynchronize(rt->own_stream);
  if (e != cudaSuccess) return fail(cuda_fail(e, "runtime create sync"));
  *out = rt;
  return ARLO_OK;
}

extern "C" void arlo_runtime_destroy(arlo_runtime* rt) {
  if (!rt) return;
  DeviceGuard g(rt->device);
  cudaStreamSynchronize(rt->stream);
  destroy_runtime(rt);
}

extern "C" int arlo_runtime_set_stream(arlo_runtime* rt, void* stream) {
  if (!rt) return set_error(ARLO_EINVAL, "null runtime");
  rt->stream = (cudaStream_t)stream;  // NULL = the legacy default stream
  return ARLO_OK;
}

extern "C" int32_t arlo_runtime_length(const arlo_runtime* rt) { return rt ? rt->L : ARLO_EINVAL; }
extern "C" int32_t arlo_runtime_max_batch(const arlo_runtime* rt) { return rt ? rt->max_batch : ARLO_EINVAL; }

extern "C" int32_t arlo_runtime_bucket(const arlo_runtime* rt, int32_t n) {
  if (!rt || n < 1 || n > rt->max_batch) return ARLO_EINVAL;
  return rt->buckets[bucket_index(rt, n)].b;
}

extern "C" int32_t arlo_runtime_kernel_count(const arlo_runtime* rt, int32_t n) {
  if (!rt) return ARLO_EINVAL;
  int bi = bucket_index(rt, n < 1 ? 1 : n);
  return bi < 0 ? ARLO_EINVAL : (int32_t)rt->buckets[bi].nodes;
}

static bool is_device_ptr(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

extern "C" int arlo_infer(arlo_runtime* rt, const int32_t* token_ids, const int32_t* lengths, float* logits) {
  clear_error();
  if (!rt || !token_ids || !lengths || !logits) return set_error(ARLO_EINVAL, "arlo_infer: null argument");
  DeviceGuard g(rt->device);
  const int L = rt->L, mb = rt->max_batch, C = rt->w->cfg.num_labels, V = rt->w->cfg.vocab;
  cudaStream_t s = rt->stream;
  const bool ids_dev = is_device_ptr(token_ids), len_dev = is_device_ptr(lengths), out_dev = is_device_ptr(logits);
  // staging layout mirrors the arena: [err(16 B) | lengths[mb] | ids[mb*L] | logits[mb*C]]
  char* hs = (char*)rt->h_stage;
  int32_t* h_err = (int32_t*)hs;
  int32_t* h_len = (int32_t*)(hs + 16);
  int32_t* h_ids = h_len + mb;
  float* h_logits = (float*)(h_ids + (size_t)mb * L);
  if (len_dev) {
    ARLO_CUDA(cudaMemcpyAsync(h_len, lengths, 4 * (size_t)mb, cudaMemcpyDeviceToHost, s), "lengths D2H");
    ARLO_CUDA(cudaStreamSynchronize(s), "lengths sync");
  } else {
    memcpy(h_len, lengths, 4 * (size_t)mb);
  }
  int n = 0;
  while (n < mb && h_len[n] > 0) ++n;
  for (int i = 0; i < n; ++i)
    if (h_len[i] > L) return set_error(ARLO_ETOOLONG, "arlo_infer: request %d has length %d > L = %d", i, h_len[i], L);
  if (n == 0) return ARLO_OK;
  const int bi = bucket_index(rt, n);
  Bucket& bk = rt->buckets[bi];
  for (int i = n; i < bk.b; ++i) h_len[i] = 0;
  *h_err = 0;
  if (!ids_dev) {
    for (int i = 0; i < n; ++i) {
      const int32_t* row = token_ids + (size_t)i * L;
      for (int t = 0; t < h_len[i]; ++t)
        if (row[t] < 0 || row[t] >= V)
          return set_error(ARLO_EINVAL, "arlo_infer: token id %d at [%d,%d] outside [0, %d)", row[t], i, t, V);
    }
    memcpy(h_ids, token_ids, 4 * (size_t)n * L);
    ARLO_CUDA(cudaMemcpyAsync(rt->err, h_err, 16 + 4 * (size_t)mb + 4 * (size_t)n * L, cudaMemcpyHostToDevice, s),
              "inputs H2D");
  } else {
    ARLO_CUDA(cudaMemcpyAsync(rt->err, h_err, 16 + 4 * (size_t)mb, cudaMemcpyHostToDevice, s), "lengths H2D");
    ARLO_CUDA(cudaMemcpyAsync(rt->ids, token_ids, 4 * (size_t)n * L, cudaMemcpyDeviceToDevice, s), "ids D2D");
  }
  ARLO_CUDA(cudaGraphLaunch(bk.exec, s), "cudaGraphLaunch");
  if (out_dev) {
    ARLO_CUDA(cudaMemcpyAsync(logits, rt->logits, 4 * (size_t)n * C, cudaMemcpyDeviceToDevice, s), "logits D2D");
  } else {
    ARLO_CUDA(cudaMemcpyAsync(h_logits, rt->logits, 4 * (size_t)n * C, cudaMemcpyDeviceToHost, s), "logits D2H");
  }
  ARLO_CUDA(cudaMemcpyAsync(h_err, rt->err, 4, cudaMemcpyDeviceToHost, s), "err D2H");
  ARLO_CUDA(cudaStreamSynchronize(s), "arlo_infer sync");
  if (*h_err) return set_error(ARLO_EINVAL, "arlo_infer: a token id at t < length is outside [0, %d)", V);
  if (!out_dev) memcpy(logits, h_logits, 4 * (size_t)n * C);
  return ARLO_OK;
}

extern "C" int arlo_enqueue(arlo_runtime* rt, int32_t n, const int32_t* token_ids, const int32_t* lengths,
                            float* logits) {
  if (!rt || !token_ids || !lengths || !logits) return set_error(ARLO_EINVAL, "arlo_enqueue: null argument");
  if (n < 1 || n > rt->max_batch) return set_error(ARLO_EINVAL, "arlo_enqueue: need 1 <= n <= max_batch");
  DeviceGuard g(rt->device);
  cudaStream_t s = rt->stream;
  const int bi = bucket_index(rt, n);
  Bucket& bk = rt->buckets[bi];
  const int L = rt->L, C = rt->w->cfg.num_labels;
  ARLO_CUDA(cudaMemcpyAsync(rt->lengths, lengths, 4 * (size_t)n, cudaMemcpyDeviceToDevice, s), "lengths D2D");
  if (bk.b > n) ARLO_CUDA(cudaMemsetAsync(rt->lengths + n, 0, 4 * (size_t)(bk.b - n), s), "lengths pad");
  ARLO_CUDA(cudaMemcpyAsync(rt->ids, token_ids, 4 * (size_t)n * L, cudaMemcpyDeviceToDevice, s), "ids D2D");
  ARLO_CUDA(cudaGraphLaunch(bk.exec, s), "cudaGraphLaunch");
  ARLO_CUDA(cudaMemcpyAsync(logits, rt->logits, 4 * (size_t)n * C, cudaMemcpyDeviceToDevice, s), "logits D2D");
  return ARLO_OK;
}

// ------------------------------------------------------------------------ ops ABI
static DType to_dt(int32_t d) { return d == ARLO_FP32 ? DT_FP32 : DT_BF16; }

extern "C" int arlo_op_gemm(int32_t dtype, int32_t M, int32_t N, int32_t K, const void* A, const void* W,
                            const float* bias, const void* residual, void* out, int32_t epi, int32_t force_bn,
                            void* stream) {
  clear_error();
  if (M < 1 || N % 64 || K % 64 || N < 64 || K < 64 || !A || !W || !bias || !out || epi < 0 || epi > 2 ||
      (epi == ARLO_EPI_BIAS_RESIDUAL && !residual))
    return set_error(ARLO_EINVAL, "arlo_op_gemm: bad arguments");
  cudaStream_t s = (cudaStream_t)stream;
  if (dtype == ARLO_BF16) {
    TcGemmPlan p;
    if (!tc_plan_gemm(&p, M, N, K, A, W, bias, residual, out, epi, force_bn))
      return set_error(ARLO_EINVAL, "arlo_op_gemm: plan failed (tile width %d / tensor map)", force_bn);
    ARLO_CUDA(tc_launch_gemm(p, s), "tcgen05 gemm");
  } else {
    ARLO_CUDA(launch_gemm_simt(DT_FP32, M, N, K, A, W, bias, residual, out, epi, s), "simt gemm");
  }
  return ARLO_OK;
}

extern "C" int arlo_op_gemm_fold(int32_t M, int32_t N, int32_t K, const void* A, const void* W, const float* v0,
                                 const float* v1, const float* v2, const float* st_in, int32_t st_in_stride,
                                 float* st_out, int32_t st_ld, float eps, const void* residual, void* out,
                                 int32_t epi, int32_t force_bn, void* stream) {
  clear_error();
  if (M < 1 || N % 64 || K % 64 || N < 64 || K < 64 || !A || !W || !v0 || !out ||
      (epi != EPI_LNFOLD && epi != EPI_LNFOLD_GELU && epi != EPI_RESID_LN) || (epi == EPI_RESID_LN && !residual) ||
      (epi != EPI_RESID_LN && (!v1 || !st_in)) || st_in_stride < 1 || ((st_in || st_out) && st_ld < M))
    return set_error(ARLO_EINVAL, "arlo_op_gemm_fold: bad arguments");
  TcGemmPlan p;
  if (!tc_plan_gemm(&p, M, N, K, A, W, v0, residual, out, epi, force_bn) || (p.splitk && epi != EPI_RESID_LN))
    return set_error(ARLO_EINVAL, "arlo_op_gemm_fold: plan failed (tile %d)", force_bn);
  p.fold = FoldArgs{v1, v2, st_in, st_in_stride, st_out, eps, st_ld};
  ARLO_CUDA(tc_launch_gemm(p, (cudaStream_t)stream), "LayerNorm-fold gemm");
  return ARLO_OK;
}

extern "C" int arlo_op_ln_gemm(int32_t M, int32_t N, int32_t K, const void* y, const float* gamma,
                               const float* beta, float eps, void* x, const void* W, const float* bias, void* out,
                               int32_t epi, int32_t force_bn, void* barrier, void* stream) {
  clear_error();
  if (M < 1 || N % 64 || K % 64 || N < 64 || K < 64 || !y || !gamma || !beta || !x || !W || !bias || !out ||
      !barrier || (epi != ARLO_EPI_BIAS && epi != ARLO_EPI_BIAS_GELU))
    return set_error(ARLO_EINVAL, "arlo_op_ln_gemm: bad arguments");
  TcGemmPlan p;
  if (!tc_plan_gemm(&p, M, N, K, x, W, bias, nullptr, out, epi, force_bn))
    return set_error(ARLO_EINVAL, "arlo_op_ln_gemm: plan failed (tile %d)", force_bn);
  LnPrologue lnp{y, gamma, beta, x, (unsigned*)barrier, eps, M, K};
  if (!tc_plan_attach_ln(&p, lnp))
    return set_error(ARLO_EINVAL, "arlo_op_ln_gemm: tile %d cannot run a LayerNorm prologue (skinny / non-persistent)",
                     force_bn);
  ARLO_CUDA(tc_launch_gemm(p, (cudaStream_t)stream), "LayerNorm-prologue gemm");
  return ARLO_OK;
}

extern "C" int arlo_op_layernorm(int32_t dtype, int32_t M, int32_t H, const void* in, const float* gamma,
                                 const float* beta, float eps, void* out, void* stream) {
  clear_error();
  if (M < 0 || H < 8 || H % 8 || !in || !gamma || !beta || !out) return set_error(ARLO_EINVAL, "arlo_op_layernorm: bad arguments");
  ARLO_CUDA(launch_layernorm(to_dt(dtype), M, H, in, gamma, beta, eps, out, (cudaStream_t)stream), "layernorm");
  return ARLO_OK;
}

extern "C" int arlo_op_embed(int32_t dtype, int32_t B, int32_t L, int32_t H, int32_t vocab, const int32_t* ids,
                             const int32_t* lengths, const void* word, const void* pos, const void* type,
                             const float* gamma, const float* beta, float eps, void* out, int32_t* err_flag,
                             void* stream) {
  clear_error();
  if (B < 0 || L < 1 || H < 8 || H % 8 || vocab < 1 || !ids || !lengths || !word || !pos || !type || !out)
    return set_error(ARLO_EINVAL, "arlo_op_embed: bad arguments");
  ARLO_CUDA(launch_embed_ln(to_dt(dtype), B, L, H, vocab, ids, lengths, word, pos, type, gamma, beta, eps, out,
                            err_flag, (cudaStream_t)stream),
            "embed");
  return ARLO_OK;
}

extern "C" int arlo_op_attention(int32_t dtype, int32_t B, int32_t L, int32_t heads, const void* qkv,
                                 const int32_t* lengths, void* o, void* stream) {
  clear_error();
  if (B < 0 || L < 1 || heads < 1 || !qkv || !lengths || !o) return set_error(ARLO_EINVAL, "arlo_op_attention: bad arguments");
  AttnPlan p;
  if (!attn_plan(&p, to_dt(dtype), B, L, heads, qkv))
    return set_error(ARLO_EINVAL, "arlo_op_attention: plan failed (bf16 needs L <= 512)");
  ARLO_CUDA(attn_launch(p, lengths, o, (cudaStream_t)stream), "attention");
  return ARLO_OK;
}

extern "C" int arlo_op_head(int32_t dtype, int32_t B, int32_t L, int32_t H, int32_t C, const void* x,
                            const void* w_p, const float* b_p, const void* w_c, const float* b_c, float* pooled,
                            float* logits, void* stream) {
  clear_error();
  if (B < 0 || L < 1 || H < 8 || H % 8 || H > 2048 || C < 1 || !x || !w_p || !b_p || !w_c || !b_c || !pooled ||
      !logits)
    return set_error(ARLO_EINVAL, "arlo_op_head: bad arguments");
  ARLO_CUDA(launch_head(to_dt(dtype), B, L, H, C, x, w_p, b_p, w_c, b_c, pooled, logits, (cudaStream_t)stream),
            "head");
  return ARLO_OK;
}

extern "C" int arlo_debug_gemm_trace(void* buf) {
  cudaError_t e = (cudaError_t)set_gemm_trace((unsigned long long*)buf);
  return e == cudaSuccess ? ARLO_OK : cuda_fail(e, "arlo_debug_gemm_trace");
}

extern "C" int32_t arlo_gemm_tile_choice(int32_t M, int32_t N, int32_t K) {
  if (M < 1 || N % 64 || K % 64 || N < 64 || K < 64) return 0;
  return tc_choose_bn(M, N, K);
}

extern "C" int arlo_debug_fused_trace(void* buf) {
  cudaError_t e = set_fused_trace((unsigned long long*)buf);
  return e == cudaSuccess ? ARLO_OK : cuda_fail(e, "arlo_debug_fused_trace");
}

extern "C" int arlo_debug_attn_trace(void* buf) {
  cudaError_t e = (cudaError_t)set_attn_trace((unsigned long long*)buf);
  return e == cudaSuccess ? ARLO_OK : cuda_fail(e, "arlo_debug_attn_trace");
}

extern "C" int arlo_op_gemm_ln(int32_t M, int32_t N, int32_t K, const void* A, const void* W, const float* bias,
                               const void* residual, const float* gamma, const float* beta, float eps, void* out,
                               void* stream) {
  clear_error();
  if (M < 1 || K % 64 || K < 64 || !A || !W || !bias || !residual || !gamma || !beta || !out)
    return set_error(ARLO_EINVAL, "arlo_op_gemm_ln: bad arguments");
  TcGemmPlan p;
  if (!tc_plan_gemm_ln(&p, M, N, K, A, W, bias, residual, gamma, beta, eps, out))
    return set_error(ARLO_EINVAL, "arlo_op_gemm_ln: N = %d not supported (needs N/192 or N/256 <= 8, or 128)", N);
  ARLO_CUDA(tc_launch_gemm(p, (cudaStream_t)stream), "fused gemm+layernorm");
  return ARLO_OK;
}
