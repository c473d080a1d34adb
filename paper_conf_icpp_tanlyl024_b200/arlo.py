"""Thin ctypes binding of libarlo.so (include/arlo.h, include/arlo_ops.h).

Argument marshalling only: every step of the hot path runs in the library's
sm_100a kernels.  torch is used for device memory and streams (tensors are
passed by ``data_ptr()``).  Importing this module loads the library and raises
immediately if it is missing; there is no fallback path.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libarlo.so")
# A/B hook for kernel experiments: ARLO_LIB_VARIANT=name loads build/libarlo_<name>.so, an
# in-tree variant built by `python -m paper_conf_icpp_tanlyl024_b200.build --variant name -D...`.
if os.environ.get("ARLO_LIB_VARIANT"):
    LIB_PATH = os.path.join(_HERE, "build", f"libarlo_{os.environ['ARLO_LIB_VARIANT']}.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_icpp_tanlyl024_b200.build` "
                      "(or __graft_entry__.build()); there is no non-CUDA fallback")
lib = C.CDLL(LIB_PATH)

OK, EINVAL, ETOOLONG, ENOMEM, ECUDA, EINFEASIBLE, ENOCAND, ENODEV = 0, -1, -2, -3, -4, -5, -6, -7
BF16, FP32 = 0, 1
DISPATCH_RS, DISPATCH_ILB, DISPATCH_IG = 0, 1, 2
EPI_BIAS, EPI_BIAS_GELU, EPI_BIAS_RESIDUAL = 0, 1, 2
EPI_LNFOLD, EPI_LNFOLD_GELU, EPI_RESID_LN = 3, 4, 5
RUNTIME_DEFAULT, RUNTIME_LATENCY, RUNTIME_THROUGHPUT, RUNTIME_FUSED, RUNTIME_SPLITK = 0, 1, 2, 3, 4
SKINNY_CODE, SPLITK_CODE, FUSED_CODE = 1000, 2000, 3000  # tile codes: kSkinnyCode + BN, kSplitKCode + BN, kFusedCode + S

EXPORTED = [
    "arlo_replace_plan", "arlo_runtime_gemm_tiles",
    "arlo_last_error", "arlo_version", "arlo_weights_count", "arlo_weights_create", "arlo_weights_destroy",
    "arlo_runtime_create", "arlo_runtime_create_ex", "arlo_runtime_family", "arlo_runtime_destroy", "arlo_runtime_set_stream", "arlo_runtime_length",
    "arlo_runtime_max_batch", "arlo_infer", "arlo_enqueue", "arlo_runtime_kernel_count", "arlo_runtime_bucket", "arlo_allocate",
    "arlo_sched_create", "arlo_sched_destroy", "arlo_sched_set_params", "arlo_sched_set_policy", "arlo_dispatch", "arlo_complete", "arlo_sched_outstanding",
    "arlo_op_gemm", "arlo_op_gemm_ln", "arlo_op_gemm_fold", "arlo_op_ln_gemm", "arlo_op_layernorm", "arlo_op_embed", "arlo_op_attention", "arlo_op_head",
    "arlo_debug_gemm_trace", "arlo_debug_attn_trace", "arlo_debug_fused_trace", "arlo_gemm_tile_choice",
]


class ModelConfigC(C.Structure):
    _fields_ = [("layers", C.c_int32), ("hidden", C.c_int32), ("heads", C.c_int32), ("ffn", C.c_int32),
                ("vocab", C.c_int32), ("max_pos", C.c_int32), ("type_vocab", C.c_int32),
                ("num_labels", C.c_int32), ("ln_eps", C.c_float), ("dtype", C.c_int32)]


_vp, _i32, _f32, _f64 = C.c_void_p, C.c_int32, C.c_float, C.c_double
_P = C.POINTER


def _sig(name, res, *args):
    f = getattr(lib, name)
    f.restype = res
    f.argtypes = list(args)
    return f


_sig("arlo_last_error", C.c_char_p)
_sig("arlo_version", C.c_char_p)
_sig("arlo_weights_count", _i32, _P(ModelConfigC))
_sig("arlo_weights_create", C.c_int, _i32, _P(ModelConfigC), _P(_vp), _i32, _P(_vp))
_sig("arlo_weights_destroy", None, _vp)
_sig("arlo_runtime_create", C.c_int, _i32, _i32, _vp, _P(_vp))
_sig("arlo_runtime_create_ex", C.c_int, _i32, _i32, _vp, _i32, _P(_vp))
_sig("arlo_runtime_family", _i32, _vp)
_sig("arlo_runtime_destroy", None, _vp)
_sig("arlo_runtime_set_stream", C.c_int, _vp, _vp)
_sig("arlo_runtime_length", _i32, _vp)
_sig("arlo_runtime_max_batch", _i32, _vp)
_sig("arlo_infer", C.c_int, _vp, _vp, _vp, _vp)
_sig("arlo_enqueue", C.c_int, _vp, _i32, _vp, _vp, _vp)
_sig("arlo_runtime_kernel_count", _i32, _vp, _i32)
_sig("arlo_runtime_bucket", _i32, _vp, _i32)
_sig("arlo_runtime_gemm_tiles", C.c_int, _vp, _i32, _P(_i32))
_sig("arlo_sched_set_policy", C.c_int, _vp, _i32)
_sig("arlo_allocate", C.c_int, _i32, _i32, _P(_f64), _P(_f64), _P(_f64), _i32, _P(_i32), _P(_f64))
_sig("arlo_replace_plan", C.c_int, _i32, _i32, _P(_i32), _P(_i32), _P(_i32), _P(_i32))
_sig("arlo_sched_create", C.c_int, _i32, _P(_i32), _P(_i32), _P(_f64), _f64, _f64, _i32, _P(_vp))
_sig("arlo_sched_destroy", None, _vp)
_sig("arlo_sched_set_params", C.c_int, _vp, _f64, _f64, _i32)
_sig("arlo_dispatch", C.c_int, _vp, _i32, _P(_i32), _P(_i32))
_sig("arlo_complete", C.c_int, _vp, _i32, _i32)
_sig("arlo_sched_outstanding", _i32, _vp, _i32, _i32)
_sig("arlo_op_gemm", C.c_int, _i32, _i32, _i32, _i32, _vp, _vp, _vp, _vp, _vp, _i32, _i32, _vp)
_sig("arlo_op_gemm_fold", C.c_int, _i32, _i32, _i32, _vp, _vp, _vp, _vp, _vp, _vp, _i32, _vp, _i32, _f32, _vp, _vp, _i32, _i32, _vp)
_sig("arlo_op_gemm_ln", C.c_int, _i32, _i32, _i32, _vp, _vp, _vp, _vp, _vp, _vp, _f32, _vp, _vp)
_sig("arlo_op_ln_gemm", C.c_int, _i32, _i32, _i32, _vp, _vp, _vp, _f32, _vp, _vp, _vp, _vp, _i32, _i32, _vp, _vp)
_sig("arlo_op_layernorm", C.c_int, _i32, _i32, _i32, _vp, _vp, _vp, _f32, _vp, _vp)
_sig("arlo_op_embed", C.c_int, _i32, _i32, _i32, _i32, _i32, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _f32, _vp, _vp, _vp)
_sig("arlo_op_attention", C.c_int, _i32, _i32, _i32, _i32, _vp, _vp, _vp, _vp)
_sig("arlo_debug_gemm_trace", C.c_int, _vp)
_sig("arlo_debug_attn_trace", C.c_int, _vp)
_sig("arlo_debug_fused_trace", C.c_int, _vp)
_sig("arlo_gemm_tile_choice", _i32, _i32, _i32, _i32)
_sig("arlo_op_head", C.c_int, _i32, _i32, _i32, _i32, _i32, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _vp)


class ArloError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"arlo error {code}: {msg}")
        self.code = code


def check(rc: int) -> int:
    if rc < 0:
        raise ArloError(rc, lib.arlo_last_error().decode())
    return rc


def _ptr(x):
    """Device/host address of a torch tensor or numpy array (no copies)."""
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    return x.data_ptr()


def _stream_ptr(stream):
    if stream is None:
        return None
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


def gemm_tile_choice(M: int, N: int, K: int) -> int:
    """BN of the single-CTA tcgen05 kernel, or -BN of the CTA-pair kernel, chosen for (M, N, K)."""
    return int(lib.arlo_gemm_tile_choice(M, N, K))


def version() -> str:
    return lib.arlo_version().decode()


def make_config(cfg, dtype: int) -> ModelConfigC:
    return ModelConfigC(cfg.layers, cfg.hidden, cfg.heads, cfg.ffn, cfg.vocab, cfg.max_pos, cfg.type_vocab,
                        cfg.num_labels, cfg.ln_eps, dtype)


def upload_weights(cfg, w: dict, dtype: int, device="cuda"):
    """Canonical tensor list on `device`: matrices/tables in bf16 or fp32, vectors fp32."""
    import torch
    from . import workload
    mat_dt = torch.bfloat16 if dtype == BF16 else torch.float32
    out = []
    for a in workload.canonical_tensor_list(cfg, w):
        t = torch.from_numpy(np.ascontiguousarray(a, np.float32))
        t = t.to(device=device, dtype=mat_dt if a.ndim == 2 else torch.float32)
        out.append(t.contiguous())
    return out


class Weights:
    """arlo_weights: borrows the device tensors (kept alive by this object)."""

    def __init__(self, cfg, tensors, dtype: int, device_index: int = 0):
        self.cfg, self.dtype, self.tensors = cfg, dtype, list(tensors)
        self._c = make_config(cfg, dtype)
        arr = (_vp * len(self.tensors))(*[t.data_ptr() for t in self.tensors])
        h = _vp()
        check(lib.arlo_weights_create(device_index, C.byref(self._c), arr, len(self.tensors), C.byref(h)))
        self.handle = h

    def close(self):
        if getattr(self, "handle", None):
            lib.arlo_weights_destroy(self.handle)
            self.handle = None

    __del__ = close


class Runtime:
    """arlo_runtime: one statically shaped per-length runtime (L, max_batch)."""

    def __init__(self, weights: Weights, L: int, max_batch: int, family: int = RUNTIME_DEFAULT):
        self.weights, self.L, self.max_batch = weights, L, max_batch
        h = _vp()
        check(lib.arlo_runtime_create_ex(L, max_batch, weights.handle, family, C.byref(h)))
        self.handle = h

    @property
    def family(self) -> int:
        """RUNTIME_THROUGHPUT, RUNTIME_LATENCY (LayerNorm fold), RUNTIME_FUSED or RUNTIME_SPLITK."""
        return check(lib.arlo_runtime_family(self.handle))

    def set_stream(self, stream):
        check(lib.arlo_runtime_set_stream(self.handle, _stream_ptr(stream)))

    def bucket_of(self, n: int) -> int:
        """Batch bucket (captured graph) that serves n requests."""
        return check(lib.arlo_runtime_bucket(self.handle, n))

    def kernel_count(self, n: int) -> int:
        return check(lib.arlo_runtime_kernel_count(self.handle, n))

    def gemm_tiles(self, n: int):
        """Tile codes (QKV, out-proj, FFN1, FFN2) of the graph serving n requests."""
        codes = (_i32 * 4)()
        check(lib.arlo_runtime_gemm_tiles(self.handle, n, codes))
        return [int(v) for v in codes]

    def infer(self, token_ids, lengths, logits):
        """Synchronous; each argument a torch tensor (host or device) or numpy array."""
        check(lib.arlo_infer(self.handle, _ptr(token_ids), _ptr(lengths), _ptr(logits)))
        return logits

    def enqueue(self, n: int, token_ids, lengths, logits):
        """Asynchronous on the runtime's stream; device tensors only."""
        check(lib.arlo_enqueue(self.handle, n, _ptr(token_ids), _ptr(lengths), _ptr(logits)))

    def close(self):
        if getattr(self, "handle", None):
            lib.arlo_runtime_destroy(self.handle)
            self.handle = None

    __del__ = close


def allocate(G: int, Q, M, lat):
    """arlo_allocate (Eqs. 1-7). lat: [I][nb]. Returns (N tuple, objective)."""
    Q = np.ascontiguousarray(Q, np.float64)
    M = np.ascontiguousarray(M, np.float64)
    lat = np.ascontiguousarray(lat, np.float64)
    I, nb = lat.shape
    N = (_i32 * I)()
    obj = _f64()
    check(lib.arlo_allocate(G, I, Q.ctypes.data_as(_P(_f64)), M.ctypes.data_as(_P(_f64)),
                            lat.ctypes.data_as(_P(_f64)), nb, N, C.byref(obj)))
    return tuple(int(v) for v in N), obj.value


def replace_plan(cur, N_new):
    """arlo_replace_plan: minimum-replacement plan from per-GPU runtime indices
    cur (-1 = none) to the allocation N_new. Returns (next list, n_replaced)."""
    G, I = len(cur), len(N_new)
    c = (_i32 * G)(*cur)
    nn = (_i32 * I)(*N_new)
    nxt = (_i32 * G)()
    rep = _i32()
    check(lib.arlo_replace_plan(G, I, c, nn, nxt, C.byref(rep)))
    return [int(v) for v in nxt], int(rep.value)


class Scheduler:
    """arlo_sched: multi-level queue + Algorithm 1."""

    def __init__(self, max_len, n_inst, capacity, lam=0.85, alpha=0.9, peek=6):
        K = len(max_len)
        ml = (_i32 * K)(*max_len)
        ni = (_i32 * K)(*n_inst)
        cap = (_f64 * K)(*capacity)
        h = _vp()
        check(lib.arlo_sched_create(K, ml, ni, cap, lam, alpha, peek, C.byref(h)))
        self.handle = h

    def set_params(self, lam: float, alpha: float, peek: int):
        check(lib.arlo_sched_set_params(self.handle, lam, alpha, peek))

    def set_policy(self, policy: int):
        """DISPATCH_RS (Algorithm 1), DISPATCH_ILB or DISPATCH_IG (PAPER.md:L373 baselines)."""
        check(lib.arlo_sched_set_policy(self.handle, policy))

    def dispatch(self, length: int):
        r, i = _i32(), _i32()
        check(lib.arlo_dispatch(self.handle, length, C.byref(r), C.byref(i)))
        return r.value, i.value

    def complete(self, runtime: int, instance: int):
        check(lib.arlo_complete(self.handle, runtime, instance))

    def outstanding(self, runtime: int, instance: int) -> int:
        return check(lib.arlo_sched_outstanding(self.handle, runtime, instance))

    def close(self):
        if getattr(self, "handle", None):
            lib.arlo_sched_destroy(self.handle)
            self.handle = None

    __del__ = close


# ------------------------------------------------------------------ per-kernel ops
def op_gemm(dtype, A, W, bias, out, epi=EPI_BIAS, residual=None, force_bn=0, stream=None):
    M, K = A.shape
    N = W.shape[0]
    check(lib.arlo_op_gemm(dtype, M, N, K, _ptr(A), _ptr(W), _ptr(bias), _ptr(residual), _ptr(out), epi,
                           force_bn, _stream_ptr(stream)))
    return out


def op_gemm_fold(A, W, v0, out, epi, v1=None, v2=None, st_in=None, st_in_stride=1, st_out=None, st_ld=None,
                 eps=1e-12, residual=None, force_bn=0, stream=None):
    """LayerNorm-fold epilogues (arlo_op_gemm_fold; include/arlo_ops.h).  Statistics tensors are
    granule-major [G, st_ld, 2] (st_ld defaults to M)."""
    M, K = A.shape
    N = W.shape[0]
    check(lib.arlo_op_gemm_fold(M, N, K, _ptr(A), _ptr(W), _ptr(v0), _ptr(v1), _ptr(v2), _ptr(st_in), st_in_stride,
                                _ptr(st_out), st_ld or M, eps, _ptr(residual), _ptr(out), epi, force_bn,
                                _stream_ptr(stream)))
    return out


def op_gemm_ln(A, W, bias, residual, gamma, beta, eps, out, stream=None):
    M, K = A.shape
    N = W.shape[0]
    check(lib.arlo_op_gemm_ln(M, N, K, _ptr(A), _ptr(W), _ptr(bias), _ptr(residual), _ptr(gamma), _ptr(beta), eps,
                              _ptr(out), _stream_ptr(stream)))
    return out


def op_ln_gemm(y, gamma, beta, eps, x, W, bias, out, epi=EPI_BIAS, force_bn=0, barrier=None, stream=None):
    """x = LN(y) and out = epi(x W^T + bias) in one launch (LayerNorm prologue of a persistent GEMM).
    barrier: >= 2 zero-initialised int32 on the device (allocated here if None)."""
    import torch
    M, K = y.shape
    N = W.shape[0]
    if barrier is None:
        barrier = torch.zeros(2, dtype=torch.int32, device=y.device)
    check(lib.arlo_op_ln_gemm(M, N, K, _ptr(y), _ptr(gamma), _ptr(beta), eps, _ptr(x), _ptr(W), _ptr(bias),
                              _ptr(out), epi, force_bn, _ptr(barrier), _stream_ptr(stream)))
    return out


def op_layernorm(dtype, x, gamma, beta, eps, out, stream=None):
    M, H = x.shape
    check(lib.arlo_op_layernorm(dtype, M, H, _ptr(x), _ptr(gamma), _ptr(beta), eps, _ptr(out), _stream_ptr(stream)))
    return out


def op_embed(dtype, ids, lengths, word, pos, type_, gamma, beta, eps, out, err_flag=None, stream=None):
    B, L = ids.shape
    V, H = word.shape
    check(lib.arlo_op_embed(dtype, B, L, H, V, _ptr(ids), _ptr(lengths), _ptr(word), _ptr(pos), _ptr(type_),
                            _ptr(gamma), _ptr(beta), eps, _ptr(out), _ptr(err_flag), _stream_ptr(stream)))
    return out


def op_attention(dtype, B, L, heads, qkv, lengths, out, stream=None):
    check(lib.arlo_op_attention(dtype, B, L, heads, _ptr(qkv), _ptr(lengths), _ptr(out), _stream_ptr(stream)))
    return out


def op_head(dtype, B, L, x, w_p, b_p, w_c, b_c, logits, stream=None):
    import torch
    H = w_p.shape[1]
    Cn = w_c.shape[0]
    pooled = torch.empty((B, H), dtype=torch.float32, device=logits.device)
    check(lib.arlo_op_head(dtype, B, L, H, Cn, _ptr(x), _ptr(w_p), _ptr(b_p), _ptr(w_c), _ptr(b_c), _ptr(pooled),
                           _ptr(logits), _stream_ptr(stream)))
    return logits
