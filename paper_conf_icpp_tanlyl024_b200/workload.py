"""Seeded synthetic inputs shared by the oracle and the CUDA path.

This module is the ONLY code both sides import.  It
holds model dimensions and random-number recipes, and none of the method's
arithmetic: no embedding sum, no LayerNorm, no attention, no GEMM.

Recipes (seeds: weights 0, lengths 1, token ids 2, arrivals 3):

* Model configs (BASELINE.json ``configs``; SURVEY.md §8 notation T/B/G/R).
  BERT = Devlin et al. [17], evaluated as "Bert-Base and
  Bert-Large" (§5 Setup).
* Weights: reading S10 of DESIGN.md — matrices/embeddings/biases N(0, 0.02),
  LayerNorm gamma 1+N(0, 0.1), beta N(0, 0.02); every value rounded to the
  nearest bf16 (ties to even) so fp32/fp64 consumers see exactly the values
  the bf16 GPU path stores.
* Lengths: reading S12/§8(d) — X ~ LogNormal(ln 21, 0.6) truncated at 125
  (median 21 / p98 72 of the Twitter trace, §2.1; max ~125 and
  "recalibrated ... up to 512", §5 Workloads), then
  len = clamp(round(X * 512 / 125), 2, 512).
* Token ids: tok[0] = CLS, tok[len-1] = SEP, the rest uniform in [5, V);
  positions t >= len are filled with 0 (zero padding).
* Arrivals: Poisson ("Twitter-Stable") or a 2-state MMPP ("Twitter-Bursty"),
  PAPER.md:L297; MMPP rates 1.6x / 0.4x the mean, exponential dwell mean 1 s.
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

SEED_WEIGHTS = 0
SEED_LENGTHS = 1
SEED_TOKENS = 2
SEED_ARRIVALS = 3

# Canonical per-layer tensor names, in the order the C ABI takes them
# (include/arlo.h, arlo_weights_create).
LAYER_TENSORS = ("w_qkv", "b_qkv", "w_o", "b_o", "ln1_g", "ln1_b",
                 "w_1", "b_1", "w_2", "b_2", "ln2_g", "ln2_b")
HEAD_TENSORS = ("w_p", "b_p", "w_c", "b_c")
EMB_TENSORS = ("word_emb", "pos_emb", "type_emb", "emb_ln_g", "emb_ln_b")


@dataclasses.dataclass(frozen=True)
class ModelConfig:
    name: str
    layers: int
    hidden: int
    heads: int
    ffn: int
    vocab: int
    max_pos: int = 512
    type_vocab: int = 2
    num_labels: int = 2
    ln_eps: float = 1e-12

    @property
    def head_dim(self) -> int:
        return self.hidden // self.heads

    @property
    def cls_id(self) -> int:
        return 101 if self.vocab > 103 else 1

    @property
    def sep_id(self) -> int:
        return 102 if self.vocab > 103 else 2


TINY = ModelConfig("tiny", layers=2, hidden=128, heads=2, ffn=512, vocab=1000)
BERT_BASE = ModelConfig("bert-base", layers=12, hidden=768, heads=12, ffn=3072, vocab=30522)
BERT_LARGE = ModelConfig("bert-large", layers=24, hidden=1024, heads=16, ffn=4096, vocab=30522)
ROBERTA_LARGE = ModelConfig("roberta-large-shaped", layers=24, hidden=1024, heads=16, ffn=4096,
                            vocab=50265, ln_eps=1e-5)
CONFIGS = {c.name: c for c in (TINY, BERT_BASE, BERT_LARGE, ROBERTA_LARGE)}

# Runtime max_length set: 64-token staircase, 512/64 = 8 runtimes (§3.3).
RUNTIME_LENGTHS = (64, 128, 192, 256, 320, 384, 448, 512)


def round_to_bf16(x: np.ndarray) -> np.ndarray:
    """Round float32 values to the nearest bf16 (ties to even); returns float32."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    u = x.view(np.uint32).astype(np.uint64)
    rounding_bias = ((u >> 16) & 1) + 0x7FFF
    u = ((u + rounding_bias) & 0xFFFF0000).astype(np.uint32)
    return u.view(np.float32)


def layer_tensor_shapes(cfg: ModelConfig) -> dict:
    H, F = cfg.hidden, cfg.ffn
    return {"w_qkv": (3 * H, H), "b_qkv": (3 * H,), "w_o": (H, H), "b_o": (H,),
            "ln1_g": (H,), "ln1_b": (H,), "w_1": (F, H), "b_1": (F,),
            "w_2": (H, F), "b_2": (H,), "ln2_g": (H,), "ln2_b": (H,)}


def make_weights(cfg: ModelConfig, seed: int = SEED_WEIGHTS, unit_ln: bool = False) -> dict:
    """Seeded random weights (reading S10), all values bf16-representable, float32 arrays.

    Matrices use the PyTorch Linear layout [out, in].  ``unit_ln`` sets every
    LayerNorm gamma to 1 and beta to 0 (used by the LayerNorm invariant tests).
    """
    rng = np.random.default_rng(seed)
    H, C = cfg.hidden, cfg.num_labels

    def normal(shape, std=0.02, mean=0.0):
        return round_to_bf16(mean + std * rng.standard_normal(shape, dtype=np.float64).astype(np.float32))

    def ln_pair():
        if unit_ln:
            return np.ones(H, np.float32), np.zeros(H, np.float32)
        return normal((H,), 0.1, 1.0), normal((H,))

    w = {"word_emb": normal((cfg.vocab, H)), "pos_emb": normal((cfg.max_pos, H)),
         "type_emb": normal((cfg.type_vocab, H))}
    w["emb_ln_g"], w["emb_ln_b"] = ln_pair()
    layers = []
    for _ in range(cfg.layers):
        lw = {}
        for name, shape in layer_tensor_shapes(cfg).items():
            if name.startswith("ln"):
                continue
            lw[name] = normal(shape)
        lw["ln1_g"], lw["ln1_b"] = ln_pair()
        lw["ln2_g"], lw["ln2_b"] = ln_pair()
        layers.append(lw)
    w["layers"] = layers
    w["w_p"], w["b_p"] = normal((H, H)), normal((H,))
    w["w_c"], w["b_c"] = normal((C, H)), normal((C,))
    return w


def canonical_tensor_list(cfg: ModelConfig, w: dict) -> list:
    """Flatten ``w`` into the canonical order of include/arlo.h (arlo_weights_create)."""
    out = [w[n] for n in EMB_TENSORS]
    for lw in w["layers"]:
        out.extend(lw[n] for n in LAYER_TENSORS)
    out.extend(w[n] for n in HEAD_TENSORS)
    return out


# ----------------------------------------------------------------------------- lengths
_LN_MU = math.log(21.0)
_LN_SIGMA = 0.600
_X_MAX = 125.0
_SCALE = 512.0 / 125.0


def _lognorm_cdf(x):
    from scipy.special import ndtr
    x = np.asarray(x, dtype=np.float64)
    with np.errstate(divide="ignore"):
        z = (np.log(np.maximum(x, 1e-300)) - _LN_MU) / _LN_SIGMA
    return np.where(x > 0, ndtr(z), 0.0)


def _lognorm_ppf(u):
    from scipy.special import ndtri
    return np.exp(_LN_MU + _LN_SIGMA * ndtri(u))


def sample_lengths(n: int, seed: int = SEED_LENGTHS, lo: int = 0, hi: int = 512) -> np.ndarray:
    """Skewed request lengths in (lo, hi] (DESIGN.md input recipe), int32.

    Inverse-CDF sampling of the truncated log-normal restricted to the X range
    that maps onto (lo, hi]; with lo=0, hi=512 it is the whole distribution.
    """
    rng = np.random.default_rng(seed)
    lo = max(lo, 1)  # len >= 2 after clamping
    # round(X*s) in (lo, hi]  <=>  X in [(lo+0.5)/s, (hi+0.5)/s)
    x_lo = 0.0 if lo <= 1 else (lo + 0.5) / _SCALE
    x_hi = min(_X_MAX, (hi + 0.5) / _SCALE)
    u_lo, u_hi = _lognorm_cdf(x_lo), _lognorm_cdf(x_hi)
    u = u_lo + (u_hi - u_lo) * rng.random(n)
    u = np.clip(u, 1e-300, 1 - 1e-16)
    x = _lognorm_ppf(u)
    lens = np.clip(np.rint(x * _SCALE), max(2, lo + 1), hi).astype(np.int32)
    return lens


def drifting_lengths(n: int, scale: float, seed: int = SEED_LENGTHS) -> np.ndarray:
    """Lengths of one re-allocation window whose distribution has drifted: the base skewed lengths
    multiplied by `scale` (re-rounded, clamped to [2, 512]).  A synthetic stand-in for the
    coarse-time-scale shifts of the length distribution the Runtime Scheduler tracks
    (§1, "every 10 minutes"; period 120 s, L299).  Generator only: no method
    arithmetic."""
    base = sample_lengths(n, seed=seed)
    return np.clip(np.rint(base * scale), 2, 512).astype(np.int32)


def sample_token_ids(cfg: ModelConfig, lengths: np.ndarray, L: int, seed: int = SEED_TOKENS) -> np.ndarray:
    """[b, L] int32 ids: CLS, uniform body, SEP, zero padding (reading S12)."""
    rng = np.random.default_rng(seed)
    lengths = np.asarray(lengths)
    b = lengths.shape[0]
    ids = np.zeros((b, L), dtype=np.int32)
    body = rng.integers(5, cfg.vocab, size=(b, L), dtype=np.int64).astype(np.int32)
    for i, n in enumerate(lengths):
        n = int(n)
        if n <= 0:
            continue
        ids[i, :n] = body[i, :n]
        ids[i, 0] = cfg.cls_id
        if n >= 2:
            ids[i, n - 1] = cfg.sep_id
    return ids


def ideal_runtime(lengths: np.ndarray, runtime_lengths=RUNTIME_LENGTHS) -> np.ndarray:
    """Index of the smallest max_length >= len (§3.2: a request of
    length len runs only on runtimes with max_length >= len)."""
    rl = np.asarray(runtime_lengths)
    return np.searchsorted(rl, np.asarray(lengths), side="left")


def poisson_arrivals(n: int, rate: float, seed: int = SEED_ARRIVALS) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return np.cumsum(rng.exponential(1.0 / rate, size=n))


def mmpp_arrivals(n: int, rate: float, seed: int = SEED_ARRIVALS, hi=1.6, lo=0.4, dwell=1.0) -> np.ndarray:
    """2-state Markov-modulated Poisson process with mean rate ``rate``."""
    rng = np.random.default_rng(seed)
    t, out, state = 0.0, [], 0
    switch = rng.exponential(dwell)
    while len(out) < n:
        r = rate * (hi if state == 0 else lo)
        dt = rng.exponential(1.0 / r)
        if t + dt > switch:
            t = switch
            state ^= 1
            switch = t + rng.exponential(dwell)
            continue
        t += dt
        out.append(t)
    return np.asarray(out)
