"""ORACLE — plain fp64 CPU forward of one per-length runtime (TEST INFRASTRUCTURE).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this module.  The product path
(``paper_conf_icpp_tanlyl024_b200``) never imports it, and it never imports
the product path: the two share only the seeded generators in
``paper_conf_icpp_tanlyl024_b200/workload.py``.

What the method computes.  A polymorphed runtime with
max_length L runs a batch of requests zero-padded to L (PAPER.md:L37, L101
§2.2 "Uniform zero-padding"; L111 §2.3; L135 §3.2: len <= max_length).
Padding costs time only ("the corresponding output would be truncated
eventually"), so the runtime's result for a request is exactly
the model's forward over the request's real tokens.  The model is BERT
(Devlin et al. [17]; "Bert-Base and Bert-Large")
with a CLS pooler and a classifier head (discriminative models "predict labels
or classifications").  The oracle therefore evaluates that
definition per request over its real prefix n = len, in fp64, in the order of
the BERT definition:

  1. x[t] = E_w[tok[t]] + E_p[t] + E_type[0],  x = LN(x; g_e, b_e)
  2. per layer:  qkv = x W_qkv^T + b_qkv;  per head j (d = H/h columns)
        o_j = softmax_rows(q_j k_j^T / sqrt(d)) v_j
     x = LN(x + o W_o^T + b_o; g_1, b_1)
     x = LN(x + GELU(x W_1^T + b_1) W_2^T + b_2; g_2, b_2)
  3. LN(y) = (y - mean) / sqrt(var + eps) * g + b   (biased variance)
  4. p = tanh(W_p x[0] + b_p);  logits = W_c p + b_c

Readings where the paper is silent (DESIGN.md "Readings" S1-S12): post-LN
BERT as in HF BertForSequenceClassification (S1); GELU is the erf form (S2);
eps = 1e-12 (S3); padding mask from ``lengths`` (S4); token type 0, learned
absolute positions 0..L-1 (S7); pooler = tanh(dense(x[0])) (S8).

``forward_padded`` is the static-shape variant (all L positions computed,
keys t >= len excluded from the softmax); it exists only as the padding-
invariance self-check of §8(c) and is never the reference for the GPU.

Pins (tests/test_oracle_*.py): HF BertForSequenceClassification fp64 on the
same weights; torch.nn.TransformerEncoderLayer fp64 per layer; brute-force
triple-loop attention; closed forms (q=0 -> mean of real V rows, n=1 -> V_0,
GELU(1) = Phi(1)); LayerNorm mean/variance invariants; padding invariance.
"""
from __future__ import annotations

import numpy as np
from scipy.special import erf

F64 = np.float64


def layer_norm(y: np.ndarray, g: np.ndarray, b: np.ndarray, eps: float) -> np.ndarray:
    """LN over the last axis: (y - mu) / sqrt(sigma^2 + eps) * g + b, sigma^2 biased (step 3)."""
    y = np.asarray(y, F64)
    mu = y.mean(axis=-1, keepdims=True)
    var = ((y - mu) ** 2).mean(axis=-1, keepdims=True)
    return (y - mu) / np.sqrt(var + eps) * np.asarray(g, F64) + np.asarray(b, F64)


def gelu(z: np.ndarray) -> np.ndarray:
    """GELU(z) = z * Phi(z) = 0.5 z (1 + erf(z / sqrt 2))  (reading S2, erf form)."""
    z = np.asarray(z, F64)
    return 0.5 * z * (1.0 + erf(z / np.sqrt(2.0)))


def softmax_rows(s: np.ndarray) -> np.ndarray:
    """Row softmax, shifted by the row max (mathematically exact shift)."""
    s = np.asarray(s, F64)
    e = np.exp(s - s.max(axis=-1, keepdims=True))
    return e / e.sum(axis=-1, keepdims=True)


def attention(q: np.ndarray, k: np.ndarray, v: np.ndarray, heads: int) -> np.ndarray:
    """Multi-head scaled dot-product attention over n real tokens (step 2).

    q, k, v: [n, H]; head j uses columns j*d:(j+1)*d; scale 1/sqrt(d).
    """
    n, H = q.shape
    d = H // heads
    out = np.empty((n, H), F64)
    for j in range(heads):
        sl = slice(j * d, (j + 1) * d)
        s = (q[:, sl] @ k[:, sl].T) / np.sqrt(d)
        out[:, sl] = softmax_rows(s) @ v[:, sl]
    return out


def attention_masked(q, k, v, heads: int, length: int) -> np.ndarray:
    """Static-shape attention over L rows where keys t >= length are excluded
    (reading S4: exactly equivalent to an additive -inf mask)."""
    L, H = q.shape
    d = H // heads
    out = np.empty((L, H), F64)
    for j in range(heads):
        sl = slice(j * d, (j + 1) * d)
        s = (q[:, sl] @ k[:length, sl].T) / np.sqrt(d)
        out[:, sl] = softmax_rows(s) @ v[:length, sl]
    return out


def embed(cfg, w: dict, tok: np.ndarray) -> np.ndarray:
    """Step 1: word + position + type-0 embedding, then the embedding LayerNorm."""
    n = tok.shape[0]
    x = (np.asarray(w["word_emb"], F64)[tok] + np.asarray(w["pos_emb"], F64)[:n]
         + np.asarray(w["type_emb"], F64)[0])
    return layer_norm(x, w["emb_ln_g"], w["emb_ln_b"], cfg.ln_eps)


def linear(x: np.ndarray, wt: np.ndarray, b: np.ndarray) -> np.ndarray:
    """x W^T + b with W in [out, in] layout."""
    return np.asarray(x, F64) @ np.asarray(wt, F64).T + np.asarray(b, F64)


def encoder_layer(cfg, lw: dict, x: np.ndarray, length: int | None = None) -> np.ndarray:
    """Step 2 for one post-LN layer; ``length`` selects the masked static-shape form."""
    H = cfg.hidden
    qkv = linear(x, lw["w_qkv"], lw["b_qkv"])
    q, k, v = qkv[:, :H], qkv[:, H:2 * H], qkv[:, 2 * H:]
    if length is None:
        o = attention(q, k, v, cfg.heads)
    else:
        o = attention_masked(q, k, v, cfg.heads, length)
    x = layer_norm(x + linear(o, lw["w_o"], lw["b_o"]), lw["ln1_g"], lw["ln1_b"], cfg.ln_eps)
    f = linear(gelu(linear(x, lw["w_1"], lw["b_1"])), lw["w_2"], lw["b_2"])
    return layer_norm(x + f, lw["ln2_g"], lw["ln2_b"], cfg.ln_eps)


def head(w: dict, x0: np.ndarray) -> np.ndarray:
    """Step 4: pooled = tanh(W_p x[0] + b_p); logits = W_c pooled + b_c."""
    pooled = np.tanh(linear(x0[None, :], w["w_p"], w["b_p"]))[0]
    return linear(pooled[None, :], w["w_c"], w["b_c"])[0]


def hidden_states(cfg, w: dict, tok: np.ndarray) -> np.ndarray:
    """Final-layer hidden states [n, H] of one request's real tokens."""
    x = embed(cfg, w, np.asarray(tok))
    for lw in w["layers"]:
        x = encoder_layer(cfg, lw, x)
    return x


def forward_request(cfg, w: dict, tok: np.ndarray) -> np.ndarray:
    """Logits [C] of one request given its real token ids (length n >= 1)."""
    return head(w, hidden_states(cfg, w, tok)[0])


def forward_batch(cfg, w: dict, token_ids: np.ndarray, lengths: np.ndarray) -> np.ndarray:
    """What ``arlo_infer`` must return: logits [n, C] for the leading requests
    with lengths > 0, each over its real prefix only (padding never enters)."""
    lengths = np.asarray(lengths)
    out = []
    for i, n in enumerate(lengths):
        n = int(n)
        if n <= 0:
            break
        out.append(forward_request(cfg, w, np.asarray(token_ids[i, :n])))
    return np.asarray(out, F64).reshape(len(out), cfg.num_labels)


def forward_padded(cfg, w: dict, tok_padded: np.ndarray, length: int) -> tuple:
    """Static-shape forward over all L positions with keys t >= length masked
    (padding self-check only).  Returns (hidden [L, H], logits [C])."""
    tok = np.asarray(tok_padded).copy()
    tok[length:] = 0
    x = embed(cfg, w, tok)
    for lw in w["layers"]:
        x = encoder_layer(cfg, lw, x, length=length)
    return x, head(w, x[0])


def label(logits: np.ndarray) -> np.ndarray:
    """argmax, lowest index wins ties (reading S11)."""
    return np.argmax(np.asarray(logits), axis=-1)

