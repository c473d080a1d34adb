"""Pins for oracle/encoder.py against things other than itself (CPU only).

Each test names what fixes the expected value: a library routine written
independently of the oracle (HF BertForSequenceClassification, torch's
TransformerEncoderLayer and scaled_dot_product_attention), brute force on tiny
inputs, closed forms, or invariants of the mathematics.
"""
import math

import numpy as np
import pytest
import torch

from oracle import encoder as orc
from paper_conf_icpp_tanlyl024_b200 import workload as wl

# A small config whose head count (3) and ffn (not 4H) catch head-slicing and
# shape mix-ups that a 2-head 4H config could hide.
ODD = wl.ModelConfig("odd", layers=2, hidden=192, heads=3, ffn=320, vocab=300, max_pos=128)


def _hf_model(cfg, w):
    from transformers import BertConfig, BertForSequenceClassification
    hc = BertConfig(vocab_size=cfg.vocab, hidden_size=cfg.hidden, num_hidden_layers=cfg.layers,
                    num_attention_heads=cfg.heads, intermediate_size=cfg.ffn, hidden_act="gelu",
                    hidden_dropout_prob=0.0, attention_probs_dropout_prob=0.0,
                    max_position_embeddings=cfg.max_pos, type_vocab_size=cfg.type_vocab,
                    layer_norm_eps=cfg.ln_eps, num_labels=cfg.num_labels)
    hc._attn_implementation = "eager"
    m = BertForSequenceClassification(hc).double().eval()
    H = cfg.hidden
    t = lambda a: torch.tensor(np.asarray(a, np.float64))
    sd = {"bert.embeddings.word_embeddings.weight": w["word_emb"],
          "bert.embeddings.position_embeddings.weight": w["pos_emb"],
          "bert.embeddings.token_type_embeddings.weight": w["type_emb"],
          "bert.embeddings.LayerNorm.weight": w["emb_ln_g"],
          "bert.embeddings.LayerNorm.bias": w["emb_ln_b"],
          "bert.pooler.dense.weight": w["w_p"], "bert.pooler.dense.bias": w["b_p"],
          "classifier.weight": w["w_c"], "classifier.bias": w["b_c"]}
    for i, lw in enumerate(w["layers"]):
        p = f"bert.encoder.layer.{i}."
        for j, nm in enumerate(("query", "key", "value")):
            sd[p + f"attention.self.{nm}.weight"] = lw["w_qkv"][j * H:(j + 1) * H]
            sd[p + f"attention.self.{nm}.bias"] = lw["b_qkv"][j * H:(j + 1) * H]
        sd[p + "attention.output.dense.weight"] = lw["w_o"]
        sd[p + "attention.output.dense.bias"] = lw["b_o"]
        sd[p + "attention.output.LayerNorm.weight"] = lw["ln1_g"]
        sd[p + "attention.output.LayerNorm.bias"] = lw["ln1_b"]
        sd[p + "intermediate.dense.weight"] = lw["w_1"]
        sd[p + "intermediate.dense.bias"] = lw["b_1"]
        sd[p + "output.dense.weight"] = lw["w_2"]
        sd[p + "output.dense.bias"] = lw["b_2"]
        sd[p + "output.LayerNorm.weight"] = lw["ln2_g"]
        sd[p + "output.LayerNorm.bias"] = lw["ln2_b"]
    missing = m.load_state_dict({k: t(v) for k, v in sd.items()}, strict=False)
    assert not [k for k in missing.missing_keys if "position_ids" not in k], missing.missing_keys
    return m


@pytest.mark.parametrize("cfg", [wl.TINY, ODD], ids=lambda c: c.name)
def test_whole_model_matches_hf_bert(cfg):
    """Library pin: HF BertForSequenceClassification (fp64, eager attention,
    padding mask) on the same weights and a zero-padded batch."""
    w = wl.make_weights(cfg, seed=7)
    L = 32
    lengths = np.array([20, 32, 1, 2, 9], np.int32)
    ids = wl.sample_token_ids(cfg, lengths, L, seed=11)
    m = _hf_model(cfg, w)
    mask = torch.tensor((np.arange(L)[None, :] < lengths[:, None]).astype(np.int64))
    with torch.no_grad():
        out = m(input_ids=torch.tensor(ids.astype(np.int64)), attention_mask=mask,
                token_type_ids=torch.zeros_like(mask), output_hidden_states=True)
    hf_logits = out.logits.numpy()
    hf_hidden = out.hidden_states[-1].numpy()
    ref = orc.forward_batch(cfg, w, ids, lengths)
    np.testing.assert_allclose(ref, hf_logits, rtol=0, atol=1e-12)
    for i, n in enumerate(lengths):
        h = orc.hidden_states(cfg, w, ids[i, :n])
        np.testing.assert_allclose(h, hf_hidden[i, :n], rtol=0, atol=1e-11)


def test_layer_matches_torch_transformer_encoder_layer():
    """Independent per-layer pin: torch.nn.TransformerEncoderLayer (post-LN,
    erf GELU, eps=1e-12, key padding mask) in fp64."""
    cfg = ODD
    w = wl.make_weights(cfg, seed=3)
    lw = w["layers"][0]
    H = cfg.hidden
    layer = torch.nn.TransformerEncoderLayer(H, cfg.heads, cfg.ffn, dropout=0.0, activation="gelu",
                                             layer_norm_eps=cfg.ln_eps, batch_first=True,
                                             norm_first=False).double().eval()
    t = lambda a: torch.tensor(np.asarray(a, np.float64))
    with torch.no_grad():
        layer.self_attn.in_proj_weight.copy_(t(lw["w_qkv"]))
        layer.self_attn.in_proj_bias.copy_(t(lw["b_qkv"]))
        layer.self_attn.out_proj.weight.copy_(t(lw["w_o"]))
        layer.self_attn.out_proj.bias.copy_(t(lw["b_o"]))
        layer.linear1.weight.copy_(t(lw["w_1"]))
        layer.linear1.bias.copy_(t(lw["b_1"]))
        layer.linear2.weight.copy_(t(lw["w_2"]))
        layer.linear2.bias.copy_(t(lw["b_2"]))
        layer.norm1.weight.copy_(t(lw["ln1_g"]))
        layer.norm1.bias.copy_(t(lw["ln1_b"]))
        layer.norm2.weight.copy_(t(lw["ln2_g"]))
        layer.norm2.bias.copy_(t(lw["ln2_b"]))
    rng = np.random.default_rng(5)
    L, n = 24, 17
    x = rng.standard_normal((L, H))
    kpm = torch.tensor(np.arange(L) >= n)[None, :]
    with torch.no_grad():
        y = layer(t(x)[None], src_key_padding_mask=kpm).numpy()[0]
    ours = orc.encoder_layer(cfg, lw, x[:n])
    np.testing.assert_allclose(ours, y[:n], rtol=0, atol=1e-12)
    ours_masked = orc.encoder_layer(cfg, lw, x, length=n)
    np.testing.assert_allclose(ours_masked[:n], y[:n], rtol=0, atol=1e-12)


def _attention_brute(q, k, v, heads):
    n, H = q.shape
    d = H // heads
    out = np.zeros((n, H))
    for j in range(heads):
        for a in range(n):
            s = [sum(q[a, j * d + c] * k[b, j * d + c] for c in range(d)) / math.sqrt(d) for b in range(n)]
            mx = max(s)
            e = [math.exp(x - mx) for x in s]
            z = sum(e)
            for c in range(d):
                out[a, j * d + c] = sum(e[b] * v[b, j * d + c] for b in range(n)) / z
    return out


@pytest.mark.parametrize("n", [1, 2, 5, 8])
def test_attention_brute_force(n):
    rng = np.random.default_rng(n)
    H, heads = 128, 2
    q, k, v = (rng.standard_normal((n, H)) for _ in range(3))
    np.testing.assert_allclose(orc.attention(q, k, v, heads), _attention_brute(q, k, v, heads),
                               rtol=0, atol=1e-13)


def test_attention_matches_torch_sdpa_with_mask():
    rng = np.random.default_rng(1)
    L, n, heads, d = 40, 23, 4, 64
    q, k, v = (rng.standard_normal((L, heads * d)) for _ in range(3))
    ours = orc.attention_masked(q, k, v, heads, n)
    t = lambda a: torch.tensor(a).reshape(L, heads, d).transpose(0, 1)
    mask = torch.tensor(np.arange(L) < n)[None, None, :].expand(heads, L, L)
    ref = torch.nn.functional.scaled_dot_product_attention(t(q), t(k), t(v), attn_mask=mask)
    ref = ref.transpose(0, 1).reshape(L, heads * d).numpy()
    np.testing.assert_allclose(ours, ref, rtol=0, atol=1e-13)


def test_attention_closed_forms():
    rng = np.random.default_rng(2)
    n, heads, d = 13, 2, 64
    H = heads * d
    q, k, v = (rng.standard_normal((n, H)) for _ in range(3))
    # q = 0: every weight is 1/n -> output = mean of the real V rows
    out = orc.attention(np.zeros_like(q), k, v, heads)
    np.testing.assert_allclose(out, np.broadcast_to(v.mean(axis=0), out.shape), rtol=0, atol=1e-14)
    # n = 1: softmax of one score is 1 -> output = V_0
    np.testing.assert_allclose(orc.attention(q[:1], k[:1], v[:1], heads), v[:1], rtol=0, atol=0)
    # permuting keys and values together leaves the output unchanged
    perm = rng.permutation(n)
    np.testing.assert_allclose(orc.attention(q, k[perm], v[perm], heads), orc.attention(q, k, v, heads),
                               rtol=0, atol=1e-13)
    # masked form: keys beyond the length do not matter, even huge ones
    kk, vv = k.copy(), v.copy()
    kk[7:] = 1e6
    vv[7:] = -1e6
    np.testing.assert_allclose(orc.attention_masked(q, kk, vv, heads, 7)[:7],
                               orc.attention(q[:7], k[:7], v[:7], heads), rtol=0, atol=1e-13)


def test_softmax_rows():
    rng = np.random.default_rng(3)
    s = rng.standard_normal((9, 31)) * 10
    p = orc.softmax_rows(s)
    np.testing.assert_allclose(p.sum(axis=1), 1.0, rtol=0, atol=1e-15)
    np.testing.assert_allclose(orc.softmax_rows(s + 123.0), p, rtol=0, atol=1e-13)  # shift invariance
    np.testing.assert_array_equal(np.argsort(s, axis=1, kind="stable"), np.argsort(p, axis=1, kind="stable"))


def test_gelu_closed_forms():
    # GELU(1) = Phi(1) (standard normal CDF at 1)
    assert abs(orc.gelu(np.array([1.0]))[0] - 0.8413447460685429) < 1e-15
    assert orc.gelu(np.array([0.0]))[0] == 0.0
    x = np.linspace(-6, 6, 101)
    np.testing.assert_allclose(orc.gelu(x) - orc.gelu(-x), x, rtol=0, atol=1e-14)  # z*Phi(z)+z*Phi(-z)... odd part
    # matches torch's erf GELU (library routine)
    np.testing.assert_allclose(orc.gelu(x), torch.nn.functional.gelu(torch.tensor(x)).numpy(), rtol=0, atol=1e-15)
    # and is NOT the tanh approximation (reading S2)
    tanh_form = torch.nn.functional.gelu(torch.tensor(x), approximate="tanh").numpy()
    assert np.max(np.abs(orc.gelu(x) - tanh_form)) > 1e-4


def test_layer_norm_invariants():
    rng = np.random.default_rng(4)
    y = rng.standard_normal((16, 768)) * 3 + 5
    H = y.shape[1]
    eps = 1e-12
    out = orc.layer_norm(y, np.ones(H), np.zeros(H), eps)
    np.testing.assert_allclose(out.mean(axis=1), 0.0, rtol=0, atol=1e-12)
    var_in = y.var(axis=1)
    np.testing.assert_allclose(out.var(axis=1), var_in / (var_in + eps), rtol=0, atol=1e-12)
    g, b = rng.standard_normal(H), rng.standard_normal(H)
    np.testing.assert_allclose(orc.layer_norm(y, g, b, eps), out * g + b, rtol=0, atol=1e-12)
    # library pin: torch layer_norm in fp64 (biased variance, eps inside the sqrt)
    ref = torch.nn.functional.layer_norm(torch.tensor(y), (H,), torch.tensor(g), torch.tensor(b), 1e-5).numpy()
    np.testing.assert_allclose(orc.layer_norm(y, g, b, 1e-5), ref, rtol=0, atol=1e-12)


def test_embedding_gather_exact():
    cfg = wl.TINY
    w = wl.make_weights(cfg, seed=1, unit_ln=True)
    tok = np.array([1, 7, 999, 0, 42])
    # with unit LN the embedding output is LN of the exact sum; check the sum itself via LN inverse
    x = orc.embed(cfg, w, tok)
    raw = w["word_emb"][tok].astype(np.float64) + w["pos_emb"][:5] + w["type_emb"][0]
    np.testing.assert_allclose(x, (raw - raw.mean(1, keepdims=True)) / np.sqrt(raw.var(1, keepdims=True) + cfg.ln_eps),
                               rtol=0, atol=1e-12)


@pytest.mark.parametrize("L", [32, 64, 128, 192, 256, 320, 384, 448, 512])
def test_padding_invariance(L):
    """The same request compiled at different L gives the same real-token
    outputs (north_star oracle check 3; reading S4/S5)."""
    cfg = wl.TINY
    w = wl.make_weights(cfg, seed=9)
    n = 19
    ids = wl.sample_token_ids(cfg, np.array([n]), L, seed=4)[0]
    h_ref = orc.hidden_states(cfg, w, ids[:n])
    logit_ref = orc.forward_request(cfg, w, ids[:n])
    garbage = ids.copy()
    garbage[n:] = 5  # ignored: positions >= len are treated as padding
    h, logits = orc.forward_padded(cfg, w, garbage, n)
    np.testing.assert_allclose(h[:n], h_ref, rtol=0, atol=1e-12)
    np.testing.assert_allclose(logits, logit_ref, rtol=0, atol=1e-12)
    assert np.all(np.isfinite(h))


def test_forward_batch_stops_at_empty_slot():
    cfg = wl.TINY
    w = wl.make_weights(cfg, seed=2)
    lengths = np.array([5, 3, 0, 4], np.int32)
    ids = wl.sample_token_ids(cfg, lengths, 8, seed=1)
    out = orc.forward_batch(cfg, w, ids, lengths)
    assert out.shape == (2, 2)


def test_label_tie_rule_and_argmax():
    """orc.label: argmax over the classes, the lowest index winning exact ties (reading S11)."""
    logits = np.array([[0.25, 0.25], [-1.0, 2.0], [3.0, -3.0], [0.0, 0.0]])
    np.testing.assert_array_equal(orc.label(logits), [0, 1, 0, 0])
    cfg = wl.TINY
    w = wl.make_weights(cfg, seed=3)
    lengths = np.array([7, 12, 3], np.int32)
    ids = wl.sample_token_ids(cfg, lengths, 16, seed=8)
    out = orc.forward_batch(cfg, w, ids, lengths)
    for i in range(3):
        assert orc.label(out[i]) == (0 if out[i, 0] >= out[i, 1] else 1)
