"""End-to-end parity of per-length runtimes (arlo_runtime_create / arlo_infer)
against the fp64 oracle, plus the cross-L invariants (needs a B200).

Tolerances come from the north_star: logits within 2e-2 of the fp64 oracle in
bf16, within 1e-4 in fp32 check mode; argmax labels agree across every L.
"""
import numpy as np
import pytest
import torch

from oracle import encoder as orc
from paper_conf_icpp_tanlyl024_b200 import workload as wl

pytestmark = pytest.mark.gpu

_CACHE = {}


def weights(arlo_lib, cfg, dtype, seed=0):
    key = (cfg.name, dtype, seed)
    if key not in _CACHE:
        w = wl.make_weights(cfg, seed=seed)
        W = arlo_lib.Weights(cfg, arlo_lib.upload_weights(cfg, w, dtype), dtype)
        _CACHE[key] = (w, W)
    return _CACHE[key]


def run(arlo_lib, W, L, max_batch, ids, lengths, where="host"):
    rt = arlo_lib.Runtime(W, L, max_batch)
    C = W.cfg.num_labels
    ids_full = np.zeros((max_batch, L), np.int32)
    ids_full[:ids.shape[0]] = ids
    len_full = np.zeros(max_batch, np.int32)
    len_full[:len(lengths)] = lengths
    if where == "host":
        out = np.full((max_batch, C), np.nan, np.float32)
        rt.infer(ids_full, len_full, out)
    else:
        out_d = torch.full((max_batch, C), float("nan"), device="cuda")
        rt.infer(torch.from_numpy(ids_full).cuda(), torch.from_numpy(len_full).cuda(), out_d)
        out = out_d.cpu().numpy()
    rt.close()
    return out


@pytest.mark.parametrize("dtype,tol", [(1, 1e-4), (0, 2e-2)])
def test_tiny_config_parity(arlo_lib, dtype, tol):
    """configs[0]: tiny encoder L=32, batch 4 (BASELINE.json)."""
    cfg = wl.TINY
    w, W = weights(arlo_lib, cfg, dtype)
    lengths = np.array([32, 17, 1, 2], np.int32)
    ids = wl.sample_token_ids(cfg, lengths, 32, seed=5)
    out = run(arlo_lib, W, 32, 4, ids, lengths)
    ref = orc.forward_batch(cfg, w, ids, lengths)
    assert np.max(np.abs(out - ref)) <= tol, np.max(np.abs(out - ref))


@pytest.mark.parametrize("dtype,tol", [(1, 1e-4), (0, 2e-2)])
def test_bert_base_parity_ragged(arlo_lib, dtype, tol):
    """BERT-base, L=128, ragged lengths and an empty tail slot; device pointers."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg, dtype)
    lengths = np.array([128, 3, 77, 64, 65, 1], np.int32)
    ids = wl.sample_token_ids(cfg, lengths, 128, seed=6)
    out = run(arlo_lib, W, 128, 8, ids, lengths, where="device")
    ref = orc.forward_batch(cfg, w, ids, lengths)
    assert np.all(np.isnan(out[6:]))  # untouched rows past n
    err = np.max(np.abs(out[:6] - ref))
    assert err <= tol, err


def test_bert_large_parity_sample(arlo_lib):
    cfg = wl.BERT_LARGE
    w, W = weights(arlo_lib, cfg, 0)
    lengths = np.array([256, 40, 129], np.int32)
    ids = wl.sample_token_ids(cfg, lengths, 256, seed=7)
    out = run(arlo_lib, W, 256, 4, ids, lengths)
    ref = orc.forward_batch(cfg, w, ids, lengths)
    assert np.max(np.abs(out[:3] - ref)) <= 2e-2


def test_cross_length_bitwise_and_labels(arlo_lib):
    """The same requests on runtimes L = 64..512: logits bitwise equal, labels equal
    (north_star: argmax labels agree across all L)."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg, 0)
    lengths = wl.sample_lengths(8, seed=11, lo=0, hi=64)
    ids = wl.sample_token_ids(cfg, lengths, 64, seed=12)
    outs = {}
    for L in (64, 128, 192, 256, 512):
        ids_L = np.zeros((8, L), np.int32)
        ids_L[:, :64] = ids
        outs[L] = run(arlo_lib, W, L, 8, ids_L, lengths)
    for L in outs:
        np.testing.assert_array_equal(outs[L], outs[64])
        np.testing.assert_array_equal(np.argmax(outs[L], 1), np.argmax(outs[64], 1))
    ref = orc.forward_batch(cfg, w, ids, lengths)
    assert np.max(np.abs(outs[64] - ref)) <= 2e-2


def test_batch_buckets_give_identical_rows(arlo_lib):
    """A request's logits do not depend on how many others share its batch (bucket 1..32)."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg, 0)
    lengths = wl.sample_lengths(32, seed=21, lo=0, hi=128)
    ids = wl.sample_token_ids(cfg, lengths, 128, seed=22)
    rt = arlo_lib.Runtime(W, 128, 32)
    full = np.zeros((32, 2), np.float32)
    rt.infer(ids, lengths, full)
    for n in (1, 2, 3, 5, 16, 31):
        len_n = np.zeros(32, np.int32)
        len_n[:n] = lengths[:n]
        part = np.zeros((32, 2), np.float32)
        rt.infer(ids, len_n, part)
        np.testing.assert_array_equal(part[:n], full[:n])
    rt.close()


def test_full_size_sampled_parity(arlo_lib):
    """BASELINE configs[1] at full size (BERT-base L=512, batch 32, the bench launch
    configuration): sampled requests checked one by one against the oracle."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg, 0)
    lengths = wl.sample_lengths(32, seed=31, lo=448, hi=512)
    lengths[5] = 512
    lengths[9] = 449
    ids = wl.sample_token_ids(cfg, lengths, 512, seed=32)
    out = run(arlo_lib, W, 512, 32, ids, lengths)
    for i in (0, 5, 9, 31):
        ref = orc.forward_request(cfg, w, ids[i, :lengths[i]])
        assert np.max(np.abs(out[i] - ref)) <= 2e-2, (i, out[i], ref)
    assert np.all(np.isfinite(out))


def test_error_codes(arlo_lib):
    cfg = wl.TINY
    w, W = weights(arlo_lib, cfg, 0)
    rt = arlo_lib.Runtime(W, 32, 4)
    ids = np.zeros((4, 32), np.int32)
    logits = np.zeros((4, 2), np.float32)
    with pytest.raises(arlo_lib.ArloError) as e:
        rt.infer(ids, np.array([33, 0, 0, 0], np.int32), logits)
    assert e.value.code == arlo_lib.ETOOLONG
    bad = ids.copy()
    bad[0, 2] = cfg.vocab
    with pytest.raises(arlo_lib.ArloError) as e:
        rt.infer(bad, np.array([5, 0, 0, 0], np.int32), logits)
    assert e.value.code == arlo_lib.EINVAL
    # device ids: the embedding kernel flags it
    with pytest.raises(arlo_lib.ArloError) as e:
        rt.infer(torch.from_numpy(bad).cuda(), np.array([5, 0, 0, 0], np.int32), logits)
    assert e.value.code == arlo_lib.EINVAL
    # out-of-range ids beyond the length are ignored
    bad2 = ids.copy()
    bad2[0, 10:] = -7
    rt.infer(bad2, np.array([5, 0, 0, 0], np.int32), logits)
    with pytest.raises(arlo_lib.ArloError) as e:
        arlo_lib.Runtime(W, 24, 4)  # L % 16 != 0
    assert e.value.code == arlo_lib.EINVAL
    rt.close()


def test_enqueue_matches_infer(arlo_lib):
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg, 0)
    lengths = wl.sample_lengths(12, seed=41, lo=0, hi=256)
    ids = wl.sample_token_ids(cfg, lengths, 256, seed=42)
    rt = arlo_lib.Runtime(W, 256, 16)
    a = np.zeros((16, 2), np.float32)
    len16 = np.zeros(16, np.int32)
    len16[:12] = lengths
    ids16 = np.zeros((16, 256), np.int32)
    ids16[:12] = ids
    rt.infer(ids16, len16, a)
    out = torch.zeros((12, 2), device="cuda")
    s = torch.cuda.Stream()
    rt.set_stream(s)
    rt.enqueue(12, torch.from_numpy(ids).cuda(), torch.from_numpy(lengths).cuda(), out)
    s.synchronize()
    np.testing.assert_array_equal(out.cpu().numpy(), a[:12])
    # embedding + 5 or 7 per layer (LayerNorm fold / kernels) + pooler + classifier
    assert rt.kernel_count(12) in (3 + 5 * cfg.layers, 3 + 7 * cfg.layers)
    rt.close()


@pytest.mark.parametrize("L,max_batch", [(64, 8), (256, 4), (512, 32)])
def test_cls_only_last_layer_is_bitwise(arlo_lib, monkeypatch, L, max_batch):
    """The CLS-only last layer (out-proj/LN/FFN on the b position-0 rows, row stride
    L*H) gives bitwise the logits of the full static-shape last layer."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg, 0)
    lengths = wl.sample_lengths(max_batch, seed=51, lo=0, hi=L)
    lengths[0] = L
    ids = wl.sample_token_ids(cfg, lengths, L, seed=52)
    pruned = run(arlo_lib, W, L, max_batch, ids, lengths)
    monkeypatch.setenv("ARLO_NO_CLS_PRUNE", "1")
    full = run(arlo_lib, W, L, max_batch, ids, lengths)
    np.testing.assert_array_equal(pruned, full)
    ref = orc.forward_batch(cfg, w, ids, lengths)
    assert np.max(np.abs(pruned - ref)) <= 2e-2


@pytest.mark.gpu
def test_autotuned_tiles_are_bitwise_the_analytic_choice(arlo_lib, monkeypatch):
    """Build-time tile selection (pick_tile) changes only which tile codes the graphs use: the
    logits of an autotuned runtime equal those of one built with the analytic chooser bit for bit,
    and every selected code is a valid tile code."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg, 0)
    L, mb = 128, 32
    lengths = wl.sample_lengths(mb, seed=21, lo=0, hi=L)
    ids = wl.sample_token_ids(cfg, lengths, L, seed=22)
    rt = arlo_lib.Runtime(W, L, mb)
    tiles = {n: rt.gemm_tiles(n) for n in (1, 8, 32)}
    rt.close()
    valid = {-256, -192, -128, 256, 192, 128, 96, 64, 1016, 1032, 1064}
    assert all(c in valid for codes in tiles.values() for c in codes), tiles
    out_tuned = run(arlo_lib, W, L, mb, ids, lengths)
    monkeypatch.setenv("ARLO_NO_AUTOTUNE", "1")
    out_plain = run(arlo_lib, W, L, mb, ids, lengths)
    assert np.array_equal(out_tuned, out_plain)


@pytest.mark.parametrize("dtype", [0, 1])
def test_head_classifier_in_pooler_is_bitwise(arlo_lib, monkeypatch, dtype):
    """ARLO_HEAD_IN_POOLER=1: the classifier runs in the pooler's last CTA of each 8-sequence group
    (one launch less per forward); its logits are bitwise those of the separate classifier kernel
    (the default), for groups of 8 and a ragged last group, over repeated replays (the arrival
    counters reset themselves)."""
    monkeypatch.setenv("ARLO_HEAD_IN_POOLER", "1")
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg, dtype)
    lengths = wl.sample_lengths(21, seed=61, lo=0, hi=128)
    ids = wl.sample_token_ids(cfg, lengths, 128, seed=62)
    n, L, mb = len(lengths), 128, 24
    ids_full = np.zeros((mb, L), np.int32)
    ids_full[:n] = ids
    len_full = np.zeros(mb, np.int32)
    len_full[:n] = lengths
    rt = arlo_lib.Runtime(W, L, mb)
    fused = []
    for _ in range(3):  # same runtime: the counters must have reset after each forward
        out = np.full((mb, 2), np.nan, np.float32)
        rt.infer(ids_full, len_full, out)
        fused.append(out[:n].copy())
    k_fused = rt.kernel_count(n)
    rt.close()
    monkeypatch.delenv("ARLO_HEAD_IN_POOLER")
    rt2 = arlo_lib.Runtime(W, L, mb)
    two = np.full((mb, 2), np.nan, np.float32)
    rt2.infer(ids_full, len_full, two)
    assert rt2.kernel_count(n) == k_fused + 1
    rt2.close()
    for f in fused:
        np.testing.assert_array_equal(f, two[:n])
    ref = orc.forward_batch(cfg, w, ids, lengths)
    assert np.max(np.abs(two[:n] - ref)) <= (2e-2 if dtype == 0 else 1e-4)
