"""The fused family: the whole batch-1 forward as one persistent kernel (needs a B200).

csrc/encoder_fused.cu runs embedding, every layer and the head of a small runtime
(max_batch * L <= 256 tokens, L <= 128) as one grid of one CTA per SM executing a static
task graph (the batch-1 runtimes of PAPER.md:L282 §5).  These tests
pin it to the oracle end to end (tiny, BERT-base, BERT-large shapes; lengths 1 .. L) and
check its contract: split factors depend on the weight shape only and every other step is
per token or per (sequence, head), so a request's logits are bitwise equal on every fused
runtime L >= its length and in every batch bucket; the counters the tasks synchronise on
are reset by the kernel itself (repeated replays give identical logits).
"""
import numpy as np
import pytest
import torch

from oracle import encoder as orc
from paper_conf_icpp_tanlyl024_b200 import workload as wl

pytestmark = pytest.mark.gpu

_W = {}


def weights(arlo_lib, cfg):
    if cfg.name not in _W:
        w = wl.make_weights(cfg)
        _W[cfg.name] = (w, arlo_lib.Weights(cfg, arlo_lib.upload_weights(cfg, w, arlo_lib.BF16), arlo_lib.BF16))
    return _W[cfg.name]


def fused(arlo_lib, W, L, max_batch=1):
    rt = arlo_lib.Runtime(W, L, max_batch, arlo_lib.RUNTIME_FUSED)
    assert rt.family == arlo_lib.RUNTIME_FUSED
    assert rt.kernel_count(1) == 1  # the whole forward is one kernel node
    assert all(c > arlo_lib.FUSED_CODE for c in rt.gemm_tiles(1))
    return rt


def run(rt, ids_rows, lens):
    n = len(lens)
    x = np.zeros((rt.max_batch, rt.L), np.int32)
    ln = np.zeros((rt.max_batch,), np.int32)
    for i, (ids, m) in enumerate(zip(ids_rows, lens)):
        x[i, :m] = ids[:m]
        ln[i] = m
    out = np.zeros((rt.max_batch, 2), np.float32)
    rt.infer(x, ln, out)
    return out[:n]


@pytest.mark.parametrize("L", [16, 48, 64, 128])
def test_fused_tiny_parity(arlo_lib, L):
    cfg = wl.TINY
    w, W = weights(arlo_lib, cfg)
    rt = fused(arlo_lib, W, L)
    for j, n in enumerate(sorted(m for m in {1, 2, 15, 17, L // 2 + 1, L} if m <= L)):
        ids = wl.sample_token_ids(cfg, np.array([n]), n, seed=300 + j)[0]
        got = run(rt, [ids], [n])[0]
        ref = orc.forward_request(cfg, w, ids[:n])
        assert np.max(np.abs(got - ref)) <= 2e-2, (L, n, got, ref)
    rt.close()


@pytest.mark.parametrize("cfg_name,Ls,lens", [
    ("bert-base", (64, 128), (1, 37, 63, 64, 65, 100, 128)),
    ("bert-large", (64, 128), (2, 64, 127)),
])
def test_fused_parity_and_cross_L_bitwise(arlo_lib, cfg_name, Ls, lens):
    """Batch-1 fused runtimes: logits within 2e-2 of the oracle, bitwise equal across every fused
    runtime that can hold the request."""
    cfg = wl.CONFIGS[cfg_name]
    w, W = weights(arlo_lib, cfg)
    rts = {L: fused(arlo_lib, W, L) for L in Ls}
    for j, n in enumerate(lens):
        ids = wl.sample_token_ids(cfg, np.array([n]), n, seed=310 + j)[0]
        outs = [run(rts[L], [ids], [n])[0] for L in Ls if L >= n]
        for o in outs[1:]:
            np.testing.assert_array_equal(o, outs[0])
        ref = orc.forward_request(cfg, w, ids[:n])
        assert np.max(np.abs(outs[0] - ref)) <= 2e-2, (n, outs[0], ref)
    for rt in rts.values():
        rt.close()


def test_fused_buckets_bitwise_and_parity(arlo_lib):
    """max_batch * L = 256: buckets 1, 2, 4 at L = 64; each request's logits are bitwise those of
    the batch-1 run and within 2e-2 of the oracle; empty slots do not disturb real ones."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg)
    rt4 = fused(arlo_lib, W, 64, max_batch=4)
    rt1 = fused(arlo_lib, W, 64)
    assert [rt4.bucket_of(n) for n in (1, 2, 3, 4)] == [1, 2, 4, 4]
    lens = [64, 1, 33, 50]
    ids = wl.sample_token_ids(cfg, np.array(lens), 64, seed=320)
    singles = [run(rt1, [ids[i]], [lens[i]])[0] for i in range(4)]
    for n in (1, 2, 3, 4):
        got = run(rt4, [ids[i] for i in range(n)], lens[:n])
        for i in range(n):
            np.testing.assert_array_equal(got[i], singles[i])
    for i in range(4):
        ref = orc.forward_request(cfg, w, ids[i][:lens[i]])
        assert np.max(np.abs(singles[i] - ref)) <= 2e-2
    rt1.close()
    rt4.close()


def test_fused_replays_identical_and_device_io(arlo_lib):
    """The task counters reset themselves: 20 back-to-back replays (arlo_enqueue on device
    buffers) give bitwise the logits of the first synchronous run."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg)
    rt = fused(arlo_lib, W, 128, max_batch=2)
    lens = np.array([128, 77], np.int32)
    ids = wl.sample_token_ids(cfg, lens, 128, seed=330)
    first = run(rt, list(ids), list(lens))
    d_ids = torch.from_numpy(ids).cuda()
    d_len = torch.from_numpy(lens).cuda()
    d_out = torch.zeros((20, 2, 2), dtype=torch.float32, device="cuda")
    for r in range(20):
        rt.enqueue(2, d_ids, d_len, d_out[r])
    torch.cuda.synchronize()
    for r in range(20):
        np.testing.assert_array_equal(d_out[r].cpu().numpy(), first)
    rt.close()


def test_fused_against_throughput_family(arlo_lib):
    """The fused and tile families agree to bf16 rounding and on every label that is not a near-tie."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg)
    fu = fused(arlo_lib, W, 128)
    thr = arlo_lib.Runtime(W, 128, 1, arlo_lib.RUNTIME_THROUGHPUT)
    lengths = wl.sample_lengths(12, seed=340, lo=0, hi=128)
    ids = wl.sample_token_ids(cfg, lengths, 128, seed=341)
    for i in range(12):
        a = run(fu, [ids[i]], [int(lengths[i])])[0]
        b = run(thr, [ids[i]], [int(lengths[i])])[0]
        assert np.max(np.abs(a - b)) <= 2e-2
        if abs(a[0] - a[1]) > 4e-2:
            assert np.argmax(a) == np.argmax(b)
    fu.close()
    thr.close()


def test_fused_rejects_unsupported_shapes(arlo_lib):
    cfg = wl.BERT_BASE
    _, W = weights(arlo_lib, cfg)
    for L, mb in ((256, 1), (128, 4), (64, 8)):
        with pytest.raises(arlo_lib.ArloError) as e:
            arlo_lib.Runtime(W, L, mb, arlo_lib.RUNTIME_FUSED)
        assert e.value.code == arlo_lib.EINVAL


def test_fused_bad_token_id_reported(arlo_lib):
    cfg = wl.TINY
    _, W = weights(arlo_lib, cfg)
    rt = fused(arlo_lib, W, 32)
    ids = torch.zeros((1, 32), dtype=torch.int32, device="cuda")
    ids[0, 3] = cfg.vocab + 5
    out = torch.zeros((1, 2), dtype=torch.float32, device="cuda")
    with pytest.raises(arlo_lib.ArloError):
        rt.infer(ids, torch.tensor([8], dtype=torch.int32, device="cuda"), out)
    ok = wl.sample_token_ids(cfg, np.array([8]), 32, seed=350)
    got = run(rt, [ok[0]], [8])[0]  # the runtime stays usable (err flag and counters reset)
    assert np.all(np.isfinite(got))
    rt.close()
