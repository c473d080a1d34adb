"""The split-K runtime family: split-K weight-streaming GEMMs for batch 1 (needs a B200).

PAPER.md:L282 §5 runs every runtime at batch 1.  The split-K family serves that setting
with the split-K kernel (csrc/gemm_splitk.cu); these tests pin it to the oracle per op and
end to end, and check its contract: the split factor depends on the weight shape only, so
a request's logits are bitwise equal on every latency runtime L >= its length, and every
tile width gives bitwise the same rows.  Against the throughput family (single K chain)
the logits agree to bf16 rounding; the labels agree wherever the oracle's top-2 margin is
not a near-tie (reading S11).
"""
import numpy as np
import pytest
import torch

from oracle import encoder as orc
from paper_conf_icpp_tanlyl024_b200 import workload as wl

pytestmark = pytest.mark.gpu


def rnd(shape, seed, std=1.0):
    return wl.round_to_bf16(np.random.default_rng(seed).standard_normal(shape).astype(np.float32) * std)


def bf16_dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.float32)).to("cuda", torch.bfloat16)


SHAPES = [(64, 2304, 768), (64, 768, 3072), (1, 768, 768), (200, 768, 768), (512, 3072, 768),
          (33, 1024, 4096), (128, 4096, 1024), (7, 384, 128), (300, 128, 512)]


@pytest.mark.parametrize("M,N,K", SHAPES)
@pytest.mark.parametrize("epi", [0, 1, 2])
def test_splitk_gemm_parity(arlo_lib, M, N, K, epi):
    A = rnd((M, K), 11)
    W = rnd((N, K), 12, 0.02)
    b = rnd((N,), 13, 0.02)
    R = rnd((M, N), 14)
    ref = orc.linear(A, W, b)
    if epi == 1:
        ref = orc.gelu(ref)
    if epi == 2:
        ref = ref + R
    out = torch.full((M, N), float("nan"), device="cuda", dtype=torch.bfloat16)
    arlo_lib.op_gemm(arlo_lib.BF16, bf16_dev(A), bf16_dev(W), torch.from_numpy(b).cuda(), out, epi=epi,
                     residual=bf16_dev(R) if epi == 2 else None, force_bn=arlo_lib.SPLITK_CODE + 32)
    torch.cuda.synchronize()
    np.testing.assert_allclose(out.float().cpu().numpy().astype(np.float64), ref, rtol=8e-3, atol=8e-3)


@pytest.mark.parametrize("epi", [0, 1, 2])
def test_splitk_tile_widths_and_M_bitwise(arlo_lib, epi):
    """Every split-K tile width gives bitwise the same rows, and a row does not depend on M
    (the same (N, K) always uses the same split factor and reduction order)."""
    M, N, K = 300, 768, 3072
    A, W = bf16_dev(rnd((M, K), 21)), bf16_dev(rnd((N, K), 22, 0.02))
    b = torch.from_numpy(rnd((N,), 23, 0.02)).cuda()
    R = bf16_dev(rnd((M, N), 24))
    outs = []
    for bn in (32, 64, 128):
        o = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
        arlo_lib.op_gemm(arlo_lib.BF16, A, W, b, o, epi=epi, residual=R if epi == 2 else None,
                         force_bn=arlo_lib.SPLITK_CODE + bn)
        outs.append(o)
    for m in (1, 64, 77):
        o = torch.empty((m, N), device="cuda", dtype=torch.bfloat16)
        arlo_lib.op_gemm(arlo_lib.BF16, A[:m].contiguous(), W, b, o, epi=epi,
                         residual=R[:m].contiguous() if epi == 2 else None, force_bn=arlo_lib.SPLITK_CODE + 32)
        outs.append(o)
    torch.cuda.synchronize()
    for o in outs[1:3]:
        assert torch.equal(o, outs[0])
    for o in outs[3:]:
        assert torch.equal(o, outs[0][:o.shape[0]])


def _latency_runtime(arlo_lib, W, L):
    rt = arlo_lib.Runtime(W, L, 1, arlo_lib.RUNTIME_SPLITK)
    assert rt.family == arlo_lib.RUNTIME_SPLITK
    assert all(c > arlo_lib.SPLITK_CODE for c in rt.gemm_tiles(1))
    return rt


_W = {}


def weights(arlo_lib, cfg):
    if cfg.name not in _W:
        w = wl.make_weights(cfg)
        _W[cfg.name] = (w, arlo_lib.Weights(cfg, arlo_lib.upload_weights(cfg, w, arlo_lib.BF16), arlo_lib.BF16))
    return _W[cfg.name]


def one(rt, ids, n):
    L = rt.L
    x = np.zeros((1, L), np.int32)
    x[0, :n] = ids[:n]
    out = np.zeros((1, 2), np.float32)
    rt.infer(x, np.array([n], np.int32), out)
    return out[0]


@pytest.mark.parametrize("cfg_name", ["bert-base", "bert-large"])
def test_latency_runtime_parity_and_cross_L_bitwise(arlo_lib, cfg_name):
    """Batch-1 runtimes L = 64..512: logits within 2e-2 of the oracle, and bitwise equal across
    every latency runtime that can hold the request."""
    cfg = wl.CONFIGS[cfg_name]
    w, W = weights(arlo_lib, cfg)
    Ls = (64, 128, 256, 512) if cfg_name == "bert-base" else (128, 512)
    rts = {L: _latency_runtime(arlo_lib, W, L) for L in Ls}
    lens = [1, 37, 64] if cfg_name == "bert-base" else [2, 100]
    for j, n in enumerate(lens):
        ids = wl.sample_token_ids(cfg, np.array([n]), n, seed=100 + j)[0]
        outs = [one(rts[L], ids, n) for L in Ls if L >= n]
        for o in outs[1:]:
            np.testing.assert_array_equal(o, outs[0])
        ref = orc.forward_request(cfg, w, ids[:n])
        assert np.max(np.abs(outs[0] - ref)) <= 2e-2, (n, outs[0], ref)
    n = 512 if cfg_name == "bert-base" else 300
    ids = wl.sample_token_ids(cfg, np.array([n]), n, seed=120)[0]
    got = one(rts[512], ids, n)
    ref = orc.forward_request(cfg, w, ids[:n])
    assert np.max(np.abs(got - ref)) <= 2e-2
    for rt in rts.values():
        rt.close()


def test_latency_vs_throughput_family_labels(arlo_lib):
    """The two families agree to bf16 rounding and on every label that is not a near-tie."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg)
    lat = _latency_runtime(arlo_lib, W, 128)
    thr = arlo_lib.Runtime(W, 128, 8)
    assert thr.family == arlo_lib.RUNTIME_THROUGHPUT
    lengths = wl.sample_lengths(24, seed=130, lo=0, hi=128)
    ids = wl.sample_token_ids(cfg, lengths, 128, seed=131)
    for s in range(0, 24, 8):
        out_t = np.zeros((8, 2), np.float32)
        thr.infer(ids[s:s + 8], lengths[s:s + 8], out_t)
        for i in range(8):
            o_l = one(lat, ids[s + i], int(lengths[s + i]))
            assert np.max(np.abs(o_l - out_t[i])) <= 2e-2
            if abs(o_l[0] - o_l[1]) > 4e-2:
                assert np.argmax(o_l) == np.argmax(out_t[i])
    lat.close()
    thr.close()
