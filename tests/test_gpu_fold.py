"""The LayerNorm fold of the throughput runtimes (needs a B200).

The bf16 throughput runtimes launch no LayerNorm kernel (BERT post-LN, PAPER.md:L422 [17]; SURVEY
§8(a) rows a5/a8): a residual GEMM (out-projection, FFN2) writes y = (x W^T + b) + LN(r) and the
per-row statistics of y in 32-column granules; the GEMM consuming LN(y) (QKV, FFN1) runs on y with
W' = bf16(W * gamma) and applies rstd * acc - rstd * mean * s + c in its epilogue
(include/arlo_ops.h arlo_op_gemm_fold).  These tests pin each epilogue to the oracle's LayerNorm and
linear maps, the statistics to their definition, and the tile-shape invariance every runtime relies
on (a row's bits do not depend on the tile width, the kernel or M).
"""
import numpy as np
import pytest
import torch

from oracle import encoder as orc
from paper_conf_icpp_tanlyl024_b200 import workload as wl

pytestmark = pytest.mark.gpu


def rnd(shape, seed, std=1.0, mean=0.0):
    return wl.round_to_bf16((np.random.default_rng(seed).standard_normal(shape) * std + mean).astype(np.float32))


def bf(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.float32)).to("cuda", torch.bfloat16)


def f32(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.float32)).cuda()


def granule_stats(y):
    """Definition of the statistics: per row, per 32 columns, (sum y, sum y^2) in fp64; [rows, G, 2]."""
    M, H = y.shape
    g = y.astype(np.float64).reshape(M, H // 32, 32)
    return np.stack([g.sum(-1), (g * g).sum(-1)], -1)


def gm(st):
    """Row-major [rows, G, 2] statistics -> the kernels' granule-major [G, rows, 2] layout."""
    return np.ascontiguousarray(np.transpose(st, (1, 0, 2)))


def ln_from_stats(y, st, gamma, beta, eps):
    """LayerNorm of y with mean / variance from granule statistics (var = E[y^2] - mean^2)."""
    H = y.shape[1]
    mean = st[..., 0].sum(-1) / H
    var = np.maximum(st[..., 1].sum(-1) / H - mean * mean, 0)
    return (y - mean[:, None]) / np.sqrt(var[:, None] + eps) * gamma + beta


CODES = [0, 64, 128, 192, 256, -128, -192, -256, 1016, 1032, 1064]


@pytest.mark.parametrize("M,N,K", [(256, 768, 768), (300, 768, 3072), (64, 1024, 1024), (4096, 768, 768)])
def test_resid_ln_epilogue_and_statistics(arlo_lib, M, N, K):
    eps = 1e-12
    A, W, b = rnd((M, K), 1), rnd((N, K), 2, 0.02), rnd((N,), 3, 0.02)
    R = rnd((M, N), 4, 1.5, 0.3)  # a residual stream with a non-zero mean
    g, be = rnd((N,), 5, 0.1, 1.0), rnd((N,), 6, 0.1)
    st_r = granule_stats(R).astype(np.float32)
    out = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
    st_out = torch.full((N // 32, M, 2), float("nan"), device="cuda")
    arlo_lib.op_gemm_fold(bf(A), bf(W), f32(b), out, arlo_lib.EPI_RESID_LN, v1=f32(g), v2=f32(be), st_in=f32(gm(st_r)),
                          st_out=st_out, eps=eps, residual=bf(R))
    torch.cuda.synchronize()
    y = out.float().cpu().numpy()
    ref = orc.linear(A, W, b) + ln_from_stats(R.astype(np.float64), st_r.astype(np.float64), g, be, eps)
    np.testing.assert_allclose(y, ref, rtol=1e-2, atol=2e-2)
    # the reading-S3 LayerNorm (two-pass) agrees with the statistics-based one on this data
    np.testing.assert_allclose(orc.layer_norm(R.astype(np.float64), g, be, eps),
                               ln_from_stats(R.astype(np.float64), st_r.astype(np.float64), g, be, eps), atol=1e-4)
    np.testing.assert_allclose(st_out.cpu().numpy(), gm(granule_stats(y)), rtol=2e-6, atol=1e-4)
    # st_in = NULL: plain residual
    out2 = torch.empty_like(out)
    arlo_lib.op_gemm_fold(bf(A), bf(W), f32(b), out2, arlo_lib.EPI_RESID_LN, v1=f32(g), v2=f32(be), residual=bf(R))
    torch.cuda.synchronize()
    np.testing.assert_allclose(out2.float().cpu().numpy(), orc.linear(A, W, b) + R, rtol=1e-2, atol=2e-2)


@pytest.mark.parametrize("epi", [3, 4])
@pytest.mark.parametrize("M,N,K", [(256, 2304, 768), (333, 3072, 768), (64, 4096, 1024), (4096, 3072, 768)])
def test_lnfold_epilogue_is_layernorm_then_linear(arlo_lib, epi, M, N, K):
    """GEMM on y with the folded weights == Linear(LN(y)) (+ GELU), the oracle's order of steps."""
    eps = 1e-12
    Y = rnd((M, K), 11, 1.2, -0.2)
    W, b = rnd((N, K), 12, 0.02), rnd((N,), 13, 0.02)
    g, be = rnd((K,), 14, 0.1, 1.0), rnd((K,), 15, 0.1)
    Wf = wl.round_to_bf16((W * g[None, :]).astype(np.float32))
    s = Wf.astype(np.float64).sum(1).astype(np.float32)
    c = (W.astype(np.float64) @ be.astype(np.float64) + b).astype(np.float32)
    st = granule_stats(Y).astype(np.float32)
    out = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
    arlo_lib.op_gemm_fold(bf(Y), bf(Wf), f32(s), out, epi, v1=f32(c), st_in=f32(gm(st)), eps=eps)
    torch.cuda.synchronize()
    ref = orc.linear(orc.layer_norm(Y.astype(np.float64), g, be, eps), W, b)
    if epi == 4:
        ref = orc.gelu(ref)
    np.testing.assert_allclose(out.float().cpu().numpy(), ref, rtol=2e-2, atol=2e-2)


@pytest.mark.parametrize("epi", [3, 4, 5])
def test_fold_epilogues_bitwise_across_tiles_and_M(arlo_lib, epi):
    """Every tile code (single CTA, CTA pair, skinny) gives bitwise the same rows and statistics, and a
    row's result does not depend on M: the runtimes' cross-L / cross-bucket contract."""
    M, K = 300, 768
    N = 768 if epi == 5 else 3072
    A = bf(rnd((M, K), 21, 1.1, 0.1))
    W = bf(rnd((N, K), 22, 0.02))
    v0, v1, v2 = f32(rnd((N,), 23, 0.02)), f32(rnd((N,), 24, 0.1, 1.0)), f32(rnd((N,), 25, 0.1))
    R = bf(rnd((M, N), 26, 1.3)) if epi == 5 else None
    Hs = N if epi == 5 else K
    st_rows = granule_stats((R if epi == 5 else A).float().cpu().numpy()).astype(np.float32)
    outs, sts = [], []
    for code in CODES:
        if code and N % abs(code % 1000 if code > 1000 else code):
            continue
        for m in (M, 64, 129):
            o = torch.empty((m, N), device="cuda", dtype=torch.bfloat16)
            so = torch.zeros((N // 32, m, 2), device="cuda") if epi == 5 else None
            arlo_lib.op_gemm_fold(A[:m].contiguous(), W, v0, o, epi, v1=v1, v2=v2 if epi == 5 else None,
                                  st_in=f32(gm(st_rows[:m])), st_out=so, eps=1e-12,
                                  residual=R[:m].contiguous() if epi == 5 else None, force_bn=code)
            outs.append(o)
            sts.append(so)
    torch.cuda.synchronize()
    ref = outs[0]
    for o in outs[1:]:
        assert torch.equal(o, ref[:o.shape[0]])
    if epi == 5:
        for s_ in sts[1:]:
            assert torch.equal(s_, sts[0][:, :s_.shape[1]])
    assert Hs % 32 == 0


_W = {}


def weights(arlo_lib, cfg):
    if cfg.name not in _W:
        w = wl.make_weights(cfg)
        _W[cfg.name] = (w, arlo_lib.Weights(cfg, arlo_lib.upload_weights(cfg, w, arlo_lib.BF16), arlo_lib.BF16))
    return _W[cfg.name]


def run(rt, ids_rows, lens):
    x = np.zeros((rt.max_batch, rt.L), np.int32)
    ln = np.zeros((rt.max_batch,), np.int32)
    for i, (ids, m) in enumerate(zip(ids_rows, lens)):
        x[i, :m] = ids[:m]
        ln[i] = m
    out = np.zeros((rt.max_batch, 2), np.float32)
    rt.infer(x, ln, out)
    return out[:len(lens)]


@pytest.mark.parametrize("cfg_name", ["tiny", "bert-base", "bert-large"])
def test_latency_family_parity_cross_L_and_buckets(arlo_lib, cfg_name):
    """LATENCY family (LayerNorm fold): within 2e-2 of the oracle, bitwise equal across runtimes
    L >= len and across batch buckets (cross-L contract), CLS-only last layer included."""
    cfg = wl.CONFIGS[cfg_name]
    w, W = weights(arlo_lib, cfg)
    Ls = (64, 128, 512) if cfg_name != "bert-large" else (128, 256)
    rts = {L: arlo_lib.Runtime(W, L, 1, arlo_lib.RUNTIME_LATENCY) for L in Ls}
    assert all(rt.family == arlo_lib.RUNTIME_LATENCY for rt in rts.values())
    rt8 = arlo_lib.Runtime(W, Ls[0], 8, arlo_lib.RUNTIME_LATENCY)
    lens = [1, 37, Ls[0]] + ([100, 300] if Ls[-1] >= 300 else [100])
    for j, n in enumerate(lens):
        ids = wl.sample_token_ids(cfg, np.array([n]), n, seed=410 + j)[0]
        outs = [run(rts[L], [ids], [n])[0] for L in Ls if L >= n]
        for o in outs[1:]:
            np.testing.assert_array_equal(o, outs[0])
        ref = orc.forward_request(cfg, w, ids[:n])
        assert np.max(np.abs(outs[0] - ref)) <= 2e-2, (n, outs[0], ref)
        if n <= Ls[0]:  # bucket 8 with other requests around it: bitwise the batch-1 result
            others = wl.sample_token_ids(cfg, np.array([Ls[0]] * 7), Ls[0], seed=430 + j)
            got = run(rt8, [ids] + list(others), [n] + [Ls[0] - 3 * k for k in range(7)])
            np.testing.assert_array_equal(got[0], outs[0])
    for rt in list(rts.values()) + [rt8]:
        rt.close()


def test_runtime_fold_against_unfolded(arlo_lib):
    """LATENCY (LayerNorm fold) and THROUGHPUT (LayerNorm kernels) runtimes: both within 2e-2 of the
    oracle, labels equal wherever not a near-tie, two LayerNorm launches per layer fewer."""
    cfg = wl.BERT_BASE
    w, W = weights(arlo_lib, cfg)
    folded = arlo_lib.Runtime(W, 128, 8, arlo_lib.RUNTIME_LATENCY)
    plain = arlo_lib.Runtime(W, 128, 8)
    assert folded.kernel_count(8) < plain.kernel_count(8)  # 2 LayerNorm launches per layer fewer
    lengths = wl.sample_lengths(8, seed=401, lo=0, hi=128)
    ids = wl.sample_token_ids(cfg, lengths, 128, seed=402)
    a, b = np.zeros((8, 2), np.float32), np.zeros((8, 2), np.float32)
    folded.infer(ids, lengths, a)
    plain.infer(ids, lengths, b)
    for i in range(8):
        ref = orc.forward_request(cfg, w, ids[i][:lengths[i]])
        assert np.max(np.abs(a[i] - ref)) <= 2e-2
        assert np.max(np.abs(b[i] - ref)) <= 2e-2
        if abs(ref[0] - ref[1]) > 4e-2:
            assert np.argmax(a[i]) == np.argmax(b[i])
    folded.close()
    plain.close()


@pytest.mark.parametrize("M,N,K", [(64, 768, 3072), (300, 768, 3072), (1, 1024, 4096)])
def test_splitk_resid_ln_epilogue(arlo_lib, M, N, K):
    """Split-K EPI_RESID_LN (the LATENCY runtimes' FFN2): oracle parity of the rows and of the output
    statistics (also with a plain residual), and every split-K tile width and M gives bitwise the same
    rows and statistics (its arithmetic is a function of N and K only: the family's cross-L contract)."""
    eps = 1e-12
    A, W, b = rnd((M, K), 31, 1.1, 0.05), rnd((N, K), 32, 0.02), rnd((N,), 33, 0.02)
    R = rnd((M, N), 34, 1.5, 0.3)
    g, be = rnd((N,), 35, 0.1, 1.0), rnd((N,), 36, 0.1)
    st_r = granule_stats(R).astype(np.float32)
    ref = orc.linear(A, W, b) + ln_from_stats(R.astype(np.float64), st_r.astype(np.float64), g, be, eps)
    runs = []  # (m, rows, statistics); the first is code 2064 at m = M
    for code in (2064, 2032, 2128, 2192):
        if N % (code - 2000):
            continue
        for m in sorted({M, min(M, 64), min(M, 7)}, reverse=True):
            o = torch.empty((m, N), device="cuda", dtype=torch.bfloat16)
            so = torch.full((N // 32, m, 2), float("nan"), device="cuda")
            arlo_lib.op_gemm_fold(bf(A[:m]), bf(W), f32(b), o, arlo_lib.EPI_RESID_LN, v1=f32(g), v2=f32(be),
                                  st_in=f32(gm(st_r[:m])), st_out=so, eps=eps, residual=bf(R[:m]), force_bn=code)
            runs.append((m, o, so))
    torch.cuda.synchronize()
    _, ref_o, ref_s = runs[0]
    y = ref_o.float().cpu().numpy()
    np.testing.assert_allclose(y, ref, rtol=1e-2, atol=2e-2)
    np.testing.assert_allclose(ref_s.cpu().numpy(), gm(granule_stats(y)), rtol=2e-6, atol=1e-4)
    for m, o, so in runs[1:]:
        assert torch.equal(o, ref_o[:m])
        assert torch.equal(so, ref_s[:, :m])
    # st_in = NULL: plain residual
    o2 = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
    arlo_lib.op_gemm_fold(bf(A), bf(W), f32(b), o2, arlo_lib.EPI_RESID_LN, v1=f32(g), v2=f32(be), residual=bf(R),
                          force_bn=2064)
    torch.cuda.synchronize()
    np.testing.assert_allclose(o2.float().cpu().numpy(), orc.linear(A, W, b) + R, rtol=1e-2, atol=2e-2)
