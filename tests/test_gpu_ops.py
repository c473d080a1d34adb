"""Per-kernel parity of the CUDA path (through the C ABI, arlo_op_*) against the
oracle's per-step functions, element by element (needs a B200)."""
import numpy as np
import pytest
import torch

from oracle import encoder as orc
from paper_conf_icpp_tanlyl024_b200 import workload as wl

pytestmark = pytest.mark.gpu


def bf16_dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.float32)).to("cuda", torch.bfloat16)


def f32_dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.float32)).to("cuda")


def host64(t):
    return t.float().cpu().numpy().astype(np.float64)


def rnd(shape, seed, std=1.0):
    return wl.round_to_bf16(np.random.default_rng(seed).standard_normal(shape).astype(np.float32) * std)


# --------------------------------------------------------------------------- GEMM
GEMM_SHAPES = [
    (64, 2304, 768), (200, 768, 768), (384, 3072, 768), (333, 768, 3072),  # ragged M tails
    (1024, 1024, 1024), (128, 128, 128), (32, 384, 128), (4096, 2304, 768),
]


@pytest.mark.parametrize("M,N,K", GEMM_SHAPES)
@pytest.mark.parametrize("epi", [0, 1, 2])
@pytest.mark.parametrize("force", [0, 96, 128, -128, -256, 192, -192, 1016, 1032, 1064])
def test_gemm_tcgen05_bf16(arlo_lib, M, N, K, epi, force):
    """force: BN single CTA, -BN CTA pair, 1000 + BN skinny (small-M) kernel, 0 = tile chooser."""
    if N % (force - 1000 if force > 1000 else abs(force or 64)):
        pytest.skip("tile width does not divide N")
    A = rnd((M, K), 1)
    W = rnd((N, K), 2, 0.02)
    b = rnd((N,), 3, 0.02)
    R = rnd((M, N), 4)
    ref = orc.linear(A, W, b)
    if epi == 1:
        ref = orc.gelu(ref)
    if epi == 2:
        ref = ref + R
    out = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
    arlo_lib.op_gemm(arlo_lib.BF16, bf16_dev(A), bf16_dev(W), f32_dev(b), out, epi=epi,
                     residual=bf16_dev(R) if epi == 2 else None, force_bn=force)
    torch.cuda.synchronize()
    got = host64(out)
    # bf16 output rounding (2^-9 relative) on fp32-accumulated exact products
    np.testing.assert_allclose(got, ref, rtol=8e-3, atol=8e-3)


@pytest.mark.parametrize("epi", [0, 1, 2])
@pytest.mark.parametrize("bn", [64, 96, 128, 192, 256, -128, -192, -256, 1016, 1032, 1064])
def test_gemm_tile_widths_agree_bitwise(arlo_lib, bn, epi):
    """Row results do not depend on the tile width, the epilogue warp count (12 for GELU at
    M <= 8192, 8 otherwise) or M (cross-L invariance contract), for every epilogue."""
    M, N, K = 300, 768, 768
    A, W, b = bf16_dev(rnd((M, K), 5)), bf16_dev(rnd((N, K), 6, 0.02)), f32_dev(rnd((N,), 7, 0.02))
    R = bf16_dev(rnd((M, N), 8))
    outs = []
    for force in (bn, -256):
        o = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
        arlo_lib.op_gemm(arlo_lib.BF16, A, W, b, o, epi=epi, residual=R if epi == 2 else None, force_bn=force)
        outs.append(o)
    torch.cuda.synchronize()
    assert torch.equal(outs[0], outs[1])
    # and a row does not depend on M (prefix of rows)
    o2 = torch.empty((77, N), device="cuda", dtype=torch.bfloat16)
    arlo_lib.op_gemm(arlo_lib.BF16, A[:77].contiguous(), W, b, o2, epi=epi,
                     residual=R[:77].contiguous() if epi == 2 else None, force_bn=64)
    torch.cuda.synchronize()
    assert torch.equal(o2, outs[0][:77])


@pytest.mark.parametrize("M,N,K", [(100, 384, 128), (64, 128, 512), (257, 192, 64)])
@pytest.mark.parametrize("epi", [0, 1, 2])
def test_gemm_fp32_check_mode(arlo_lib, M, N, K, epi):
    rng = np.random.default_rng(M + N + K)
    A = rng.standard_normal((M, K)).astype(np.float32)
    W = (rng.standard_normal((N, K)) * 0.05).astype(np.float32)
    b = (rng.standard_normal(N) * 0.05).astype(np.float32)
    R = rng.standard_normal((M, N)).astype(np.float32)
    ref = orc.linear(A, W, b)
    if epi == 1:
        ref = orc.gelu(ref)
    if epi == 2:
        ref = ref + R
    out = torch.empty((M, N), device="cuda", dtype=torch.float32)
    arlo_lib.op_gemm(arlo_lib.FP32, f32_dev(A), f32_dev(W), f32_dev(b), out, epi=epi,
                     residual=f32_dev(R) if epi == 2 else None)
    torch.cuda.synchronize()
    np.testing.assert_allclose(host64(out), ref, rtol=0, atol=2e-5)


# ---------------------------------------------------------------------- LayerNorm
@pytest.mark.parametrize("H", [128, 768, 1024])
@pytest.mark.parametrize("dtype", [0, 1])
def test_layernorm(arlo_lib, H, dtype):
    M = 257
    x = wl.round_to_bf16(rnd((M, H), H) * 3 + 1)
    g = wl.round_to_bf16(rnd((H,), 1, 0.1) + 1)
    b = rnd((H,), 2, 0.02)
    ref = orc.layer_norm(x, g, b, 1e-12)
    dev = bf16_dev if dtype == 0 else f32_dev
    out = torch.empty((M, H), device="cuda", dtype=torch.bfloat16 if dtype == 0 else torch.float32)
    arlo_lib.op_layernorm(dtype, dev(x), f32_dev(g), f32_dev(b), 1e-12, out)
    torch.cuda.synchronize()
    tol = 2e-2 if dtype == 0 else 1e-5
    np.testing.assert_allclose(host64(out), ref, rtol=0, atol=tol)


# ---------------------------------------------------------------------- embedding
@pytest.mark.parametrize("dtype", [0, 1])
def test_embedding_ln(arlo_lib, dtype):
    cfg = wl.BERT_BASE
    w = wl.make_weights(wl.ModelConfig("emb", 1, 768, 12, 3072, 2000), seed=1)
    L = 96
    lengths = np.array([96, 1, 50, 0], np.int32)
    ids = wl.sample_token_ids(wl.ModelConfig("emb", 1, 768, 12, 3072, 2000), lengths, L, seed=3)
    ids_garbage = ids.copy()
    ids_garbage[2, 50:] = 123456  # beyond len: ignored, no error
    dev = bf16_dev if dtype == 0 else f32_dev
    out = torch.empty((4 * L, 768), device="cuda", dtype=torch.bfloat16 if dtype == 0 else torch.float32)
    err = torch.zeros(1, dtype=torch.int32, device="cuda")
    arlo_lib.op_embed(dtype, torch.from_numpy(ids_garbage).cuda(), torch.from_numpy(lengths).cuda(),
                      dev(w["word_emb"]), dev(w["pos_emb"]), dev(w["type_emb"]), f32_dev(w["emb_ln_g"]),
                      f32_dev(w["emb_ln_b"]), 1e-12, out, err)
    torch.cuda.synchronize()
    assert err.item() == 0
    got = host64(out).reshape(4, L, 768)
    tol = 2e-2 if dtype == 0 else 1e-5
    for i in range(4):
        tok = ids[i].copy()
        tok[lengths[i]:] = 0
        ref = orc.embed(cfg, w, tok)
        np.testing.assert_allclose(got[i], ref, rtol=0, atol=tol)
    # out-of-range id at a real position sets the flag
    bad = ids.copy()
    bad[0, 3] = 5000
    err.zero_()
    arlo_lib.op_embed(dtype, torch.from_numpy(bad).cuda(), torch.from_numpy(lengths).cuda(),
                      dev(w["word_emb"]), dev(w["pos_emb"]), dev(w["type_emb"]), f32_dev(w["emb_ln_g"]),
                      f32_dev(w["emb_ln_b"]), 1e-12, out, err)
    torch.cuda.synchronize()
    assert err.item() == 1


# ---------------------------------------------------------------------- attention
@pytest.mark.parametrize("L,heads,lengths", [
    (128, 12, [128, 1, 65, 64, 0, 100]),
    (512, 2, [512, 300, 7]),
    (32, 2, [32, 5, 1, 17]),
    (64, 16, [63, 64]),
    (256, 4, [256, 200, 129, 1, 128]),
    (384, 2, [384, 257, 100]),
    (192, 3, [192, 191, 129, 128, 1]),
    (320, 2, [320, 257, 200, 0]),
    (448, 2, [448, 385, 300, 64]),
    (64, 3, [64, 0, 17]),          # packed tiles (L = 64): odd B, empty slot in a pair
    (64, 2, [1, 64, 40, 2, 0]),
])
@pytest.mark.parametrize("dtype", [0, 1])
def test_attention_masked(arlo_lib, L, heads, lengths, dtype):
    B = len(lengths)
    H = 64 * heads
    qkv = rnd((B * L, 3 * H), L + heads, 1.0)
    lens = np.array(lengths, np.int32)
    dev = bf16_dev if dtype == 0 else f32_dev
    out = torch.full((B * L, H), float("nan"), device="cuda",
                     dtype=torch.bfloat16 if dtype == 0 else torch.float32)
    arlo_lib.op_attention(dtype, B, L, heads, dev(qkv), torch.from_numpy(lens).cuda(), out)
    torch.cuda.synchronize()
    got = host64(out).reshape(B, L, H)
    assert np.all(np.isfinite(got)), "pad rows must be finite"
    tol = 2e-2 if dtype == 0 else 2e-5
    for i, n in enumerate(lengths):
        x = qkv[i * L:(i + 1) * L].astype(np.float64)
        q, k, v = x[:, :H], x[:, H:2 * H], x[:, 2 * H:]
        if n > 0:
            ref = orc.attention(q[:n], k[:n], v[:n], heads)
            np.testing.assert_allclose(got[i, :n], ref, rtol=0, atol=tol)
            # rows of a partially padded query tile attend the real keys
            end = min(L, ((n + 127) // 128) * 128)
            if end > n:
                refm = orc.attention_masked(q[:end], k[:end], v[:end], heads, n)
                np.testing.assert_allclose(got[i, n:end], refm[n:end], rtol=0, atol=tol)
        start = ((n + 127) // 128) * 128
        assert np.all(got[i, start:] == 0)


# --------------------------------------------------------------------------- head
@pytest.mark.parametrize("dtype", [0, 1])
def test_head(arlo_lib, dtype):
    cfg = wl.BERT_BASE
    w = wl.make_weights(wl.ModelConfig("hd", 1, 768, 12, 3072, 100), seed=4)
    B, L = 5, 64
    x = rnd((B * L, 768), 9)
    dev = bf16_dev if dtype == 0 else f32_dev
    logits = torch.empty((B, 2), device="cuda", dtype=torch.float32)
    arlo_lib.op_head(dtype, B, L, dev(x), dev(w["w_p"]), f32_dev(w["b_p"]), dev(w["w_c"]), f32_dev(w["b_c"]), logits)
    torch.cuda.synchronize()
    ref = np.stack([orc.head(w, x[i * L].astype(np.float64)) for i in range(B)])
    np.testing.assert_allclose(logits.cpu().numpy(), ref, rtol=0, atol=1e-5)


@pytest.mark.parametrize("dtype", [0, 1])
def test_attention_lazy_rescale_path(arlo_lib, dtype):
    """Later key tiles with much larger scores force the running-max rescale of O
    (bf16 kernel: tile max exceeding the stale max by > 2^8 in p)."""
    B, L, heads = 2, 512, 4
    H = 64 * heads
    qkv = rnd((B * L, 3 * H), 77, 1.0)
    x = qkv.reshape(B, L, 3 * H)
    x[:, 300:330, H:2 * H] *= 8.0   # keys in tile 2 dominate
    x[:, 400:410, H:2 * H] *= 12.0  # and tile 3 even more
    qkv = wl.round_to_bf16(x.reshape(B * L, 3 * H))
    lens = np.array([512, 420], np.int32)
    dev = bf16_dev if dtype == 0 else f32_dev
    out = torch.empty((B * L, H), device="cuda", dtype=torch.bfloat16 if dtype == 0 else torch.float32)
    arlo_lib.op_attention(dtype, B, L, heads, dev(qkv), torch.from_numpy(lens).cuda(), out)
    torch.cuda.synchronize()
    got = host64(out).reshape(B, L, H)
    tol = 2e-2 if dtype == 0 else 2e-5
    for i, n in enumerate(lens):
        xx = qkv[i * L:(i + 1) * L].astype(np.float64)
        ref = orc.attention(xx[:n, :H], xx[:n, H:2 * H], xx[:n, 2 * H:], heads)
        np.testing.assert_allclose(got[i, :n], ref, rtol=0, atol=tol)


@pytest.mark.parametrize("M,N,K", [(4096, 768, 768), (333, 768, 3072), (64, 1024, 1024), (700, 1024, 4096),
                                   (100, 128, 512), (2048, 768, 768)])
def test_gemm_fused_layernorm(arlo_lib, M, N, K):
    """Residual + LayerNorm fused into the GEMM epilogue (cluster row statistics)."""
    A = rnd((M, K), 1)
    W = rnd((N, K), 2, 0.02)
    b = rnd((N,), 3, 0.02)
    R = rnd((M, N), 4)
    g = wl.round_to_bf16(rnd((N,), 5, 0.1) + 1)
    be = rnd((N,), 6, 0.02)
    ref = orc.layer_norm(orc.linear(A, W, b) + R, g, be, 1e-12)
    out = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
    arlo_lib.op_gemm_ln(bf16_dev(A), bf16_dev(W), f32_dev(b), bf16_dev(R), f32_dev(g), f32_dev(be), 1e-12, out)
    torch.cuda.synchronize()
    np.testing.assert_allclose(host64(out), ref, rtol=0, atol=3e-2)
    # in place (out aliases the residual), as the runtime uses it
    Rd = bf16_dev(R)
    arlo_lib.op_gemm_ln(bf16_dev(A), bf16_dev(W), f32_dev(b), Rd, f32_dev(g), f32_dev(be), 1e-12, Rd)
    torch.cuda.synchronize()
    assert torch.equal(Rd, out)


@pytest.mark.parametrize("B", [5, 32])
def test_attention_packed_L64_bitwise(arlo_lib, B):
    """L = 64 runs two sequences per 128-row tile; every row equals bit for bit the row an
    unpacked tile computes (the same sequences at L = 128, one sequence per tile)."""
    heads, H = 12, 768
    rng = np.random.default_rng(B)
    lens = rng.integers(1, 65, B).astype(np.int32)
    lens[0] = 64
    q64 = rnd((B * 64, 3 * H), 300 + B)
    q128 = rnd((B * 128, 3 * H), 400 + B)  # garbage in rows 64..127 of each sequence
    q128.reshape(B, 128, 3 * H)[:, :64] = q64.reshape(B, 64, 3 * H)
    o64 = torch.empty((B * 64, H), device="cuda", dtype=torch.bfloat16)
    o128 = torch.empty((B * 128, H), device="cuda", dtype=torch.bfloat16)
    ld = torch.from_numpy(lens).cuda()
    arlo_lib.op_attention(0, B, 64, heads, bf16_dev(q64), ld, o64)
    arlo_lib.op_attention(0, B, 128, heads, bf16_dev(q128), ld, o128)
    torch.cuda.synchronize()
    assert torch.equal(o64.view(B, 64, H), o128.view(B, 128, H)[:, :64])


@pytest.mark.parametrize("M,N,K,epi,force", [(4096, 3072, 768, 1, 0), (4096, 2304, 768, 0, -192), (300, 3072, 768, 1, 128),
                                             (2048, 4096, 1024, 1, -256), (777, 384, 128, 0, 64), (16384, 3072, 1024, 0, 0)])
def test_ln_prologue_gemm_bitwise(arlo_lib, M, N, K, epi, force):
    """LayerNorm as the prologue of the consuming GEMM (one launch, grid barrier) gives bit for bit
    the LayerNorm kernel's rows and the GEMM of those rows; repeated launches reuse the barrier."""
    y = bf16_dev(wl.round_to_bf16(rnd((M, K), 50) * 2 + 0.5))
    g = f32_dev(wl.round_to_bf16(rnd((K,), 51, 0.1) + 1))
    be = f32_dev(rnd((K,), 52, 0.02))
    W, b = bf16_dev(rnd((N, K), 53, 0.02)), f32_dev(rnd((N,), 54, 0.02))
    x_ref = torch.empty((M, K), device="cuda", dtype=torch.bfloat16)
    arlo_lib.op_layernorm(0, y, g, be, 1e-12, x_ref)
    o_ref = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
    arlo_lib.op_gemm(arlo_lib.BF16, x_ref, W, b, o_ref, epi=epi, force_bn=force)
    bar = torch.zeros(2, dtype=torch.int32, device="cuda")
    for _ in range(3):
        x = torch.full((M, K), float("nan"), device="cuda", dtype=torch.bfloat16)
        o = torch.full((M, N), float("nan"), device="cuda", dtype=torch.bfloat16)
        arlo_lib.op_ln_gemm(y, g, be, 1e-12, x, W, b, o, epi=epi, force_bn=force, barrier=bar)
        torch.cuda.synchronize()
        assert torch.equal(x, x_ref)
        assert torch.equal(o, o_ref)
    assert bar[0].item() == 0 and bar[1].item() == 3  # arrivals reset, one generation per launch
    ref = orc.layer_norm(host64(y), g.cpu().numpy().astype(np.float64), be.cpu().numpy().astype(np.float64), 1e-12)
    np.testing.assert_allclose(host64(x), ref, rtol=0, atol=2e-2)
