"""-m gpu: each kernel of the split path vs the oracle's definition of the
same step, through the C ABI (include/e3_ops.h).  Sizes span several tiles
and a ragged tail; the full-size shapes of EE-BERT-base are checked on
sampled rows."""
import numpy as np
import pytest
import torch

from tests.gpu_util import DEV, bf16_tensor, bf16_ulp, rand_bf16, requires_cuda, to64

pytestmark = [pytest.mark.gpu, requires_cuda]


@pytest.fixture(scope="module")
def api():
    from paper_conf_sosp_iyergdpgn24_b200 import api as A
    return A


def _gemm_ref(A, W, b, epi, R=None):
    from oracle.encoder import gelu, linear
    y = linear(A.astype(np.float64), W.astype(np.float64), b.astype(np.float64))
    if epi == "bias_gelu":
        y = gelu(y)
    if epi == "bias_resid":
        y = y + R.astype(np.float64)
    return y


def _assert_bf16_close(got, ref, ulps=1.0, atol=1e-4, min_exact=0.97):
    """|got - ref| <= ulps bf16 ulps + atol.  atol covers fp32-vs-fp64
    accumulation on near-cancelling outputs (K <= 3072 terms of size ~1)."""
    from oracle.numerics import bf16_rne
    tol = ulps * bf16_ulp(np.maximum(np.abs(ref), np.abs(got))) + atol
    bad = np.abs(got - ref) > tol
    if bad.any():
        idx = np.argwhere(bad)[:8]
        detail = [(tuple(int(v) for v in i), float(got[tuple(i)]), float(ref[tuple(i)])) for i in idx]
        raise AssertionError(f"{bad.sum()} elements off; max err {np.abs(got - ref).max()}; {detail}")
    exact = np.mean(got == bf16_rne(ref))
    assert exact >= min_exact, f"only {exact:.4f} bit-exact vs RNE of the fp64 value"


@pytest.mark.parametrize("M,N,K", [(128, 64, 128), (300, 384, 128), (1024, 512, 512), (4100, 768, 768)])
@pytest.mark.parametrize("epi", ["bias", "bias_gelu", "bias_resid"])
def test_gemm_matches_definition(api, M, N, K, epi):
    rng = np.random.default_rng(M + N + K)
    A = rand_bf16(rng, (M, K))
    W = rand_bf16(rng, (N, K), K ** -0.5)
    b = rand_bf16(rng, (N,), 0.5)
    R = rand_bf16(rng, (M, N)) if epi == "bias_resid" else None
    out = api.ops.gemm(bf16_tensor(A), bf16_tensor(W), bf16_tensor(b), epi,
                       resid=None if R is None else bf16_tensor(R))
    torch.cuda.synchronize()
    _assert_bf16_close(to64(out), _gemm_ref(A, W, b, epi, R))


@pytest.mark.parametrize("N,K,epi", [(2304, 768, "bias"), (768, 768, "bias_resid"),
                                     (3072, 768, "bias_gelu"), (768, 3072, "bias_resid")])
def test_gemm_full_bert_base_shapes_sampled(api, N, K, epi):
    M = 64 * 128
    g = torch.Generator(device=DEV).manual_seed(N + K)
    A = torch.randn(M, K, device=DEV, generator=g).to(torch.bfloat16)
    W = (torch.randn(N, K, device=DEV, generator=g) * K ** -0.5).to(torch.bfloat16)
    b = (torch.randn(N, device=DEV, generator=g) * 0.1).to(torch.bfloat16)
    R = torch.randn(M, N, device=DEV, generator=g).to(torch.bfloat16) if epi == "bias_resid" else None
    out = api.ops.gemm(A, W, b, epi, resid=R)
    torch.cuda.synchronize()
    rows = np.random.default_rng(0).choice(M, 96, replace=False)
    rows = np.concatenate([rows, [0, 127, 128, M - 1]])
    ref = _gemm_ref(to64(A[rows]), to64(W), to64(b), epi, None if R is None else to64(R[rows]))
    _assert_bf16_close(to64(out[rows]), ref)


@pytest.mark.parametrize("B,S,H,heads", [(2, 32, 128, 2), (3, 128, 768, 12), (2, 197, 128, 2),
                                         (1, 256, 64, 1), (2, 77, 192, 3), (3, 150, 128, 2), (2, 170, 64, 1),
                                         (80, 197, 128, 2), (90, 128, 128, 2)])
def test_attention_matches_oracle(api, B, S, H, heads):
    from oracle.encoder import attention
    rng = np.random.default_rng(S * H)
    qkv = rand_bf16(rng, (B, S, 3 * H))
    out = api.ops.attention(bf16_tensor(qkv.reshape(B * S, 3 * H)), B, S, H, heads)
    torch.cuda.synchronize()
    got = to64(out).reshape(B, S, H)
    ref = attention(qkv.astype(np.float64), heads, mode="bf16")
    # atol: a bf16(p) rounding flip (ex2.approx vs exp) moves one weight by 2^-8
    _assert_bf16_close(got, ref, ulps=2.0, atol=2e-3, min_exact=0.9)


@pytest.mark.parametrize("B,S,H,heads", [(64, 128, 768, 12), (40, 197, 768, 12)])
def test_attention_back_to_back_launches(api, B, S, H, heads):
    """Work items come from a device counter that each launch leaves zeroed
    (two counter pairs alternate): launches queued back to back under PDL --
    eagerly, and 5 per CUDA graph replayed twice -- must each reproduce the
    isolated launch bit for bit (a launch taking items from its still-running
    predecessor's counter recomputes or skips items)."""
    g = torch.Generator(device=DEV).manual_seed(S)
    xs = [torch.randn(B * S, 3 * H, device=DEV, generator=g).to(torch.bfloat16) for _ in range(3)]
    ref = []
    for x in xs:
        ref.append(api.ops.attention(x, B, S, H, heads).clone())
        torch.cuda.synchronize()
    outs = [torch.empty(B * S, H, device=DEV, dtype=torch.bfloat16) for _ in range(7)]
    for i, o in enumerate(outs):
        api.ops.attention(xs[i % 3], B, S, H, heads, out=o)
    torch.cuda.synchronize()
    for i, o in enumerate(outs):
        assert torch.equal(o, ref[i % 3]), i
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        api.ops.attention(xs[0], B, S, H, heads, out=outs[0], stream=st)   # warm-up outside capture
        st.synchronize()
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=st):
            for i in range(5):
                api.ops.attention(xs[i % 3], B, S, H, heads, out=outs[i], stream=st)
    for _ in range(2):
        for o in outs[:5]:
            o.fill_(0)
        graph.replay()
        torch.cuda.synchronize()
        for i in range(5):
            assert torch.equal(outs[i], ref[i % 3]), i


@pytest.mark.parametrize("rows,H,eps", [(37, 128, 1e-12), (1000, 768, 1e-12), (64, 1024, 1e-6), (5, 64, 1e-5)])
def test_layernorm_matches_oracle(api, rows, H, eps):
    from oracle.encoder import layer_norm
    rng = np.random.default_rng(rows)
    x = rand_bf16(rng, (rows, H), 3.0)
    g = rand_bf16(rng, (H,), 0.1) + 1.0
    b = rand_bf16(rng, (H,), 0.1)
    from e3data import bf16_round
    g = bf16_round(g)
    out = api.ops.layernorm(bf16_tensor(x), bf16_tensor(g), bf16_tensor(b), eps)
    torch.cuda.synchronize()
    ref = layer_norm(x.astype(np.float64), g.astype(np.float64), b.astype(np.float64), eps)
    _assert_bf16_close(to64(out), ref, ulps=1.0, atol=1e-5)


@pytest.mark.parametrize("B,alive_pattern", [(64, "random"), (64, "none"), (64, "all"), (33, "ends"),
                                             (1, "all"), (200, "random")])
def test_compaction_is_stable_and_exact(api, B, alive_pattern):
    rng = np.random.default_rng(B)
    S, H = 16, 128
    x = torch.randn(B, S, H, device=DEV).to(torch.bfloat16)
    ids = torch.arange(1000, 1000 + B, device=DEV, dtype=torch.int64)
    if alive_pattern == "random":
        a = rng.random(B) < 0.5
    elif alive_pattern == "none":
        a = np.zeros(B, bool)
    elif alive_pattern == "all":
        a = np.ones(B, bool)
    else:
        a = np.zeros(B, bool)
        a[0] = a[-1] = True
    alive = torch.from_numpy(a.astype(np.uint8)).to(DEV)
    x_out = torch.full_like(x, 7.0)
    id_out = torch.full((B,), -5, dtype=torch.int64, device=DEV)
    n = torch.full((1,), -1, dtype=torch.int32, device=DEV)
    api.ops.compact(x, ids, alive, x_out, id_out, n)
    torch.cuda.synchronize()
    k = int(a.sum())
    assert int(n.item()) == k
    sel = np.nonzero(a)[0]                      # numpy boolean-mask order = stable
    assert torch.equal(x_out[:k].view(torch.int16), x[sel].view(torch.int16))
    assert id_out[:k].cpu().tolist() == (1000 + sel).tolist()
    assert torch.all(x_out[k:] == 7.0) and torch.all(id_out[k:] == -5)   # nothing beyond n_surv


def test_compaction_matches_torch_masked_select_full_size(api):
    B, S, H = 64, 128, 768
    x = torch.randn(B, S, H, device=DEV).to(torch.bfloat16)
    ids = torch.arange(B, device=DEV, dtype=torch.int64)
    alive = (torch.rand(B, device=DEV) < 0.5).to(torch.uint8)
    x_out = torch.empty_like(x)
    id_out = torch.empty_like(ids)
    n = torch.zeros(1, dtype=torch.int32, device=DEV)
    api.ops.compact(x, ids, alive, x_out, id_out, n)
    torch.cuda.synchronize()
    k = int(alive.sum())
    assert int(n) == k
    assert torch.equal(x_out[:k], x[alive.bool()])
    assert torch.equal(id_out[:k], ids[alive.bool()])


@pytest.mark.parametrize("test,C", [("maxprob", 2), ("entropy", 2), ("entropy", 3), ("maxprob", 16)])
def test_ramp_matches_oracle(api, test, C):
    import dataclasses
    import e3data
    from oracle import ramp as oramp
    cfg = dataclasses.replace(e3data.get("tiny"), test=test, classes=C)
    W = e3data.make_weights(cfg, seed=11)
    model = api.DeviceModel(cfg, W, DEV)
    B = 50
    rng = np.random.default_rng(3)
    x = rand_bf16(rng, (B, cfg.seq, cfg.hidden))
    xt = bf16_tensor(x)
    ids = torch.arange(B, device=DEV, dtype=torch.int64) * 3
    n_valid = torch.tensor([45], dtype=torch.int32, device=DEV)
    z = oramp.ramp_logits(cfg, x.astype(np.float64), {k: v.astype(np.float64) for k, v in W["ramps"][0].items()})
    m = oramp.metric(test, z)
    tau = float(np.float32(np.median(m[:45])))
    alive = torch.zeros(B, dtype=torch.uint8, device=DEV)
    ex = api.ExitBuffers(3 * B, C, cfg.n_ramps, DEV)
    api.ops.ramp(cfg, model, 0, xt, ids, tau, alive, ex, final=False, n_valid=n_valid)
    torch.cuda.synchronize()
    passed = oramp.passes(test, m, tau)
    margin = np.abs(m - np.float64(np.float32(tau)))
    al = alive.cpu().numpy().astype(bool)
    el = ex.exit_layer.cpu().numpy()
    for b in range(B):
        if b >= 45:
            assert not al[b] and el[3 * b] == -1           # padding never exits
            continue
        if margin[b] > 1e-3:
            assert al[b] == (not passed[b])
        if not al[b]:
            i = 3 * b
            assert el[i] == cfg.ramp_layers[0]
            assert ex.label.cpu().numpy()[i] == int(np.argmax(z[b]))
            assert abs(ex.conf.cpu().numpy()[i] - m[b]) < 1e-5
            assert np.max(np.abs(ex.logits.cpu().numpy()[i] - z[b])) < 1e-4
    assert int(ex.n_exit.item()) == int((~al[:45]).sum())
    # final ramp exits every alive valid row regardless of tau
    alive2 = torch.zeros(B, dtype=torch.uint8, device=DEV)
    ex2 = api.ExitBuffers(3 * B, C, cfg.n_ramps, DEV)
    api.ops.ramp(cfg, model, 1, xt, ids, 2.0 if test == "maxprob" else -1.0, alive2, ex2, final=True,
                 n_valid=n_valid)
    torch.cuda.synchronize()
    assert int(ex2.n_exit.item()) == 45 and int(alive2.sum()) == 0


@pytest.mark.parametrize("base,test,C", [("tiny", "maxprob", 10), ("tiny", "entropy", 1000),
                                         ("tiny", "maxprob", 1500), ("vt", "maxprob", 1000)])
def test_vit_ramp_matches_oracle(api, base, test, C):
    """ViT ramp (LN + linear over C classes, cluster-merged softmax statistics)
    vs oracle.ramp on the same bf16 rows: decisions exact where the margin
    exceeds 1e-3, label = argmax, logits / metric within fp32 accumulation."""
    import dataclasses
    import e3data
    from oracle import ramp as oramp
    cfg = dataclasses.replace(e3data.get(base), arch="vit", test=test, classes=C, norm_eps=1e-6)
    W = {"layers": [], "ramps": [e3data.make_ramp(cfg, 0, seed=13), e3data.make_ramp(cfg, 1, seed=13)]}
    model = api.DeviceModel(cfg, W, DEV)
    B, nv = 45, 40
    rng = np.random.default_rng(C)
    x = rand_bf16(rng, (B, cfg.seq if base == "tiny" else 4, cfg.hidden))
    xt = bf16_tensor(x)
    ids = torch.arange(B, device=DEV, dtype=torch.int64) * 2 + 1
    n_valid = torch.tensor([nv], dtype=torch.int32, device=DEV)
    R = {k: v.astype(np.float64) for k, v in W["ramps"][0].items()}
    z = oramp.ramp_logits(cfg, x.astype(np.float64), R)
    m = oramp.metric(test, z)
    tau = float(np.float32(np.median(m[:nv])))
    alive = torch.zeros(B, dtype=torch.uint8, device=DEV)
    ex = api.ExitBuffers(2 * B + 2, C, 2, DEV)
    api.ops.ramp(cfg, model, 0, xt, ids, tau, alive, ex, final=False, layer=5, n_valid=n_valid)
    torch.cuda.synchronize()
    passed = oramp.passes(test, m, tau)
    margin = np.abs(m - np.float64(np.float32(tau)))
    al = alive.cpu().numpy().astype(bool)
    el, lab = ex.exit_layer.cpu().numpy(), ex.label.cpu().numpy()
    conf, lg = ex.conf.cpu().numpy(), ex.logits.cpu().numpy()
    n_dec = 0
    for b in range(B):
        i = 2 * b + 1
        if b >= nv:
            assert not al[b] and el[i] == -1
            continue
        if margin[b] > 1e-3:
            assert al[b] == (not passed[b])
            n_dec += 1
        if not al[b]:
            assert el[i] == 5
            top2 = np.sort(z[b])[-2:]
            if top2[1] - top2[0] > 1e-4:
                assert lab[i] == int(np.argmax(z[b]))
            assert abs(conf[i] - m[b]) < 1e-4
            assert np.max(np.abs(lg[i] - z[b])) < 1e-3
        else:
            assert el[i] == -1
    assert n_dec >= nv - 3
    assert int(ex.n_exit.item()) == int((~al[:nv]).sum())
    # final ramp exits every alive valid row
    alive2 = torch.zeros(B, dtype=torch.uint8, device=DEV)
    ex2 = api.ExitBuffers(2 * B + 2, C, 2, DEV)
    api.ops.ramp(cfg, model, 1, xt, ids, 2.0 if test == "maxprob" else -1.0, alive2, ex2, final=True,
                 n_valid=n_valid)
    torch.cuda.synchronize()
    assert int(ex2.n_exit.item()) == nv and int(alive2.sum()) == 0


@pytest.mark.parametrize("T,N,K", [(32, 256, 128), (64, 1280, 4096), (128, 384, 640), (64, 4096, 11008),
                                   (64, 6144, 1024)])
@pytest.mark.parametrize("epi", ["store", "resid", "swiglu"])
def test_dec_gemm_matches_definition(api, T, N, K, epi):
    """Decode GEMM (swap-AB tcgen05): Y = X W^T (+ R) or SiLU(X Wg^T) *
    (X Wu^T), one bf16 rounding.  Store / residual GEMMs of <= 37 tiles take
    the cluster split-K path (4 CTAs per tile, DSMEM reduction); N = 6144
    (48 tiles) and every SwiGLU case take stream-K (tiles shared between CTAs,
    global partials and tickets)."""
    from oracle.llama import silu
    rng = np.random.default_rng(T + N + K)
    X = rand_bf16(rng, (T, K))
    W = rand_bf16(rng, (N, K), K ** -0.5)
    W2 = rand_bf16(rng, (N, K), K ** -0.5) if epi == "swiglu" else None
    R = rand_bf16(rng, (T, N)) if epi == "resid" else None
    out = api.ops.dec_gemm(bf16_tensor(X), bf16_tensor(W), epi, W2=None if W2 is None else bf16_tensor(W2),
                           resid=None if R is None else bf16_tensor(R))
    torch.cuda.synchronize()
    y = X.astype(np.float64) @ W.astype(np.float64).T
    if epi == "resid":
        y = y + R
    if epi == "swiglu":
        y = silu(y) * (X.astype(np.float64) @ W2.astype(np.float64).T)
    # fp32 accumulation over up to 11008 terms + SiLU in fp32: 1 ulp + small atol
    _assert_bf16_close(to64(out), y, ulps=1.0, atol=2e-3 if K > 4096 else 5e-4, min_exact=0.9)


@pytest.mark.parametrize("M,N,K", [(300, 128, 128), (1000, 768, 768), (520, 1024, 1024), (256, 384, 3072)])
@pytest.mark.parametrize("with_pre", [False, True])
def test_gemm_ln_matches_definition(api, M, N, K, with_pre):
    """Fused O projection + residual + LayerNorm (cluster of 2 CTAs per row
    block, row statistics exchanged through DSMEM) vs the oracle's
    definition: y = bf16(A W^T + b + R), out = bf16(LN(y))."""
    from oracle.encoder import layer_norm, linear
    from oracle.numerics import bf16_rne
    rng = np.random.default_rng(M + N + K)
    A = rand_bf16(rng, (M, K))
    W = rand_bf16(rng, (N, K), K ** -0.5)
    b = rand_bf16(rng, (N,), 0.1)
    R = rand_bf16(rng, (M, N))
    from e3data import bf16_round
    g = bf16_round(rand_bf16(rng, (N,), 0.1) + 1.0)     # gamma must be bf16-representable
    beta = rand_bf16(rng, (N,), 0.1)
    pre = torch.zeros((M, N), dtype=torch.bfloat16, device=DEV) if with_pre else None
    out = api.ops.gemm_ln(bf16_tensor(A), bf16_tensor(W), bf16_tensor(b), bf16_tensor(R), bf16_tensor(g),
                          bf16_tensor(beta), 1e-12, pre=pre)
    torch.cuda.synchronize()
    y = bf16_rne(linear(A.astype(np.float64), W.astype(np.float64), b.astype(np.float64)) + R)
    if with_pre:
        _assert_bf16_close(to64(pre), linear(A.astype(np.float64), W.astype(np.float64), b.astype(np.float64)) + R,
                           atol=1e-4)
    # on the GPU's own rounded y: one rounding of the LN output (1 ulp); on
    # the oracle's y, a 1-ulp difference of a y element (fp32 vs fp64
    # accumulation) moves that output element by about one more ulp
    yg = to64(pre) if with_pre else y
    ref = layer_norm(yg, g.astype(np.float64), beta.astype(np.float64), 1e-12)
    # (single-pass statistics E[y^2] - mean^2 in fp32: ~1e-7 relative on var)
    # (a y element one ulp (<= 2^-7 |y|) off moves its output by <= 2^-7 |y| rstd g)
    _assert_bf16_close(to64(out), ref, ulps=1.0 if with_pre else 2.0, atol=1e-3 if with_pre else 1e-2,
                       min_exact=0.9 if with_pre else 0.5)
