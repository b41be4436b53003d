"""Pins for oracle.ramp: closed forms of the exit metrics and library routines."""
import numpy as np
import scipy.special as sp

from oracle import ramp


def test_maxprob_closed_form_point_nine():
    z = np.array([0.0, np.log(9.0)])
    assert abs(ramp.max_prob(z) - 0.9) < 1e-15


def test_uniform_logits():
    for C in (2, 10, 1000):
        z = np.full(C, 1.7)
        assert abs(ramp.max_prob(z) - 1.0 / C) < 1e-15
        assert abs(ramp.entropy(z) - np.log(C)) < 1e-12


def test_binary_entropy_at_default_threshold():
    # P:1616-1617 default entropy 0.4 <-> binary max-prob 0.8627
    p = 0.8627
    z = np.array([np.log(p), np.log(1 - p)])
    assert abs(ramp.entropy(z) - 0.4000) < 1e-4


def test_metrics_match_scipy():
    rng = np.random.default_rng(0)
    Z = rng.standard_normal((50, 7)) * 5
    q = sp.softmax(Z, axis=-1)
    assert np.allclose(ramp.max_prob(Z), q.max(-1), rtol=1e-14)
    assert np.allclose(ramp.entropy(Z), sp.entr(q).sum(-1), rtol=1e-12, atol=1e-14)
    # large logits stay finite
    assert np.isfinite(ramp.entropy(np.array([1e4, -1e4]))).all()


def test_threshold_direction_and_strictness():
    assert ramp.passes("maxprob", 0.95, 0.9) and not ramp.passes("maxprob", 0.85, 0.9)
    assert ramp.passes("entropy", 0.3, 0.4) and not ramp.passes("entropy", 0.5, 0.4)
    t = float(np.float32(0.9))
    assert not ramp.passes("maxprob", t, 0.9)          # equal -> no exit (R12)
    assert not ramp.passes("entropy", float(np.float32(0.4)), 0.4)


def test_bert_ramp_is_pooler_then_fc():
    from e3data.configs import ModelConfig
    cfg = ModelConfig(name="t", arch="bert", layers=1, hidden=4, heads=1, ffn=4, seq=3,
                      classes=2, norm_eps=1e-12, ramp_layers=(0,), batch=1, test="maxprob")
    h = np.zeros((3, 4)); h[0] = [1.0, -1.0, 0.5, 0.0]; h[1:] = 99.0   # only token 0 used
    R = {"w_p": np.eye(4), "b_p": np.zeros(4), "w_c": np.array([[1, 0, 0, 0], [0, 1, 0, 0.0]]),
         "b_c": np.array([0.0, 0.25])}
    z = ramp.ramp_logits(cfg, h, R)
    assert np.allclose(z, [np.tanh(1.0), np.tanh(-1.0) + 0.25])


def test_vit_ramp_matches_torch_layernorm_linear():
    """ViT ramp = LayerNorm(CLS) then Linear (R1), pinned to torch.nn in fp64."""
    import torch
    from e3data.configs import ModelConfig
    H, C = 16, 1000
    cfg = ModelConfig(name="t", arch="vit", layers=1, hidden=H, heads=1, ffn=H, seq=5,
                      classes=C, norm_eps=1e-6, ramp_layers=(0,), batch=1, test="maxprob")
    rng = np.random.default_rng(4)
    h = rng.standard_normal((3, 5, H)) * 2 + 0.3
    R = {"ln_g": 1 + 0.1 * rng.standard_normal(H), "ln_b": 0.1 * rng.standard_normal(H),
         "w_c": rng.standard_normal((C, H)), "b_c": rng.standard_normal(C)}
    ln = torch.nn.LayerNorm(H, eps=1e-6).double()
    lin = torch.nn.Linear(H, C).double()
    with torch.no_grad():
        ln.weight.copy_(torch.from_numpy(R["ln_g"])); ln.bias.copy_(torch.from_numpy(R["ln_b"]))
        lin.weight.copy_(torch.from_numpy(R["w_c"])); lin.bias.copy_(torch.from_numpy(R["b_c"]))
        ref = lin(ln(torch.from_numpy(h[:, 0, :]))).numpy()
    assert np.allclose(ramp.ramp_logits(cfg, h, R), ref, rtol=1e-12, atol=1e-12)
