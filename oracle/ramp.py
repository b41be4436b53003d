"""Exit ramps and exit criteria — TEST INFRASTRUCTURE ONLY.

Ramp architecture (R1 = SURVEY C1): DeeBERT adds "a bertpooler, a
dropout layer, and a fully connected layer" after each encoder block
(P:399-403).  Pooler = tanh(W_p h[token 0] + b_p); dropout is the identity at
inference; FC = W_c p + b_c.  ViT ramp: LN + linear on the CLS token.

Criteria: confidence-based ("certainty level is higher than a
pre-defined threshold": exit iff max softmax > tau) and entropy-based
("entropy ... smaller than pre-defined threshold": exit iff H < tau, natural
log; R3/R4).  Comparisons are strict (R12); tau is an fp32 value compared in
float64.

Pins (tests/test_oracle_ramp.py): closed forms — logits [0, ln 9] give
max-prob exactly 0.9; uniform logits give max-prob 1/C and entropy ln C;
binary entropy at p = 0.8627 is 0.4000 (P:1616-1617 default); entropy equals
-sum q ln q computed from scipy.special.entr; max-prob equals
scipy.special.softmax's maximum.
"""
from __future__ import annotations

import numpy as np

from .encoder import layer_norm


def ramp_logits(cfg, h, R):
    """Logits z of the ramp R applied to encoder output h ([..., S, H])."""
    c = h[..., 0, :]                              # CLS / token 0 (R2)
    if cfg.arch == "bert":
        p = np.tanh(np.matmul(c, R["w_p"].T) + R["b_p"])
        return np.matmul(p, R["w_c"].T) + R["b_c"]
    if cfg.arch == "vit":
        n = layer_norm(c, R["ln_g"], R["ln_b"], cfg.norm_eps)
        return np.matmul(n, R["w_c"].T) + R["b_c"]
    raise NotImplementedError(cfg.arch)


def softmax(z):
    e = np.exp(z - z.max(axis=-1, keepdims=True))
    return e / e.sum(axis=-1, keepdims=True)


def max_prob(z):
    """Softmax confidence: max_c softmax(z)_c."""
    return softmax(z).max(axis=-1)


def entropy(z):
    """Entropy of softmax(z) in nats: H = lse(z) - sum_c q_c z_c."""
    m = z.max(axis=-1, keepdims=True)
    lse = m[..., 0] + np.log(np.exp(z - m).sum(axis=-1))
    q = softmax(z)
    return lse - (q * z).sum(axis=-1)


def metric(test, z):
    if test == "maxprob":
        return max_prob(z)
    if test == "entropy":
        return entropy(z)
    raise ValueError(test)


def passes(test, m, tau):
    """Strict exit test against an fp32 threshold (R12)."""
    t = np.float64(np.float32(tau))
    if test == "maxprob":
        return m > t
    if test == "entropy":
        return m < t
    raise ValueError(test)
