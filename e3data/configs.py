"""Model / workload configurations shared by the oracle, the tests and bench.py.

Pure data: dimensions, ramp placement, exit test, thresholds and the synthetic
exit profile of every BASELINE.json config (SURVEY.md §8 "Configs", §8(d)).
No arithmetic of the method lives here.

Layer and ramp indices are 0-based: "a ramp after layer 2" (1-based, as the
paper and BASELINE.json count) is ``ramp_layers = (1, ...)``.
"""
from __future__ import annotations

from dataclasses import dataclass, field, replace
from typing import Optional, Tuple


@dataclass(frozen=True)
class ModelConfig:
    name: str
    arch: str                  # "bert" (post-LN) | "vit" (pre-LN) | "llama" (decode)
    layers: int
    hidden: int
    heads: int
    ffn: int
    seq: int                   # tokens per input (S); 1 for llama decode
    classes: int               # ramp classes C (vocab V for llama)
    norm_eps: float
    ramp_layers: Tuple[int, ...]   # 0-based layer index each ramp follows, ascending
    batch: int                 # constant batch B
    test: str                  # "maxprob" | "entropy"
    tau: Optional[Tuple[float, ...]] = None        # per-ramp thresholds (None: calibrate)
    exit_profile: Optional[Tuple[float, ...]] = None  # target exit fraction per ramp
    cls_gain: float = 4.0      # classifier init gain g
    kv_heads: int = 0          # llama only
    ctx: int = 0               # llama only: pre-filled KV length
    rope_theta: float = 10000.0

    @property
    def head_dim(self) -> int:
        return self.hidden // self.heads

    @property
    def n_ramps(self) -> int:
        return len(self.ramp_layers)

    def with_tau(self, tau) -> "ModelConfig":
        return replace(self, tau=tuple(float(t) for t in tau))


def survival_profile(ramp_layers, half_life_layers):
    """Per-ramp exit fractions e_r for survival S(l) = 2^(-l/h) after 1-based
    layer l, the last ramp taking every remaining input.

    h = 6 reproduces "roughly half of the samples exit ... by ramp 6"
    (Fig. 3) for a 12-layer DeeBERT."""
    prev = 1.0
    out = []
    for i, l in enumerate(ramp_layers):
        s = 0.0 if i == len(ramp_layers) - 1 else 2.0 ** (-(l + 1) / half_life_layers)
        out.append(prev - s)
        prev = s
    return tuple(out)


TINY = ModelConfig(
    name="tiny", arch="bert", layers=4, hidden=128, heads=2, ffn=512, seq=32,
    classes=2, norm_eps=1e-12, ramp_layers=(1, 3), batch=32, test="maxprob",
    tau=(0.9, 0.9),
)

# ViT-shaped tiny case: pre-LN layers, LN + linear ramp over 10 classes, a
# token count (37) that leaves a ragged tail in every 128-row tile
TINY_VIT = ModelConfig(
    name="tiny-vit", arch="vit", layers=4, hidden=128, heads=2, ffn=512, seq=37,
    classes=10, norm_eps=1e-6, ramp_layers=(1, 3), batch=32, test="maxprob",
    tau=(0.77, 0.77),
)

BERT_BASE = ModelConfig(
    name="ee-bert-base", arch="bert", layers=12, hidden=768, heads=12, ffn=3072,
    seq=128, classes=2, norm_eps=1e-12, ramp_layers=tuple(range(12)), batch=64,
    test="entropy", exit_profile=survival_profile(tuple(range(12)), 6.0),
)

BERT_LARGE = ModelConfig(
    name="ee-bert-large", arch="bert", layers=24, hidden=1024, heads=16, ffn=4096,
    seq=128, classes=2, norm_eps=1e-12, ramp_layers=(3, 7, 11, 15, 19, 23),
    batch=128, test="entropy",
    exit_profile=survival_profile((3, 7, 11, 15, 19, 23), 12.0),
)

VIT_BASE = ModelConfig(
    name="ee-vit-b16", arch="vit", layers=12, hidden=768, heads=12, ffn=3072,
    seq=197, classes=1000, norm_eps=1e-6, ramp_layers=(1, 3, 5, 7, 9, 11),
    batch=256, test="maxprob",
    exit_profile=survival_profile((1, 3, 5, 7, 9, 11), 6.0),
)

# LLaMA-shaped tiny decode case: head_dim 128 as Llama-2, 2 heads, V = 1000,
# 40 cached positions
TINY_LLAMA = ModelConfig(
    name="tiny-llama", arch="llama", layers=4, hidden=256, heads=2, ffn=512, seq=1,
    classes=1000, norm_eps=1e-5, ramp_layers=(1, 3), batch=32, test="maxprob",
    tau=(0.74, 0.74), cls_gain=8.0, kv_heads=2, ctx=40,
)

LLAMA_7B = ModelConfig(
    name="ee-llama-7b-decode", arch="llama", layers=32, hidden=4096, heads=32,
    ffn=11008, seq=1, classes=32000, norm_eps=1e-5, ramp_layers=(7, 15, 23, 31),
    batch=64, test="maxprob", exit_profile=(0.05, 0.10, 0.35, 0.50),
    kv_heads=32, ctx=512, cls_gain=8.0,
)

# Llama-3.1-8B shape (SURVEY §8(f) NEXT-2's variant): grouped-query attention
# (32 query heads over 8 KV heads), F 14336, V = 128256, RoPE theta 5e5; the
# same four ramps and exit profile as the Llama-2-7B case
LLAMA3_8B = ModelConfig(
    name="ee-llama3-8b-decode", arch="llama", layers=32, hidden=4096, heads=32,
    ffn=14336, seq=1, classes=128256, norm_eps=1e-5, ramp_layers=(7, 15, 23, 31),
    batch=64, test="maxprob", exit_profile=(0.05, 0.10, 0.35, 0.50),
    kv_heads=8, ctx=512, cls_gain=8.0, rope_theta=500000.0,
)

# Dependent exits (NEXT-4; PABEE): the counter-based criterion
# with patience t (DESIGN R26).  TINY_PABEE: tiny dims, a ramp after every
# layer; BERT_BASE_PABEE: EE-BERT-base's shape and weights, patience 2.
TINY_PABEE = ModelConfig(
    name="tiny-pabee", arch="bert", layers=4, hidden=128, heads=2, ffn=512, seq=32,
    classes=2, norm_eps=1e-12, ramp_layers=(0, 1, 2, 3), batch=32, test="patience",
    tau=(1.0, 1.0, 1.0, 1.0),
)

BERT_BASE_PABEE = ModelConfig(
    name="ee-bert-base-pabee", arch="bert", layers=12, hidden=768, heads=12, ffn=3072,
    seq=128, classes=2, norm_eps=1e-12, ramp_layers=tuple(range(12)), batch=64,
    test="patience", tau=(2.0,) * 12,
)

CONFIGS = {c.name: c for c in (TINY, TINY_VIT, BERT_BASE, BERT_LARGE, VIT_BASE, TINY_LLAMA, LLAMA_7B, LLAMA3_8B,
                               TINY_PABEE, BERT_BASE_PABEE)}
ALIASES = {"t": "tiny", "tv": "tiny-vit", "tl": "tiny-llama", "bb": "ee-bert-base", "bl": "ee-bert-large",
           "vt": "ee-vit-b16", "lm": "ee-llama-7b-decode", "l8": "ee-llama3-8b-decode", "tp": "tiny-pabee",
           "bbp": "ee-bert-base-pabee"}


def get(name: str) -> ModelConfig:
    return CONFIGS[ALIASES.get(name, name)]


def tau_path(cfg: ModelConfig) -> str:
    import os
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    return os.path.join(root, "tests", "golden", f"tau_{cfg.name}.json")


def tau_for(cfg: ModelConfig):
    """Per-ramp thresholds: cfg.tau, else the calibrated values committed in
    tests/golden/tau_<name>.json (written by ``python -m oracle.calibrate``)."""
    if cfg.tau is not None:
        return cfg.tau
    import json
    with open(tau_path(cfg)) as f:
        return tuple(json.load(f)["tau"])
