"""Seeded synthetic data for E3 workloads (no method arithmetic; see gen.py)."""
from .configs import ModelConfig, CONFIGS, get, survival_profile, tau_for  # noqa: F401
from .gen import (bf16_round, bf16_bits, make_weights, make_layer, make_ramp,  # noqa: F401
                  make_inputs, make_kv, make_embed)
