"""CPU oracle for the E3 early-exit split path — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct NumPy float64 implementation of what the
hot path computes.  Only ``tests/``,
``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import it.  The CUDA product path never imports,
links or executes anything under ``oracle/``; the two share no code.  Their
only common dependency is ``e3data`` (seeded input generators, no arithmetic
of the method).

Modules
  numerics      bf16 round-to-nearest-even emulation (storage-point rounding)
  encoder       BERT post-LN / ViT pre-LN encoder layer (fp64 | bf16-emulate)
  ramp          exit ramps, max-prob / entropy metrics, exit test
  model         per-input early-exit forward + brute-force variant
  llama         early-exit LLM decode step (RMSNorm/RoPE/KV cache/SwiGLU, LM-head ramp)
  pipeline_sim  split/queue bookkeeping of the constant-batch pipeline
  calibrate     per-ramp thresholds from a target exit profile

Parity status per function is stated in each module header and in DESIGN.md
§"Oracle pins".  Functions without an external pin say "parity unpinned".
"""
from .model import run, run_input, brute_force, ExitRecord  # noqa: F401
from .pipeline_sim import simulate_pipeline, Plan  # noqa: F401
