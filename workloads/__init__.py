"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This package holds NO arithmetic of the method (no norm, projection, attention,
LoRA or optimizer math).  It only draws random numbers, rounds them to
bf16-representable values (an input *encoding*, so both sides see identical
bits), and describes the BASELINE.json workloads (shapes, client mix).
The recipe is documented in DESIGN.md §"Input recipe".
"""
from .synth import *  # noqa: F401,F403
