"""Seeded synthetic inputs shared by the oracle tests and the CUDA path (no method arithmetic)."""
from .batch import Batch, Params  # noqa: F401
from .synth import make, seed_for  # noqa: F401
