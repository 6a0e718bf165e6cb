"""Seeded input generators shared by tests, smoke() and bench.py (no method arithmetic)."""
from .synth import *  # noqa: F401,F403
from .synth import CONFIGS, Config, DTDG  # noqa: F401
