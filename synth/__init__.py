"""Seeded synthetic input generators (no method arithmetic). See synth/gen.py."""
from .gen import *  # noqa: F401,F403
