"""Seeded synthetic inputs shared by the oracle-side tests and the CUDA path (no method arithmetic)."""
from .netlist import *  # noqa: F401,F403
