"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This package holds input formats and generators only -- none of the method's
arithmetic (no execution, marking, conflict detection or write-back).
"""
from . import formats, ycsb, tpcc  # noqa: F401
