"""Seeded synthetic input generators shared by the oracle-side tests and the CUDA-side tests/bench.

This module holds NO arithmetic of the method (no SAXPY, SpMV, stencil, GEMM, wrapper or
scheduling logic): it only draws random inputs with the shapes, value distributions and
structure stated in SURVEY.md §8(d) / DESIGN.md "Input recipe". Both `oracle/` and the product
path may consume what it returns; neither side imports the other.
"""
from .gen import *  # noqa: F401,F403
