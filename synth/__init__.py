"""Seeded synthetic inputs shared by the CUDA path, the oracle and the benchmark.

This package holds NONE of the method's arithmetic (no assembly, no SpMV, no
PCG, no preconditioner): it only draws the inputs of K·d = F — per-block
diagonal terms and contact springs — from a seeded jittered-brick slope model
(DESIGN.md §3 "Input recipe").  Both `oracle/` and the product package consume
its arrays; neither imports the other.
"""
from .slope import (SlopeConfig, SlopeProblem, make_slope, preset, PRESETS,
                    random_vector, warm_start, case1_like)

__all__ = ["SlopeConfig", "SlopeProblem", "make_slope", "preset", "PRESETS",
           "random_vector", "warm_start", "case1_like"]
