"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This package holds NONE of the transposition arithmetic: only the
counter-based input generator (SplitMix64 over the linear input index) and
the catalogue of workload shapes/permutations taken from BASELINE.json's
configs (recipe in DESIGN.md "Inputs").
"""
from .gen import (splitmix64_np, gen_bits_np, gen_tensor_np, gen_tensor_torch, gen_at_np,
                  case_seed, SEED_BASE)
from . import configs

__all__ = ["splitmix64_np", "gen_at_np", "gen_bits_np", "gen_tensor_np", "gen_tensor_torch",
           "case_seed", "SEED_BASE", "configs"]
