"""Seeded synthetic inputs shared by the tests, the bench and smoke().

Holds NONE of the method's arithmetic (no SAD, no interpolation filter, no
spiral order): only random-number generation and plain array indexing.  Both
the oracle and the CUDA path receive the same arrays from here.  Recipes are
stated in DESIGN.md §5 (workload shapes follow BASELINE.json `configs` and the
paper's 1080p IPPP workloads, P:258-P:260).
"""
from .frames import (CONFIGS, Config, gen_flat, gen_noise, gen_shifted, gen_tex,
                     ippp_sequence, make_workload)

__all__ = ["CONFIGS", "Config", "gen_flat", "gen_noise", "gen_shifted", "gen_tex",
           "ippp_sequence", "make_workload"]
