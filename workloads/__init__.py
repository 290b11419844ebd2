"""Seeded synthetic workload generators shared by the CUDA path's tests/bench and the oracle.

Holds graph construction and file I/O only — none of the method's arithmetic (SURVEY.md §8(c),
task rule ③): no simulation, truth tables, supports or comparisons live here.
"""
from .aig import Aig, Builder, read_aag, write_aag, write_checks, write_pairs  # noqa: F401
from .circuits import (  # noqa: F401
    Miter, c1_add8, c2_mul12, c2_mul12_bug, c3_rand, c4_dp, c5_big, concat_miter, flip_fanin, random_miter,
    replicate, rewrite_copy, tiny_random,
)
