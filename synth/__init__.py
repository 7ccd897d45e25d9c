"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle.

Holds none of the sampling method's arithmetic: only R-MAT graph generation,
edge-weight data and seed permutations.
"""
from .graphs import (CONFIGS, GraphSpec, degree_stats, make_graph, make_seeds,  # noqa: F401
                     small_graph)
