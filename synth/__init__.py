"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle.

Holds none of the sampling method's arithmetic: only R-MAT graph generation,
edge-weight data, seed permutations and grid-valued dense matrices (PASS
features / projections).
"""
from .graphs import (CONFIGS, GraphSpec, degree_stats, make_graph, make_grid_matrix, make_feature_matrix,  # noqa: F401
                     make_seeds, small_graph)
