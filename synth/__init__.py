"""Seeded synthetic graph inputs shared by the tests, the bench and smoke().

This package holds NO arithmetic of the MSF method: it only draws graphs
(CSR with both edge directions, integer weights) with the shapes of the
paper's input families (§4, Table 2).  Both the CUDA
path and the CPU oracle consume its output; neither is imported here.
"""
from .rng import splitmix64_py, hash_u64, uniform_int31, uniform_f64
from .graphs import (
    Graph,
    csr_from_pairs,
    grid2d,
    road_like,
    rgg2d,
    rmat,
    uniform_random,
    random_small,
    complete_graph,
    path_graph,
    cycle_graph,
    star_graph,
    make_config,
    CONFIGS,
)

__all__ = [
    "splitmix64_py", "hash_u64", "uniform_int31", "uniform_f64",
    "Graph", "csr_from_pairs", "grid2d", "road_like", "rgg2d", "rmat",
    "uniform_random", "random_small", "complete_graph", "path_graph",
    "cycle_graph", "star_graph", "make_config", "CONFIGS",
]
