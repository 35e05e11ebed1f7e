"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This package holds NO arithmetic of the enumeration method (no intersections, no ordering,
no checksum): it only produces edge lists.  Both sides of every parity check draw their input
from here and nowhere else.
"""
from .gen import (  # noqa: F401
    CONFIGS,
    SHAPES,
    er_bipartite,
    chung_lu_bipartite,
    planted_blocks,
    make_config,
    graph_stats,
)
from .small import g0_edges, crown_edges, complete_edges, star_edges, matching_edges  # noqa: F401
