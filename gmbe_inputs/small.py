"""Tiny hand-made bipartite graphs (edge lists only, 0-based ids, rows are (u, v)).

G0 is the paper's running example (Fig 1; Fig 2): u1..u5 -> 0..4,
v1..v4 -> 0..3, with N(v1)={u1,u2}, N(v2)={u1,u2,u3,u4} (Fig 2),
N(v3)={u1,u2,u4}, N(v4)={u2,u4,u5}.
"""
import numpy as np


def _arr(pairs):
    a = np.asarray(pairs, dtype=np.uint32)
    return a.reshape(-1, 2)


def g0_edges():
    """Paper Fig 1 graph G0 (exactly 6 maximal bicliques)."""
    nv = {0: [0, 1], 1: [0, 1, 2, 3], 2: [0, 1, 3], 3: [1, 3, 4]}
    pairs = sorted((u, v) for v, us in nv.items() for u in us)
    return 5, 4, _arr(pairs)


def crown_edges(n):
    """Crown graph: K_{n,n} minus a perfect matching (2^n - 2 maximal bicliques)."""
    pairs = [(u, v) for u in range(n) for v in range(n) if u != v]
    return n, n, _arr(pairs)


def complete_edges(a, b):
    pairs = [(u, v) for u in range(a) for v in range(b)]
    return a, b, _arr(pairs)


def star_edges(n, center_on_u=True):
    if center_on_u:
        return 1, n, _arr([(0, v) for v in range(n)])
    return n, 1, _arr([(u, 0) for u in range(n)])


def matching_edges(n):
    return n, n, _arr([(i, i) for i in range(n)])
