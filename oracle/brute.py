"""Brute-force MBE -- TEST INFRASTRUCTURE ONLY; pins the C++ oracle.

(i)  literal: every non-empty R ⊆ V, L = Γ(R); keep (L, R) if L ≠ ∅ and Γ(L) = R
     (definition of a maximal biclique, with both sides non-empty, reading A1).
(ii) restricted-exact: every non-empty R ⊆ N(u) for each u (complete because u ∈ L ⇒ R ⊆ N(u)).

Pure Python sets; the checksum formula is re-implemented here from DESIGN.md "Checksum" so the
brute force shares no code with the C++ oracle either.
"""
from itertools import combinations

M64 = (1 << 64) - 1


def _mix(x):
    x &= M64
    x ^= x >> 30
    x = (x * 0xBF58476D1CE4E5B9) & M64
    x ^= x >> 27
    x = (x * 0x94D049BB133111EB) & M64
    x ^= x >> 31
    return x


def h_u(u):
    return _mix(2 * u + 0x9E3779B97F4A7C15)


def h_v(v):
    return _mix(2 * v + 1 + 0x9E3779B97F4A7C15)


def h_pair(l_ids, r_ids):
    sl = sum(h_u(u) for u in l_ids) & M64
    sr = sum(h_v(v) for v in r_ids) & M64
    return _mix(sl + 0xD6E8FEB86659FD93 * _mix(sr))


def checksum(bicliques):
    return sum(h_pair(l_, r_) for l_, r_ in bicliques) & M64


def _adj(n_u, n_v, edges):
    nu = [set() for _ in range(n_u)]
    nv = [set() for _ in range(n_v)]
    for u, v in edges:
        nu[int(u)].add(int(v))
        nv[int(v)].add(int(u))
    return nu, nv


def _gamma(sets, members, universe):
    g = set(universe)
    for x in members:
        g &= sets[x]
    return g


def brute_literal(n_u, n_v, edges):
    """All maximal bicliques by enumerating every non-empty R ⊆ V (|V| <= ~16)."""
    nu, nv = _adj(n_u, n_v, edges)
    out = set()
    vs = range(n_v)
    for size in range(1, n_v + 1):
        for r in combinations(vs, size):
            l_ = _gamma(nv, r, range(n_u))
            if not l_:
                continue
            if _gamma(nu, l_, range(n_v)) == set(r):
                out.add((tuple(sorted(l_)), tuple(r)))
    return sorted(out)


def brute_restricted(n_u, n_v, edges):
    """All maximal bicliques via every non-empty R ⊆ N(u), deduplicated."""
    nu, nv = _adj(n_u, n_v, edges)
    out = set()
    for u in range(n_u):
        nbr = sorted(nu[u])
        for size in range(1, len(nbr) + 1):
            for r in combinations(nbr, size):
                l_ = _gamma(nv, r, range(n_u))
                if _gamma(nu, l_, range(n_v)) == set(r):
                    out.add((tuple(sorted(l_)), tuple(r)))
    return sorted(out)
