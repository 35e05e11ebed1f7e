"""Seeded synthetic bipartite generators (numpy PCG64), shaped like the paper's KONECT graphs.

Shapes (|U|, |V|, |E|, Delta(U), Delta(V)) come from PAPER.md Table 1; the recipe
is SURVEY.md Appendix A, reproduced call-for-call so the survey's seed-0 probe counts are a
full-scale cross-check.  See DESIGN.md "Input recipe".

Every function returns (n_u, n_v, edges) with edges a C-contiguous uint32 array of shape (m, 2),
rows (u, v), in the caller's orientation.  Nothing here knows about bicliques.
"""
import numpy as np

# (n_u, n_v, m, dmax_u, dmax_v) -- Table 1; GH |V| per SURVEY A13.
SHAPES = {
    "yg": (94238, 30087, 293360, 1035, 7591),
    "gh": (120867, 56519, 440237, 3675, 884),
    "bx": (340523, 105278, 1149739, 2502, 13601),
    "dblp": (5624219, 1953085, 12282059, 287, 1386),
}

# Named workloads.  "*_work" = Chung-Lu background + planted noisy dense blocks
# (SURVEY 8(d) "work-calibrated" variant); block parameters frozen here.  gh_work was calibrated
# (scripts/calibrate.py, seed 0) to 49,778,694 maximal bicliques vs Table 1's 55,346,398 for the
# real Github graph: 0.90x.
CONFIGS = {
    "er40": dict(kind="er", n_u=40, n_v=40, p=0.15, seed=0),
    "yg": dict(kind="cl", shape="yg", seed=0),
    "gh": dict(kind="cl", shape="gh", seed=0),
    "bx": dict(kind="cl", shape="bx", seed=0),
    "dblp": dict(kind="cl", shape="dblp", seed=0),
    "gh_work": dict(kind="work", shape="gh", seed=0, K=120, amin=26, amax=42, p_in=0.75),
    "gh_work_small": dict(kind="work", shape="gh", seed=0, K=40, amin=16, amax=40, p_in=0.6),
    # calibrated like gh_work (scripts/calibrate.py on B200, seed 0): yg_work 1,447,618 bicliques vs
    # Table 1's 1,826,587 for real YouTube (0.79x); bx_work 52,587,920 vs 54,458,953 for
    # real BookCrossing (0.96x)
    "yg_work": dict(kind="work", shape="yg", seed=0, K=100, amin=16, amax=40, p_in=0.6),
    "bx_work": dict(kind="work", shape="bx", seed=0, K=100, amin=26, amax=42, p_in=0.75),
}


def er_bipartite(n_u, n_v, p, seed):
    """Erdos-Renyi bipartite: A = default_rng(seed).random((n_u, n_v)) < p, edges = argwhere(A)."""
    rng = np.random.default_rng(seed)
    a = rng.random((n_u, n_v)) < p
    e = np.argwhere(a).astype(np.uint32)
    return n_u, n_v, np.ascontiguousarray(e)


def _weights(n, dmax, m):
    i = np.arange(1, n + 1, dtype=np.float64)
    lo, hi = 0.01, 3.0
    a = (lo + hi) / 2
    for _ in range(100):
        a = (lo + hi) / 2
        if np.sum(dmax * i ** -a) > m:
            lo = a
        else:
            hi = a
    return dmax * i ** -a


def chung_lu_bipartite(n_u, n_v, m, d_u, d_v, seed):
    """Power-law Chung-Lu bipartite graph with exactly m unique edges."""
    rng = np.random.default_rng(seed)
    wu = _weights(n_u, d_u, m)
    wv = _weights(n_v, d_v, m)
    pu_w = wu / wu.sum()
    pv_w = wv / wv.sum()
    big_m = m
    key = None
    for _ in range(20):
        u = rng.choice(n_u, size=big_m, p=pu_w)
        v = rng.choice(n_v, size=big_m, p=pv_w)
        key = np.unique(u.astype(np.int64) * n_v + v)
        if len(key) >= m:
            break
        big_m = int(big_m * m / len(key) * 1.02) + 1
    key = key[rng.permutation(len(key))[:m]]
    u = key // n_v
    v = key % n_v
    pu = rng.permutation(n_u)
    pv = rng.permutation(n_v)
    e = np.stack([pu[u], pv[v]], axis=1).astype(np.uint32)
    return n_u, n_v, np.ascontiguousarray(e)


def planted_blocks(n_u, n_v, edges, K, amin, amax, p_in, seed):
    """Plant K noisy dense a x b blocks (a, b uniform in [amin, amax], density p_in) whose members are
    drawn proportionally to (background degree + 1), then delete random background-only edges so the
    total stays |E| (block edges count against the budget)."""
    m = len(edges)
    rng2 = np.random.default_rng(1000 + seed)
    u = edges[:, 0].astype(np.int64)
    v = edges[:, 1].astype(np.int64)
    wu = np.bincount(u, minlength=n_u).astype(np.float64) + 1.0
    wv = np.bincount(v, minlength=n_v).astype(np.float64) + 1.0
    blocks = []
    for _ in range(K):
        a = int(rng2.integers(amin, amax + 1))
        b = int(rng2.integers(amin, amax + 1))
        ub = rng2.choice(n_u, a, replace=False, p=wu / wu.sum())
        vb = rng2.choice(n_v, b, replace=False, p=wv / wv.sum())
        mask = rng2.random((a, b)) < p_in
        ii, jj = np.nonzero(mask)
        blocks.append(ub[ii].astype(np.int64) * n_v + vb[jj])
    bkey = np.unique(np.concatenate(blocks)) if blocks else np.zeros(0, np.int64)
    bg = u * n_v + v
    bg_only = bg[~np.isin(bg, bkey)]
    keep_bg = m - len(bkey)
    if keep_bg < 0:
        raise ValueError("planted blocks exceed the edge budget")
    sel = np.sort(rng2.choice(len(bg_only), keep_bg, replace=False))
    key = np.concatenate([bg_only[sel], bkey])
    key = key[rng2.permutation(len(key))]
    e = np.stack([key // n_v, key % n_v], axis=1).astype(np.uint32)
    return n_u, n_v, np.ascontiguousarray(e)


def make_config(name_or_dict):
    """Build a named (or explicit) workload -> (n_u, n_v, edges uint32[m,2])."""
    c = CONFIGS[name_or_dict] if isinstance(name_or_dict, str) else dict(name_or_dict)
    kind = c["kind"]
    if kind == "er":
        return er_bipartite(c["n_u"], c["n_v"], c["p"], c["seed"])
    n_u, n_v, m, du, dv = SHAPES[c["shape"]]
    g = chung_lu_bipartite(n_u, n_v, m, du, dv, c["seed"])
    if kind == "cl":
        return g
    if kind == "work":
        return planted_blocks(g[0], g[1], g[2], c["K"], c["amin"], c["amax"], c["p_in"], c["seed"])
    raise ValueError(kind)


def graph_stats(n_u, n_v, edges):
    """Achieved |E| (unique) and max degrees -- for recording, not for the method."""
    key = np.unique(edges[:, 0].astype(np.int64) * n_v + edges[:, 1])
    u = key // n_v
    v = key % n_v
    du = np.bincount(u, minlength=n_u)
    dv = np.bincount(v, minlength=n_v)
    return dict(n_u=n_u, n_v=n_v, m=int(len(key)), delta_u=int(du.max(initial=0)),
                delta_v=int(dv.max(initial=0)))
