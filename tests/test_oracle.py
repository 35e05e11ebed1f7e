"""Pins for the CPU oracle: paper worked example, brute force, closed forms,
Galois closure, invariances.  CPU only."""
import json
import os

import numpy as np
import pytest

import oracle
from oracle.brute import brute_literal, brute_restricted, checksum, h_pair
from gmbe_inputs import (complete_edges, crown_edges, g0_edges, make_config, matching_edges,
                         star_edges)

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def _set(res):
    return sorted(res.bicliques)


# ---------------------------------------------------------------- paper's G0 (Fig 1/2, Ex 2.1, 4.1)
def test_g0_paper_bicliques():
    g = _gold("g0_paper.json")
    nu, nv, e = g0_edges()
    expect = sorted((tuple(l_), tuple(r_)) for l_, r_ in g["maximal"].values())
    for order in ("degree", "identity"):
        for prune in (True, False):
            r = oracle.oracle_mbe(nu, nv, e, order=order, prune=prune, records=True,
                                  check_closure=True)
            assert r.count == g["count"] == 6
            assert _set(r) == expect
            assert r.closure_failures == 0
    # the non-maximal nodes of Fig 2 are indeed not maximal
    for l_, r_ in g["non_maximal"].values():
        assert (tuple(l_), tuple(r_)) not in expect


def test_g0_tree_mechanics_identity_order():
    """Fig 2 / Ex 4.1: identity order, root v3 skipped (Alg 3 L7), t1 pruned by Thm 4.1."""
    g = _gold("g0_paper.json")["identity_order_tree"]
    nu, nv, e = g0_edges()
    on = oracle.oracle_mbe(nu, nv, e, order="identity", prune=True, per_root=True)
    off = oracle.oracle_mbe(nu, nv, e, order="identity", prune=False)
    assert on.roots_run == g["roots_run"] == 3
    assert (on.nodes, on.nonmax) == (g["prune_on"]["nodes"], g["prune_on"]["nonmax"])
    assert (off.nodes, off.nonmax) == (g["prune_off"]["nodes"], g["prune_off"]["nonmax"])
    # per-root ownership: p-root+q under v1, r+s+t under v2, nothing under v3 (skipped), x under v4
    assert on.per_root_count.tolist() == [2, 3, 0, 1]


def test_g0_checksum_vs_brute_and_survey():
    kn = _gold("survey_known_answers.json")
    nu, nv, e = g0_edges()
    b = brute_literal(nu, nv, e)
    for (l_, r_) in b:
        key = json.dumps([list(l_), list(r_)]).replace(" ", "")
        assert h_pair(l_, r_) == int(kn["g0_h"][key], 16)
    r = oracle.oracle_mbe(nu, nv, e)
    assert r.checksum == checksum(b) == int(kn["g0_checksum"], 16)
    # transposition: U <-> V swaps the roles, so the domain-separated hash changes (by design)
    rt = oracle.oracle_mbe(nv, nu, e[:, ::-1].copy())
    assert rt.count == 6 and rt.checksum == int(kn["g0_transposed_checksum"], 16)


# ---------------------------------------------------------------- brute force on random tiny graphs
def _rand_graph(rng):
    nu = int(rng.integers(1, 10))
    nv = int(rng.integers(1, 10))
    p = float(rng.choice([0.2, 0.35, 0.5, 0.65, 0.8]))
    a = rng.random((nu, nv)) < p
    e = np.argwhere(a).astype(np.uint32)
    if len(e) and rng.random() < 0.3:  # duplicate some edges (multi-edges collapse)
        e = np.concatenate([e, e[rng.integers(0, len(e), size=3)]])
    return nu, nv, e


@pytest.mark.parametrize("block", range(6))
def test_random_tiny_vs_brute(block):
    rng = np.random.default_rng(1234 + block)
    for _ in range(250):
        nu, nv, e = _rand_graph(rng)
        b = brute_literal(nu, nv, e)
        cs = checksum(b)
        for order in ("degree", "identity"):
            for prune in (True, False):
                r = oracle.oracle_mbe(nu, nv, e, order=order, prune=prune, records=True,
                                      check_closure=True)
                assert r.count == len(b)
                assert r.checksum == cs
                assert _set(r) == b
                assert r.closure_failures == 0
                # every biclique exactly once (no duplicates in the record stream)
                assert len(set(r.bicliques)) == len(r.bicliques)


def test_pruning_reduces_exactly_nonmaximal_nodes():
    """Thm 4.1 only removes non-maximal nodes: nodes_off - nodes_on == nonmax_off - nonmax_on."""
    rng = np.random.default_rng(7)
    for _ in range(300):
        nu, nv, e = _rand_graph(rng)
        on = oracle.oracle_mbe(nu, nv, e, prune=True)
        off = oracle.oracle_mbe(nu, nv, e, prune=False)
        assert on.count == off.count and on.checksum == off.checksum
        assert off.nodes - on.nodes == off.nonmax - on.nonmax >= 0


# ---------------------------------------------------------------- ER(40,40,.15): restricted brute force
def test_er40_restricted_brute():
    nu, nv, e = make_config("er40")
    assert len(e) == 239
    b = brute_restricted(nu, nv, e)
    assert len(b) == 211
    for prune in (True, False):
        r = oracle.oracle_mbe(nu, nv, e, prune=prune, records=True, check_closure=True)
        assert r.count == 211 and _set(r) == b and r.checksum == checksum(b)
        assert r.closure_failures == 0


# ---------------------------------------------------------------- closed forms
@pytest.mark.parametrize("n", range(2, 11))
def test_crown_graph(n):
    nu, nv, e = crown_edges(n)
    r = oracle.oracle_mbe(nu, nv, e)
    assert r.count == 2 ** n - 2


def test_crown_brute_checksum():
    for n in range(2, 8):
        nu, nv, e = crown_edges(n)
        assert oracle.oracle_mbe(nu, nv, e).checksum == checksum(brute_literal(nu, nv, e))


@pytest.mark.parametrize("a,b", [(1, 1), (3, 5), (7, 2), (10, 10)])
def test_complete(a, b):
    nu, nv, e = complete_edges(a, b)
    r = oracle.oracle_mbe(nu, nv, e, records=True)
    assert r.count == 1 and r.bicliques == [(tuple(range(a)), tuple(range(b)))]


def test_star_matching_empty():
    for cu in (True, False):
        nu, nv, e = star_edges(9, cu)
        assert oracle.oracle_mbe(nu, nv, e).count == 1
    nu, nv, e = matching_edges(12)
    r = oracle.oracle_mbe(nu, nv, e, records=True)
    assert r.count == 12 and r.bicliques == sorted(((i,), (i,)) for i in range(12))
    r = oracle.oracle_mbe(5, 7, np.zeros((0, 2), np.uint32))
    assert (r.count, r.checksum) == (0, 0)
    r = oracle.oracle_mbe(0, 0, np.zeros((0, 2), np.uint32))
    assert (r.count, r.checksum) == (0, 0)


def test_invalid_ids_rejected():
    with pytest.raises(ValueError):
        oracle.oracle_mbe(2, 2, np.array([[0, 2]], np.uint32))


# ---------------------------------------------------------------- invariances
def test_invariances_er40():
    nu, nv, e = make_config("er40")
    base = oracle.oracle_mbe(nu, nv, e)
    rng = np.random.default_rng(3)
    # edge permutation
    r = oracle.oracle_mbe(nu, nv, e[rng.permutation(len(e))])
    assert (r.count, r.checksum) == (base.count, base.checksum)
    # relabelling: bicliques map through the permutation
    pu, pv = rng.permutation(nu), rng.permutation(nv)
    e2 = np.stack([pu[e[:, 0]], pv[e[:, 1]]], 1).astype(np.uint32)
    a = oracle.oracle_mbe(nu, nv, e, records=True)
    b = oracle.oracle_mbe(nu, nv, e2, records=True)
    mapped = sorted((tuple(sorted(pu[list(l_)].tolist())), tuple(sorted(pv[list(r_)].tolist())))
                    for l_, r_ in a.bicliques)
    assert mapped == _set(b)
    # transposition: pairs swap sides
    t = oracle.oracle_mbe(nv, nu, e[:, ::-1].copy(), records=True)
    assert sorted((r_, l_) for l_, r_ in t.bicliques) == _set(a)
    # order / prune
    for order in ("degree", "identity"):
        for prune in (True, False):
            r = oracle.oracle_mbe(nu, nv, e, order=order, prune=prune)
            assert (r.count, r.checksum) == (base.count, base.checksum)


def test_shards_are_additive():
    """Ownership invariant: each biclique is emitted under exactly one root (its min-rank R vertex),
    so shards over roots partition the output."""
    nu, nv, e = make_config("er40")
    base = oracle.oracle_mbe(nu, nv, e)
    for n in (2, 3, 8):
        parts = [oracle.oracle_mbe(nu, nv, e, shard=(i, n)) for i in range(n)]
        assert sum(p.count for p in parts) == base.count
        assert sum(p.checksum for p in parts) % (1 << 64) == base.checksum
        assert sum(p.nodes for p in parts) == base.nodes
        assert sum(p.algo_bytes for p in parts) == base.algo_bytes


def test_swapped_orientation_counts():
    """|U| < |V| => the sides are swapped internally; output stays in caller roles."""
    rng = np.random.default_rng(11)
    for _ in range(100):
        nu = int(rng.integers(1, 6))
        nv = int(rng.integers(nu + 1, 10))
        e = np.argwhere(rng.random((nu, nv)) < 0.5).astype(np.uint32)
        b = brute_literal(nu, nv, e)
        r = oracle.oracle_mbe(nu, nv, e, records=True, check_closure=True)
        assert _set(r) == b and r.checksum == checksum(b) and r.closure_failures == 0


# ---------------------------------------------------------------- survey cross-check table
def test_survey_counter_table():
    kn = _gold("survey_known_answers.json")
    graphs = {"g0": g0_edges(), "er40": make_config("er40"), "crown4": crown_edges(4),
              "crown12": crown_edges(12)}
    for row in kn["counters"]:
        nu, nv, e = graphs[row["graph"]]
        r = oracle.oracle_mbe(nu, nv, e, order=row["order"], prune=row["prune"])
        got = dict(count=r.count, nodes=r.nodes, nonmax=r.nonmax, algo_bytes=r.algo_bytes,
                   algo_bytes_qfull=r.algo_bytes_qfull)
        assert got == {k: row[k] for k in got}, row
    nu, nv, e = crown_edges(4)
    assert oracle.oracle_mbe(nu, nv, e).checksum == int(kn["crown4"]["checksum"], 16)


def test_config_goldens_match_survey_probe():
    """The stored oracle goldens of the degree-shaped configs reproduce the survey's independent
    probe numbers (seed-0 Chung-Lu, a third implementation): count, nodes and
    nonmax of the canonical tree.  Pins the goldens bench.py and the GPU tests compare against."""
    probe = _gold("survey_known_answers.json")["probe_counts_seed0"]
    cfg = _gold("configs_oracle.json")
    for name in ("yg", "gh", "bx", "dblp"):
        assert cfg[name]["count"] == probe[name], name
        for k in ("nodes", "nonmax"):
            if "%s_%s" % (name, k) in probe:
                assert cfg[name][k] == probe["%s_%s" % (name, k)], (name, k)
