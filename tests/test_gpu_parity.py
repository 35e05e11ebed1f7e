"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by element.

Count and checksum must be bit-exact; on small inputs the full biclique SET must be equal; the
canonical-tree counters (nodes, nonmax, algo_bytes_cand) must match exactly (schedule-independent,
DESIGN.md reading A9).  Marked gpu: run on the B200 box."""
import json
import os

import numpy as np
import pytest

import oracle
from gmbe_inputs import complete_edges, crown_edges, g0_edges, make_config, matching_edges, star_edges

pytestmark = pytest.mark.gpu

GOLD = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module")
def gmbe():
    import torch
    assert torch.cuda.is_available()
    import paper_conf_sc_panhlzwc23_b200 as m
    return m


def _run(gmbe, nu, nv, e, order="degree", **kw):
    g = gmbe.load(nu, nv, e, order=order)
    try:
        return g.enumerate(**kw)
    finally:
        g.free()


def _same(r, o):
    assert (r.count, r.checksum) == (o.count, o.checksum)
    assert (r.roots_run, r.nodes, r.nonmax) == (o.roots_run, o.nodes, o.nonmax)
    assert r.algo_bytes_cand == o.algo_bytes_cand


# ---------------------------------------------------------------- paper worked example
def test_g0_sets_and_tree(gmbe):
    nu, nv, e = g0_edges()
    for order in ("identity", "degree"):
        for prune in (True, False):
            r = _run(gmbe, nu, nv, e, order=order, prune=prune, records=True,
                     per_root=True)
            o = oracle.oracle_mbe(nu, nv, e, order=order, prune=prune, records=True, per_root=True)
            _same(r, o)
            assert r.bicliques == sorted(o.bicliques)
            assert r.algo_bytes_cand == o.algo_bytes_cand
            assert r.per_root_count.tolist() == o.per_root_count.tolist()
    # Fig 2 / Ex 4.1: identity order, t1 pruned
    r = _run(gmbe, nu, nv, e, order="identity")
    assert (r.count, r.nodes, r.nonmax, r.roots_run) == (6, 3, 0, 3)


# ---------------------------------------------------------------- random tiny graphs
def _rand_graph(rng, nmax=10):
    nu = int(rng.integers(1, nmax))
    nv = int(rng.integers(1, nmax))
    p = float(rng.choice([0.2, 0.35, 0.5, 0.65, 0.8]))
    e = np.argwhere(rng.random((nu, nv)) < p).astype(np.uint32)
    if len(e) and rng.random() < 0.3:
        e = np.concatenate([e, e[rng.integers(0, len(e), size=3)]])
    return nu, nv, e


def test_random_tiny_sets(gmbe):
    rng = np.random.default_rng(99)
    for _ in range(300):
        nu, nv, e = _rand_graph(rng)
        order = "degree" if rng.random() < 0.7 else "identity"
        prune = bool(rng.random() < 0.8)
        r = _run(gmbe, nu, nv, e, order=order, prune=prune, records=True)
        o = oracle.oracle_mbe(nu, nv, e, order=order, prune=prune, records=True)
        _same(r, o)
        assert r.bicliques == sorted(o.bicliques)
        assert r.algo_bytes_cand == o.algo_bytes_cand


def test_random_medium_dense(gmbe):
    """Denser and larger than tiny: spans several 32-bit words per row (W > 1) and ragged tails."""
    rng = np.random.default_rng(5)
    for it in range(40):
        nu = int(rng.integers(20, 140))
        nv = int(rng.integers(10, 60))
        p = float(rng.uniform(0.05, 0.35))
        e = np.argwhere(rng.random((nu, nv)) < p).astype(np.uint32)
        o = oracle.oracle_mbe(nu, nv, e)
        r = _run(gmbe, nu, nv, e)
        _same(r, o)
        assert r.algo_bytes_cand == o.algo_bytes_cand


# ---------------------------------------------------------------- closed forms / edge cases
def test_closed_forms(gmbe):
    for n in range(2, 15):
        nu, nv, e = crown_edges(n)
        r = _run(gmbe, nu, nv, e)
        assert r.count == 2 ** n - 2
        if n <= 10:
            o = oracle.oracle_mbe(nu, nv, e)
            _same(r, o)
    for a, b in ((1, 1), (3, 5), (40, 2), (33, 70)):
        r = _run(gmbe, *complete_edges(a, b), records=True)
        assert r.count == 1 and r.bicliques == [(tuple(range(a)), tuple(range(b)))]
    r = _run(gmbe, *matching_edges(50))
    assert r.count == 50
    r = _run(gmbe, *star_edges(100))
    assert r.count == 1
    r = _run(gmbe, 7, 9, np.zeros((0, 2), np.uint32))
    assert (r.count, r.checksum) == (0, 0)


def test_invalid_ids(gmbe):
    with pytest.raises(gmbe.GmbeError) as ei:
        gmbe.load(3, 3, np.array([[0, 3]], np.uint32))
    assert ei.value.code == gmbe.GMBE_EINVAL


def test_swapped_orientation_sets(gmbe):
    """|U| < |V|: the library swaps sides internally; output stays in caller roles."""
    rng = np.random.default_rng(12)
    for _ in range(50):
        nu = int(rng.integers(1, 8))
        nv = int(rng.integers(nu + 1, 14))
        e = np.argwhere(rng.random((nu, nv)) < 0.45).astype(np.uint32)
        r = _run(gmbe, nu, nv, e, records=True)
        o = oracle.oracle_mbe(nu, nv, e, records=True)
        _same(r, o)
        assert r.bicliques == sorted(o.bicliques)


# ---------------------------------------------------------------- ER(40,40,.15)
def test_er40(gmbe):
    nu, nv, e = make_config("er40")
    for prune in (True, False):
        r = _run(gmbe, nu, nv, e, prune=prune, records=True)
        o = oracle.oracle_mbe(nu, nv, e, prune=prune, records=True)
        _same(r, o)
        assert r.count == 211
        assert r.bicliques == sorted(o.bicliques)
        assert r.algo_bytes_cand == o.algo_bytes_cand


# ---------------------------------------------------------------- schedule freedom (A9)
@pytest.fixture(scope="module")
def dense_case():
    rng = np.random.default_rng(2024)
    nu, nv = 90, 60
    a = rng.random((nu, nv)) < 0.12
    a[:24, :20] |= rng.random((24, 20)) < 0.75  # one dense block -> deep, heavy subtrees
    e = np.argwhere(a).astype(np.uint32)
    o = oracle.oracle_mbe(nu, nv, e, records=True)
    return nu, nv, e, o


def test_split_and_schedule_invariance(gmbe, dense_case):
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        variants = [dict(), dict(split=False), dict(bound_height=1, bound_size=1),
                    dict(bound_height=1, bound_size=1, pool_words=64),
                    dict(bound_height=1, bound_size=1, pool_words=4096),
                    dict(warps_per_sm=8), dict(warps_per_sm=64),
                    dict(bound_height=2, bound_size=8, pool_words=2048), dict(arena_words=4096)]
        for kw in variants:
            r = g.enumerate(**kw)
            _same(r, o)
            assert r.algo_bytes_cand == o.algo_bytes_cand, kw
        for pw in (0, 1024):
            r = g.enumerate(bound_height=1, bound_size=1, records=True, pool_words=pw)
            assert r.splits > 0 and (r.tasks > 0 or pw)
            assert r.bicliques == sorted(o.bicliques)
    finally:
        g.free()


def test_donation_invariance(gmbe, dense_case):
    """Dynamic donation (debug bit 8: donate at every opportunity, bit 4: never) hands the remaining
    children of a warp's shallowest level to the queue; the tree, the counters and the records must
    be those of the canonical tree (DESIGN.md §5.2 "Dynamic donation")."""
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        for dbg in (8, 4, 12):
            r = g.enumerate(debug=dbg, records=True)
            _same(r, o)
            assert r.algo_bytes_cand == o.algo_bytes_cand
            assert r.bicliques == sorted(o.bicliques)
            assert (r.donations > 0) == (dbg == 8), (dbg, r.donations)
        r = g.enumerate(debug=8, bound_height=1, bound_size=1, records=True)
        _same(r, o)
        assert r.bicliques == sorted(o.bicliques)
    finally:
        g.free()


def test_parts_are_additive(gmbe, dense_case):
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        for n in (2, 3, 8):
            rs = [g.enumerate(part=(i, n)) for i in range(n)]
            assert sum(x.count for x in rs) == o.count
            assert sum(x.checksum for x in rs) % (1 << 64) == o.checksum
            assert sum(x.nodes for x in rs) == o.nodes
            assert sum(x.algo_bytes_cand for x in rs) == o.algo_bytes_cand
            for i in range(n):  # per-shard parity (ownership invariant)
                os_ = oracle.oracle_mbe(nu, nv, e, shard=(i, n))
                assert (rs[i].count, rs[i].checksum) == (os_.count, os_.checksum)
    finally:
        g.free()


def test_output_truncation(gmbe, dense_case):
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        r = g.enumerate(records=True, rec_cap=10, ids_cap=1 << 20)
        assert r.truncated == 1 and r.count == o.count and r.checksum == o.checksum
        assert r.n_written == 10 and set(r.bicliques) <= set(o.bicliques)
        r = g.enumerate(records=True, rec_cap=1 << 16, ids_cap=100)
        assert r.truncated == 1 and r.count == o.count
    finally:
        g.free()


def test_device_edges_and_duplicates(gmbe):
    import torch
    nu, nv, e = make_config("er40")
    dup = np.concatenate([e, e[::3]])
    t = torch.from_numpy(dup.astype(np.int32)).cuda()
    g = gmbe.load(nu, nv, t)
    r = g.enumerate()
    info = g.info()
    g.free()
    assert info["n_edges_unique"] == 239
    assert (r.count, r.checksum) == (211, 0x357D6B7B401275D4)


# ---------------------------------------------------------------- full-size configs
def _gold_cfg():
    p = os.path.join(GOLD, "configs_oracle.json")
    with open(p) as f:
        return json.load(f)


@pytest.mark.parametrize("name", ["yg", "gh", "dblp", "bx", "gh_work", "yg_work", "bx_work"])
def test_full_config_vs_oracle_golden(gmbe, name):
    gold = _gold_cfg()
    if name not in gold:
        pytest.skip("no golden for %s" % name)
    gd = gold[name]
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    try:
        r = g.enumerate()
        assert (r.count, r.checksum) == (gd["count"], int(gd["checksum"], 16))
        assert (r.nodes, r.nonmax, r.roots_run) == (gd["nodes"], gd["nonmax"], gd["roots_run"])
        if "algo_bytes_cand" in gd:
            assert r.algo_bytes_cand == gd["algo_bytes_cand"]
    finally:
        g.free()


@pytest.mark.parametrize("name,n", [("gh_work", 8), ("dblp", 8), ("gh", 2)])
def test_full_config_shards_vs_golden(gmbe, name, n):
    """The bench's multi-GPU launch configuration (root shard i of n per rank, one all-reduce):
    the shards' sums equal the whole-graph golden bit-exactly."""
    gd = _gold_cfg()[name]
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    try:
        rs = [g.enumerate(part=(i, n)) for i in range(n)]
        assert sum(r.count for r in rs) == gd["count"]
        assert sum(r.checksum for r in rs) % (1 << 64) == int(gd["checksum"], 16)
        assert sum(r.nodes for r in rs) == gd["nodes"]
        assert sum(r.nonmax for r in rs) == gd["nonmax"]
    finally:
        g.free()


@pytest.mark.parametrize("name", ["gh_work_small", "yg"])
def test_full_config_forced_donation(gmbe, name):
    gd = _gold_cfg()[name]
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    try:
        r = g.enumerate(debug=8)
        assert r.donations > 0 or name != "gh_work_small"
        assert (r.count, r.checksum) == (gd["count"], int(gd["checksum"], 16))
        assert (r.nodes, r.nonmax, r.roots_run) == (gd["nodes"], gd["nonmax"], gd["roots_run"])
    finally:
        g.free()


# ---------------------------------------------------------------- thread-level tier (run_thr)
def test_thread_tier_invariance(gmbe, dense_case):
    """The thread-level subtree tier (one subtree per lane, in-warp donation) and the warp-level tier
    walk the same canonical tree: identical sets, counts, checksums and counters."""
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        st = g.enumerate(thr_min=1, debug=32, phases=True)
        ph = list(st.phase_cycles.values())
        assert ph[1] > 0, "thread tier not exercised"
        _same(st, o)
        for kw in (dict(debug=16), dict(thr_min=1), dict(thr_min=1, debug=8), dict(thr_min=1, debug=4),
                   dict(thr_min=1, bound_height=1, bound_size=1), dict(thr_min=1, warps_per_sm=64),
                   dict(thr_min=1 << 20)):
            r = g.enumerate(records=True, **kw)
            _same(r, o)
            assert r.bicliques == sorted(o.bicliques), kw
        o2 = oracle.oracle_mbe(nu, nv, e, prune=False)
        r = g.enumerate(prune=False, thr_min=1)
        _same(r, o2)
    finally:
        g.free()


def test_thread_tier_random(gmbe):
    """Random dense graphs with planted blocks, every eligible job on the thread tier."""
    rng = np.random.default_rng(31)
    for it in range(60):
        nu, nv = int(rng.integers(8, 70)), int(rng.integers(8, 64))
        a = rng.random((nu, nv)) < float(rng.uniform(0.05, 0.4))
        a[: nu // 2, : nv // 3] |= rng.random((nu // 2, nv // 3)) < 0.8
        e = np.argwhere(a).astype(np.uint32)
        o = oracle.oracle_mbe(nu, nv, e, records=True)
        g = gmbe.load(nu, nv, e)
        try:
            for kw in (dict(thr_min=1), dict(thr_min=1, debug=8)):
                r = g.enumerate(records=True, rec_cap=1 << 18, ids_cap=1 << 24, **kw)
                _same(r, o)
                if not r.truncated:
                    assert r.bicliques == sorted(o.bicliques), (it, kw)
        finally:
            g.free()


def test_suffix_mode_roots(gmbe, dense_case):
    """Suffix-mode roots (k counted over later ranks only, Alg 3 L7 by an earlier-dominator search,
    no Γ index; reading B5) give the canonical tree: forced on every root (debug 128)."""
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        for kw in (dict(debug=128), dict(debug=128 | 16), dict(debug=128, bound_height=1, bound_size=1)):
            r = g.enumerate(records=True, **kw)
            _same(r, o)
            assert r.bicliques == sorted(o.bicliques), kw
    finally:
        g.free()
    rng = np.random.default_rng(77)
    for it in range(80):
        nu, nv, e = _rand_graph(rng, nmax=14)
        o = oracle.oracle_mbe(nu, nv, e, records=True)
        r = _run(gmbe, nu, nv, e, records=True, debug=128)
        _same(r, o)
        assert r.bicliques == sorted(o.bicliques)


def test_wide_universe_splitting(gmbe):
    """Universes above 64 bits (W > 2 words per row) with the wide-universe split rule forced on
    every node with >= 2 candidates (split_wide=1): same tree, counters and sets."""
    rng = np.random.default_rng(123)
    for it in range(12):
        nu, nv = int(rng.integers(120, 260)), int(rng.integers(20, 45))
        a = rng.random((nu, nv)) < float(rng.uniform(0.25, 0.5))
        e = np.argwhere(a).astype(np.uint32)
        o = oracle.oracle_mbe(nu, nv, e, records=True)
        g = gmbe.load(nu, nv, e)
        try:
            for kw in (dict(split_wide=1), dict(split_wide=1, debug=128), dict(split_wide=1 << 30)):
                r = g.enumerate(records=True, rec_cap=1 << 18, ids_cap=1 << 24, **kw)
                _same(r, o)
                if not r.truncated:
                    assert r.bicliques == sorted(o.bicliques), (it, kw)
        finally:
            g.free()


def test_dense_mode_roots(gmbe, dense_case):
    """Dense-mode roots (the warp table indexed by rank, rank-ordered occupied list, no candidate
    sort) forced on every root (debug 512), alone and with suffix mode (debug 128)."""
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        for dbg in (512, 512 | 128, 512 | 16):
            r = g.enumerate(records=True, debug=dbg)
            _same(r, o)
            assert r.bicliques == sorted(o.bicliques), dbg
    finally:
        g.free()
    rng = np.random.default_rng(78)
    for it in range(60):
        nu, nv, e = _rand_graph(rng, nmax=14)
        o = oracle.oracle_mbe(nu, nv, e, records=True)
        for dbg in (512, 512 | 128):
            r = _run(gmbe, nu, nv, e, records=True, debug=dbg)
            _same(r, o)
            assert r.bicliques == sorted(o.bicliques)
    # wide universes (pass 2 builds candidate rows through the dense table)
    for it in range(6):
        nu, nv = int(rng.integers(120, 200)), int(rng.integers(20, 40))
        e = np.argwhere(rng.random((nu, nv)) < 0.35).astype(np.uint32)
        o = oracle.oracle_mbe(nu, nv, e)
        for dbg in (512, 512 | 128):
            _same(_run(gmbe, nu, nv, e, debug=dbg), o)


def test_sort_mode_roots(gmbe, dense_case):
    """Sort-mode roots (rows built by radix-sorting the wedge keys rank << 6 | member, runs of equal
    rank OR-ed into rows; no per-warp table) forced on every small-universe full-scan root
    (debug 8192), and switched off (debug 4096): the canonical tree, sets and counters."""
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        for dbg in (8192, 8192 | 16, 4096):
            r = g.enumerate(records=True, debug=dbg)
            _same(r, o)
            assert r.bicliques == sorted(o.bicliques), dbg
        r = g.enumerate(records=True, debug=8192, bound_height=1, bound_size=1)
        _same(r, o)
    finally:
        g.free()
    rng = np.random.default_rng(79)
    for it in range(60):
        nu, nv, e = _rand_graph(rng, nmax=14)
        o = oracle.oracle_mbe(nu, nv, e, records=True)
        r = _run(gmbe, nu, nv, e, records=True, debug=8192)
        _same(r, o)
        assert r.bicliques == sorted(o.bicliques)
    # many wedges per root over a 64-bit universe, rows across the 32-bit boundary, ranks > 2^9
    for it in range(3):
        nu, nv = int(rng.integers(2500, 3500)), int(rng.integers(600, 1400))
        e = np.argwhere(rng.random((nu, nv)) < 0.015).astype(np.uint32)
        o = oracle.oracle_mbe(nu, nv, e)
        for dbg in (8192, 4096, 0):
            _same(_run(gmbe, nu, nv, e, debug=dbg), o)


# ---------------------------------------------------------------- streaming output (N2)
def _stream_all(g, **kw):
    got = []

    def sink(words, n_records):
        got.extend((tuple(sorted(l.tolist())), tuple(sorted(r.tolist()))) for l, r in gmbe_mod().iter_records(words))
    r = g.enumerate_stream(sink, **kw)
    return r, got


def gmbe_mod():
    import paper_conf_sc_panhlzwc23_b200 as m
    return m


def test_stream_sets_small_ring(gmbe, dense_case):
    """Every record streamed exactly once through a ring far smaller than the output (wrap-around
    and back-pressure), on every tier: sets equal the oracle's, count == records delivered."""
    from oracle.brute import checksum
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        for kw in (dict(), dict(debug=16), dict(debug=8), dict(debug=128 | 512), dict(thr_min=1)):
            r, got = _stream_all(g, ring_words=1, **kw)  # rounded up to the minimum ring
            assert (r.count, r.checksum) == (o.count, o.checksum), kw
            assert r.n_written == r.count == len(got), kw
            assert sorted(got) == sorted(o.bicliques), kw
            assert checksum(got) == o.checksum
    finally:
        g.free()
    for n in (8, 12):  # crown graphs: 2^n - 2 records
        nu, nv, e = crown_edges(n)
        g = gmbe.load(nu, nv, e)
        try:
            r, got = _stream_all(g, ring_words=1)
            assert r.count == len(got) == 2 ** n - 2 and len(set(got)) == len(got)
            assert checksum(got) == r.checksum
        finally:
            g.free()


def test_stream_full_config(gmbe):
    """A full-size config streamed with the default ring: delivered records reproduce the golden
    count and checksum (computed on the host from the streamed sets)."""
    from oracle.brute import checksum
    gd = _gold_cfg()["gh"]
    nu, nv, e = make_config("gh")
    g = gmbe.load(nu, nv, e)
    try:
        r, got = _stream_all(g)
        assert (r.count, r.checksum) == (gd["count"], int(gd["checksum"], 16))
        assert r.n_written == len(got) == gd["count"]
        assert checksum(got) == int(gd["checksum"], 16)
    finally:
        g.free()


def test_stream_rejects_bounded_buffers(gmbe):
    nu, nv, e = g0_edges()
    g = gmbe.load(nu, nv, e)
    try:
        with pytest.raises(ZeroDivisionError):  # a sink error propagates after the ring is drained
            g.enumerate_stream(lambda w, n: 1 / 0)
        r, got = _stream_all(g)  # the workspace stays usable
        assert r.count == 6 and len(got) == 6
    finally:
        g.free()


# ---------------------------------------------------------------- N1: shared root cursor
def test_shared_cursor_concurrent_calls(gmbe):
    """Two concurrent gmbe_enumerate calls (two replicas, two streams, two host threads) draw roots
    from one shared cursor with system-scope atomics: their results add up to the whole-graph golden
    bit-exactly, whoever wins which root.  An exhausted slot yields nothing; a reset slot everything."""
    import threading
    import torch
    gd = _gold_cfg()["gh"]
    nu, nv, e = make_config("gh")
    cur = gmbe.SharedCursor.create(0)
    gs = [gmbe.load(nu, nv, e) for _ in range(2)]
    ss = [torch.cuda.Stream() for _ in range(2)]
    try:
        for k in range(3):
            out = [None, None]

            def run(i):
                out[i] = gs[i].enumerate(root_cursor=cur.slot_ptr(k), stream=ss[i])

            th = [threading.Thread(target=run, args=(i,)) for i in range(2)]
            for t in th:
                t.start()
            for t in th:
                t.join()
            assert sum(r.count for r in out) == gd["count"]
            assert sum(r.checksum for r in out) % (1 << 64) == int(gd["checksum"], 16)
            assert sum(r.nodes for r in out) == gd["nodes"]
            assert sum(r.roots_run for r in out) == gd["roots_run"]
        r = gs[0].enumerate(root_cursor=cur.slot_ptr(0))  # slot 0 is exhausted
        assert r.count == 0 and r.roots_run == 0
        cur.reset(0)
        torch.cuda.synchronize()
        r = gs[0].enumerate(root_cursor=cur.slot_ptr(0))
        assert (r.count, r.checksum) == (gd["count"], int(gd["checksum"], 16))
        with pytest.raises(gmbe.GmbeError):
            gs[0].enumerate(root_cursor=cur.slot_ptr(1), part=(0, 2))
    finally:
        for g in gs:
            g.free()
        cur.close()


def _ipc_worker(rank, world, port, name, q):
    import torch
    import torch.distributed as dist
    import paper_conf_sc_panhlzwc23_b200 as m
    from paper_conf_sc_panhlzwc23_b200 import dist as gdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        nu, nv, e = make_config(name)
        g = m.load(nu, nv, e)
        for i in range(world):  # processes sharing one GPU size their workspaces in turn
            if rank == i:
                g.enumerate(part=(rank, world))
            dist.barrier()
        dr = gdist.DynamicRoots(rank, world, device=0)
        outs = []
        for _ in range(3):
            r, tot = dr.enumerate(g)
            outs.append((r.count, tot["count"], tot["checksum"], tot["nodes"]))
        q.put((rank, dr.dynamic, dr.error, outs))
        g.free()
        if rank:
            dr.close()
        dist.barrier()
        if not rank:
            dr.close()
    except Exception as ex:  # report instead of leaving the parent waiting on the queue
        q.put((rank, False, "%s: %s" % (type(ex).__name__, ex), []))
        raise
    finally:
        dist.destroy_process_group()


def test_dynamic_roots_two_processes_ipc(gmbe):
    """bench.py's N>1 launch shape with the N1 cursor: two processes (here both on GPU 0), rank 0's
    cursor mapped into rank 1 through CUDA IPC; three consecutive collective calls."""
    import socket
    import torch.multiprocessing as mp
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    gd = _gold_cfg()["gh"]
    g = gmbe.load(2, 2, np.array([[0, 0]], np.uint32))  # hand this process's idle workspace back
    g.release_workspace()
    g.free()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_ipc_worker, args=(r, 2, port, "gh", q)) for r in range(2)]
    for p in ps:
        p.start()
    out = sorted(q.get(timeout=300) for _ in range(2))
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    for rank, dyn, err, outs in out:
        assert dyn, err
        for mine, cnt, cks, nodes in outs:
            assert (cnt, cks, nodes) == (gd["count"], int(gd["checksum"], 16), gd["nodes"])
    for step in range(3):
        assert sum(o[3][step][0] for o in out) == gd["count"]


# ---------------------------------------------------------------- N4: cost-model (snake/LPT) parts
@pytest.mark.parametrize("n", [2, 3, 8])
def test_cost_parts_partition(gmbe, dense_case, n):
    """part_mode="cost" deals the issue list (heaviest wedge count first) out in snake order: the
    parts partition the roots -- disjoint per-root supports whose per-root counts equal the oracle's,
    and totals bit-exact."""
    nu, nv, e, o = dense_case
    op = oracle.oracle_mbe(nu, nv, e, per_root=True)
    g = gmbe.load(nu, nv, e)
    try:
        rs = [g.enumerate(part=(i, n), part_mode="cost", per_root=True) for i in range(n)]
        assert sum(r.count for r in rs) == o.count
        assert sum(r.checksum for r in rs) % (1 << 64) == o.checksum
        assert sum(r.nodes for r in rs) == o.nodes and sum(r.nonmax for r in rs) == o.nonmax
        assert sum(r.roots_run for r in rs) == o.roots_run
        acc = np.zeros_like(op.per_root_count)
        for r in rs:
            sup = r.per_root_count > 0
            assert not (acc[sup] > 0).any()  # no root in two parts
            acc += r.per_root_count
        assert (acc == op.per_root_count).all()
    finally:
        g.free()


@pytest.mark.parametrize("name,n", [("gh_work", 8), ("bx", 4)])
def test_cost_parts_full_config(gmbe, name, n):
    gd = _gold_cfg()[name]
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    try:
        rs = [g.enumerate(part=(i, n), part_mode="cost") for i in range(n)]
        assert sum(r.count for r in rs) == gd["count"]
        assert sum(r.checksum for r in rs) % (1 << 64) == int(gd["checksum"], 16)
        assert sum(r.nodes for r in rs) == gd["nodes"]
    finally:
        g.free()


def test_cost_parts_and_cursor_edge_cases(gmbe):
    """More parts than roots (empty parts), an empty graph, and a shared cursor over a graph with
    fewer roots than the callers' warps."""
    nu, nv = 5, 3
    e = np.array([[0, 0], [1, 0], [1, 1], [2, 1], [3, 2], [4, 2], [4, 0]], np.uint32)
    o = oracle.oracle_mbe(nu, nv, e)
    g = gmbe.load(nu, nv, e)
    try:
        for n in (2, 3, 4, 8):
            rs = [g.enumerate(part=(i, n), part_mode="cost") for i in range(n)]
            assert sum(r.count for r in rs) == o.count
            assert sum(r.checksum for r in rs) % (1 << 64) == o.checksum
            assert sum(1 for r in rs if r.roots_run) <= nv
        cur = gmbe.SharedCursor.create(0)
        try:
            a = g.enumerate(root_cursor=cur.slot_ptr(0))
            b = g.enumerate(root_cursor=cur.slot_ptr(0))
            assert (a.count, a.checksum) == (o.count, o.checksum) and b.count == 0
        finally:
            cur.close()
    finally:
        g.free()
    g = gmbe.load(4, 4, np.zeros((0, 2), np.uint32))
    try:
        for n in (1, 3):
            r = g.enumerate(part=(n - 1, n), part_mode="cost")
            assert (r.count, r.checksum) == (0, 0)
    finally:
        g.free()


# ---------------------------------------------------------------- stream ordering of device edges
def test_device_edges_computed_on_torch_stream(gmbe):
    """Edges produced by torch kernels (here a non-contiguous view that load() must copy, after a
    computation on torch's current stream) are read by the graph build only after that work: the
    binding builds on torch's current stream (the default stream is passed as cudaStreamLegacy)."""
    import torch
    gd = _gold_cfg()["gh"]
    nu, nv, e = make_config("gh")
    for rep in range(3):
        base = torch.zeros((len(e), 4), dtype=torch.int32, device="cuda")
        src = torch.from_numpy(e.astype(np.int32)).cuda()
        base[:, 0] = src[:, 0] * 3 + 7   # some device work the build must wait for ...
        base[:, 2] = src[:, 1] + 11
        base[:, 0] = (base[:, 0] - 7) // 3
        base[:, 2] -= 11
        t = base[:, 0::2]                  # ... and a non-contiguous view (load() copies it)
        assert not t.is_contiguous()
        g = gmbe.load(nu, nv, t)
        try:
            r = g.enumerate()
            assert (r.count, r.checksum) == (gd["count"], int(gd["checksum"], 16)), rep
        finally:
            g.free()


# ---------------------------------------------------------------- real multi-GPU (>= 2 devices)
def _multi_gpu_worker(rank, world, port, name, mode, q):
    import torch
    import torch.distributed as dist
    import paper_conf_sc_panhlzwc23_b200 as m
    from paper_conf_sc_panhlzwc23_b200 import dist as gdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dev = torch.device("cuda", rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=dev)
    try:
        nu, nv, e = make_config(name)
        g = m.load(nu, nv, torch.from_numpy(e.astype(np.int32)).to(dev), device=rank)
        outs = []
        if mode == "dynamic":
            dr = gdist.DynamicRoots(rank, world, device=rank, dev=dev)
            for _ in range(3):
                r, tot = dr.enumerate(g)
                outs.append((r.count, tot["count"], tot["checksum"], tot["nodes"]))
            q.put((rank, dr.dynamic, dr.error, outs))
            if rank:
                dr.close()
            dist.barrier()
            if not rank:
                dr.close()
        else:
            for pm in ("interleave", "cost"):
                r = g.enumerate(part=(rank, world), part_mode=pm)
                tot = gdist.allreduce_result(r, device=dev)
                outs.append((r.count, tot["count"], tot["checksum"], tot["nodes"]))
            q.put((rank, True, None, outs))
        g.free()
    except Exception as ex:
        q.put((rank, False, "%s: %s" % (type(ex).__name__, ex), []))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["dynamic", "static"])
def test_multi_gpu_distinct_devices(gmbe, mode):
    """bench.py's N>1 launch on DISTINCT devices (one process per GPU, NCCL): the N1 shared cursor in
    rank 0's HBM mapped by peers over NVLink (cudaIpcMemLazyEnablePeerAccess, atomicAdd_system
    across devices), and the static interleave / cost parts -- totals bit-exact vs the golden.
    Needs >= 2 GPUs (skipped on the one-GPU box)."""
    import socket
    import torch
    import torch.multiprocessing as mp
    n = torch.cuda.device_count()
    if n < 2:
        pytest.skip("needs >= 2 GPUs (found %d)" % n)
    world = min(n, 8)
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    gd = _gold_cfg()["gh_work"]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_multi_gpu_worker, args=(r, world, port, "gh_work", mode, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = sorted(q.get(timeout=600) for _ in range(world))
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    for rank, ok, err, outs in out:
        assert ok, err
        for mine, cnt, cks, nodes in outs:
            assert (cnt, cks, nodes) == (gd["count"], int(gd["checksum"], 16), gd["nodes"])
    for step in range(len(out[0][3])):
        assert sum(o[3][step][0] for o in out) == gd["count"]


# ---------------------------------------------------------------- N3: GMBE-WARP / GMBE-BLOCK schedulers
@pytest.mark.parametrize("sched", ["warp", "block"])
def test_scheduler_variants_small(gmbe, dense_case, sched):
    """The paper's warp-centric and block-centric schemes (Sec 4.3; the variants of Sec 6.3)
    walk the same canonical tree as GMBE: identical sets, counts, checksums and counters -- on the
    paper's G0, ER40, random tiny graphs, the dense block case (deep subtrees) with the Γ-index
    roots, suffix-mode roots (no Γ index: binary-search maximality), dense-table roots, wide
    universes (Γ columns), prune off, and output records."""
    nu, nv, e = g0_edges()
    for order in ("identity", "degree"):
        for prune in (True, False):
            r = _run(gmbe, nu, nv, e, order=order, prune=prune, records=True, scheduler=sched)
            o = oracle.oracle_mbe(nu, nv, e, order=order, prune=prune, records=True)
            _same(r, o)
            assert r.bicliques == sorted(o.bicliques)
    nu, nv, e = make_config("er40")
    r = _run(gmbe, nu, nv, e, records=True, scheduler=sched)
    o = oracle.oracle_mbe(nu, nv, e, records=True)
    _same(r, o)
    assert r.bicliques == sorted(o.bicliques)
    rng = np.random.default_rng(404)
    for _ in range(60):
        nu, nv, e = _rand_graph(rng, nmax=14)
        prune = bool(rng.random() < 0.8)
        r = _run(gmbe, nu, nv, e, prune=prune, records=True, scheduler=sched)
        o = oracle.oracle_mbe(nu, nv, e, prune=prune, records=True)
        _same(r, o)
        assert r.bicliques == sorted(o.bicliques)
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        for kw in (dict(), dict(debug=128), dict(debug=512), dict(warps_per_sm=16)):
            r = g.enumerate(records=True, scheduler=sched, **kw)
            _same(r, o)
            assert r.bicliques == sorted(o.bicliques), kw
            assert r.splits == 0 and r.tasks == 0 and r.donations == 0
        o2 = oracle.oracle_mbe(nu, nv, e, prune=False)
        _same(g.enumerate(prune=False, scheduler=sched), o2)
    finally:
        g.free()
    for it in range(6):  # wide universes: Γ columns / binary searches
        nu, nv = int(rng.integers(120, 260)), int(rng.integers(20, 45))
        e = np.argwhere(rng.random((nu, nv)) < float(rng.uniform(0.25, 0.5))).astype(np.uint32)
        o = oracle.oracle_mbe(nu, nv, e)
        for dbg in (0, 128):
            _same(_run(gmbe, nu, nv, e, debug=dbg, scheduler=sched), o)


@pytest.mark.parametrize("name", ["gh", "gh_work", "bx"])
@pytest.mark.parametrize("sched", ["warp", "block"])
def test_scheduler_variants_full_config(gmbe, name, sched):
    gd = _gold_cfg()[name]
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    try:
        r = g.enumerate(scheduler=sched)
        assert (r.count, r.checksum) == (gd["count"], int(gd["checksum"], 16))
        assert (r.nodes, r.nonmax, r.roots_run) == (gd["nodes"], gd["nonmax"], gd["roots_run"])
        assert r.algo_bytes_cand == gd["algo_bytes_cand"]
    finally:
        g.free()


# ---------------------------------------------------------------- chunked root claims
def test_root_chunk_invariance(gmbe, dense_case):
    """Warps claim root_chunk consecutive issue positions per atomic past the heavy head (local and
    N1 shared cursor): any chunk size gives the same sets and canonical-tree counters."""
    nu, nv, e, o = dense_case
    g = gmbe.load(nu, nv, e)
    try:
        for ch in (1, 2, 7, 32, 1000):
            r = g.enumerate(records=True, root_chunk=ch)
            _same(r, o)
            assert r.bicliques == sorted(o.bicliques), ch
        cur = gmbe.SharedCursor.create(0)
        try:
            for k, ch in enumerate((1, 5, 32)):
                a = g.enumerate(root_cursor=cur.slot_ptr(k), root_chunk=ch)
                b = g.enumerate(root_cursor=cur.slot_ptr(k), root_chunk=ch)  # exhausted: nothing left
                assert (a.count, a.checksum, b.count) == (o.count, o.checksum, 0)
        finally:
            cur.close()
    finally:
        g.free()
    gd = _gold_cfg()["dblp"]
    nu, nv, e = make_config("dblp")
    g = gmbe.load(nu, nv, e)
    try:
        for ch in (1, 32):
            r = g.enumerate(root_chunk=ch)
            assert (r.count, r.checksum, r.nodes) == (gd["count"], int(gd["checksum"], 16), gd["nodes"])
    finally:
        g.free()


# ---------------------------------------------------------------- arena overflow degrade path
@pytest.mark.parametrize("name", ["gh", "bx"])
def test_arena_overflow_degrade_path(gmbe, name):
    """A per-warp dynamic region far too small for the graph's root records (arena_words=4096) no
    longer fails the call: it is re-run with 4x larger regions until it fits (result.retries > 0),
    and the result is the golden's, bit-exact.  The next call with the default sizing needs no
    re-run."""
    gd = _gold_cfg()[name]
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    try:
        r = g.enumerate(arena_words=4096)
        assert r.retries > 0
        assert (r.count, r.checksum) == (gd["count"], int(gd["checksum"], 16))
        assert (r.nodes, r.nonmax, r.roots_run) == (gd["nodes"], gd["nonmax"], gd["roots_run"])
        r = g.enumerate()
        assert r.retries == 0 and (r.count, r.checksum) == (gd["count"], int(gd["checksum"], 16))
    finally:
        g.free()
