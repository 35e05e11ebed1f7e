"""A/B check of an enumerate() option set against the oracle and the goldens (GPU).
    python scripts/ab_check.py debug=16 [configs...]"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config, g0_edges, crown_edges  # noqa: E402

kw = {}
for a in filter(None, sys.argv[1].split(",")):
    k, v = a.split("=")
    kw[k] = int(v)
cfgs = sys.argv[2:] or ["gh_work", "gh_work_small", "yg", "gh", "bx", "dblp"]
gold = json.load(open(os.path.join(ROOT, "tests", "golden", "configs_oracle.json")))
bad = 0


def same(r, o, tag):
    global bad
    ok = (r.count, r.checksum, r.nodes, r.nonmax, r.roots_run, r.algo_bytes_cand) == (
        o.count, o.checksum, o.nodes, o.nonmax, o.roots_run, o.algo_bytes_cand)
    if not ok:
        bad += 1
        print("MISMATCH", tag, (r.count, hex(r.checksum), r.nodes, r.nonmax, r.algo_bytes_cand),
              (o.count, hex(o.checksum), o.nodes, o.nonmax, o.algo_bytes_cand), flush=True)
    return ok


rng = np.random.default_rng(7)
t = time.time()
for it in range(200):
    nu, nv = int(rng.integers(2, 70)), int(rng.integers(2, 60))
    p = float(rng.uniform(0.05, 0.6))
    a = rng.random((nu, nv)) < p
    if it % 3 == 0:
        a[: nu // 2, : nv // 2] |= rng.random((nu // 2, nv // 2)) < 0.8
    e = np.argwhere(a).astype(np.uint32)
    o = oracle.oracle_mbe(nu, nv, e, records=True)
    g = gmbe.load(nu, nv, e)
    for extra in ({}, {"bound_height": 1, "bound_size": 1}, {"debug": 8}):
        k2 = dict(kw)
        for kk, vv in extra.items():
            k2[kk] = k2.get(kk, 0) | vv if kk == "debug" else vv
        r = g.enumerate(records=True, **k2)
        if same(r, o, ("rand", it, extra)) and not r.truncated and r.bicliques != sorted(o.bicliques):
            bad += 1
            print("SET MISMATCH", it, extra, "n_written", r.n_written, "truncated", r.truncated, "count", r.count)
            if bad < 3:
                sg, so = set(r.bicliques), set(o.bicliques)
                print("  gpu-only", sorted(sg - so)[:5], "\n  oracle-only", sorted(so - sg)[:5],
                      "\n  dup", len(r.bicliques) - len(sg))
    g.free()
print("random small: %d bad (%.1fs)" % (bad, time.time() - t), flush=True)
for name in cfgs:
    gd = gold[name]
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    g.enumerate()
    for tag, k2 in (("base", {}), ("opt", kw)):
        ts = []
        for _ in range(3):
            r = g.enumerate(**k2)
            ts.append(r.kernel_ms)
        ok = (r.count, r.checksum, r.nodes, r.nonmax) == (gd["count"], int(gd["checksum"], 16), gd["nodes"], gd["nonmax"])
        bad += not ok
        print("%-14s %-5s %s ms %s  donations %d tasks %d" % (name, tag, " ".join("%.2f" % x for x in ts),
              "ok" if ok else "MISMATCH", r.donations, r.tasks), flush=True)
    r = g.enumerate(debug=kw.get("debug", 0) | 32, phases=True)
    ph = list(r.phase_cycles.values())
    print("   path stats: thr jobs %d nodes %d | reg jobs %d nodes %d (total nodes %d)" % (ph[0], ph[1], ph[2], ph[3], r.nodes))
    g.free()
print("TOTAL BAD", bad)
