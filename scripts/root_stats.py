"""Tier statistics of single roots (non-profiling build, debug bit 32): thread-tier jobs / nodes vs
warp-tier jobs / nodes, and the time of the root alone.
    python scripts/root_stats.py gh_work 55430 ..."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1]
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
inf = g.info()
nroots = inf["n_u"] if inf["swapped"] else inf["n_v"]
g.enumerate()
for rk in map(int, sys.argv[2:]):
    for extra in ({}, {"debug": 16}):
        d = extra.get("debug", 0) | 32
        r = g.enumerate(part=(rk, nroots), phases=True, debug=d)
        r = g.enumerate(part=(rk, nroots), phases=True, debug=d)
        ph = list(r.phase_cycles.values())
        print("rank %d %s: %.2f ms count %d nodes %d splits %d tasks %d | thr jobs %d nodes %d | reg jobs %d nodes %d"
              " | wide gamma: deg %d cols %d bsearch %d" % (
            rk, extra, r.kernel_ms, r.count, r.nodes, r.splits, r.tasks, ph[0], ph[1], ph[2], ph[3], ph[4], ph[5], ph[6]),
              flush=True)
