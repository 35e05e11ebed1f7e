"""Tier statistics of one root run alone (or the full graph): jobs / nodes per tier and why jobs stayed
on the register tier (GMBE_STATS_WHY build).   python scripts/stats_part.py gh_work [rank ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1]
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
inf = g.info()
nroots = inf["n_u"] if inf["swapped"] else inf["n_v"]
for rk in ([None] + [int(a) for a in sys.argv[2:]]):
    part = (0, 1) if rk is None else (rk, nroots)
    r = g.enumerate(debug=32, phases=True, part=part)
    ph = list(r.phase_cycles.values())
    print("%s %s: %.2f ms nodes %d thr_jobs %d thr_nodes %d reg_jobs %d reg_nodes %d | reg nodes: split-top %d no-gx %d "
          "below-thr_min %d declined %d" % (name, "all" if rk is None else rk, r.kernel_ms, r.nodes, ph[0], ph[1], ph[2],
                                             ph[3], ph[12], ph[13], ph[14], ph[15]), flush=True)
