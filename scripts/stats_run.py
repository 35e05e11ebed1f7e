"""Thread-tier path statistics (GMBE_STATS build, debug bit 32) per config: jobs / nodes per tier
and mean |L|, |L'|, |later| per thread-tier node.  GMBE_LIB=build_variants/libgmbe_stats.so."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

for name in sys.argv[1:]:
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    r = g.enumerate(debug=32, phases=True)
    ph = list(r.phase_cycles.values())
    n = max(1, ph[1])
    print("%s: nodes %d thr_jobs %d thr_nodes %d reg_jobs %d reg_nodes %d | gen_child lc1 %d cols %d gis %d | "
          "thr mean |L| %.2f |L'| %.2f |later| %.2f push %.3f" % (
              name, r.nodes, ph[0], ph[1], ph[2], ph[3], ph[4], ph[5], ph[6],
              ph[8] / n, ph[9] / n, ph[10] / n, ph[11] / n), flush=True)
    g.free()
