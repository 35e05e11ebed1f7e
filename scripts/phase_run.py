"""Phase shares of k_enum's warp cycles (profiling build libgmbe_prof.so, GMBE_PROFILE) per config.
    GMBE_LIB=paper_conf_sc_panhlzwc23_b200/libgmbe_prof.so python scripts/phase_run.py gh_work dblp"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

for name in sys.argv[1:]:
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    g.enumerate()
    r = g.enumerate(phases=True)
    tot = sum(r.phase_cycles.values()) or 1
    print(name, "%.2f ms" % r.kernel_ms,
          {k: round(100 * v / tot, 1) for k, v in r.phase_cycles.items() if v}, flush=True)
    g.free()
