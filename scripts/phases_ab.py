import sys, os
sys.path.insert(0, os.getcwd())
import paper_conf_sc_panhlzwc23_b200 as gmbe
from gmbe_inputs import make_config
nu, nv, e = make_config("gh_work")
g = gmbe.load(nu, nv, e)
for dbg in (0, 16):
    r = g.enumerate(debug=dbg, phases=True)
    tot = sum(r.phase_cycles.values())
    print(dbg, r.kernel_ms, {k: round(100 * v / tot, 1) for k, v in r.phase_cycles.items()})
