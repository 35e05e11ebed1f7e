"""Kernel ms of single roots run alone (part=(rank, n_roots)): the critical path of a heavy root's
tree on an otherwise idle GPU.   python scripts/roots_alone_times.py gh_work 54177 54411 ..."""
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
g.enumerate()
out = []
for rk in map(int, sys.argv[2:]):
    g.enumerate(part=(rk, nroots))
    r = g.enumerate(part=(rk, nroots))
    out.append("%d:%.2f(t%d,d%d)" % (rk, r.kernel_ms, r.tasks, r.donations))
print(" ".join(out))
