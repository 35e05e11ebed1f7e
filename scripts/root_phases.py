"""Phase breakdown of single heavy roots (profiling build): part=(rank, n_v) runs exactly one root.
    python scripts/root_phases.py bx [n_roots]   -> the n heaviest roots by per-root cycles"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("GMBE_LIB", os.path.join(ROOT, "paper_conf_sc_panhlzwc23_b200", "libgmbe_prof.so"))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 5
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
inf = g.info()
nroots = inf["n_u"] if inf["swapped"] else inf["n_v"]
g.enumerate()
r = g.enumerate(root_cycles=True)
cyc = r.per_root_cycles.astype(np.float64)
print(name, "kernel %.2f ms" % r.kernel_ms)
for rk in np.argsort(-cyc)[:n]:
    rr = g.enumerate(part=(int(rk), nroots), phases=True)
    rr = g.enumerate(part=(int(rk), nroots), phases=True)
    tot = sum(rr.phase_cycles.values()) or 1
    ph = {k: round(100.0 * v / tot, 1) for k, v in rr.phase_cycles.items() if v / tot > 0.01}
    print("rank %d: %.2f ms (in full run %.2f ms) count %d nodes %d nonmax %d splits %d tasks %d | %s" % (
        rk, rr.kernel_ms, cyc[rk] / 1.965e6, rr.count, rr.nodes, rr.nonmax, rr.splits, rr.tasks, ph), flush=True)
