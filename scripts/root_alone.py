"""Run single roots alone (part=(rank, n_roots)): time, counters, phase breakdown (profiling build).
    python scripts/root_alone.py bx 105260 105264 ..."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("GMBE_LIB", os.path.join(ROOT, "paper_conf_sc_panhlzwc23_b200", "libgmbe_prof.so"))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1]
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
inf = g.info()
nroots = inf["n_u"] if inf["swapped"] else inf["n_v"]
g.enumerate()
for rk in map(int, sys.argv[2:]):
    for extra in ({}, {"split": False}):
        rr = g.enumerate(part=(rk, nroots), phases=True, **extra)
        rr = g.enumerate(part=(rk, nroots), phases=True, **extra)
        tot = sum(rr.phase_cycles.values()) or 1
        ph = {k: round(100.0 * v / tot, 1) for k, v in rr.phase_cycles.items() if v / tot > 0.01}
        print("rank %d %s: %.2f ms count %d nodes %d nonmax %d splits %d tasks %d | %s" % (
            rk, extra, rr.kernel_ms, rr.count, rr.nodes, rr.nonmax, rr.splits, rr.tasks, ph), flush=True)
