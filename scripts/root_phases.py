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
cyc = r.per_root_cycles.astype(np.float64)  # indexed by caller id on the library's V side
print(name, "kernel %.2f ms" % r.kernel_ms)
# degree rank of each id (ascending (deg, id), the library's order): part=(rk, n) selects by rank
ue = np.unique(np.asarray(e, np.int64).reshape(-1, 2), axis=0)
vcol = ue[:, 0] if inf["swapped"] else ue[:, 1]
deg = np.bincount(vcol, minlength=nroots)
rank_of = np.empty(nroots, np.int64)
rank_of[np.lexsort((np.arange(nroots), deg))] = np.arange(nroots)
for vid in np.argsort(-cyc)[:n]:
    rk = rank_of[vid]
    rr = g.enumerate(part=(int(rk), nroots), phases=True)
    rr = g.enumerate(part=(int(rk), nroots), phases=True)
    tot = sum(rr.phase_cycles.values()) or 1
    ph = {k: round(100.0 * v / tot, 1) for k, v in rr.phase_cycles.items() if v / tot > 0.01}
    print("id %d rank %d deg %d: %.2f ms (in full run, summed over warps %.2f ms) count %d nodes %d nonmax %d splits %d tasks %d | %s" % (
        vid, rk, deg[vid], rr.kernel_ms, cyc[vid] / 1.965e6, rr.count, rr.nodes, rr.nonmax, rr.splits, rr.tasks, ph), flush=True)
