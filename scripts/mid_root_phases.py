"""Phase breakdown of the root build alone (debug 1024: no subtree) for roots sampled from a band of
issue positions (profiling build).   python scripts/mid_root_phases.py gh_work 2000 5000 [n]"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("GMBE_LIB", os.path.join(ROOT, "paper_conf_sc_panhlzwc23_b200", "libgmbe_prof.so"))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name, lo, hi = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
n = int(sys.argv[4]) if len(sys.argv) > 4 else 24
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
inf = g.info()
ue = np.unique(np.asarray(e, np.int64).reshape(-1, 2), axis=0)
ucol, vcol = (ue[:, 1], ue[:, 0]) if inf["swapped"] else (ue[:, 0], ue[:, 1])
nU, nV = (nv, nu) if inf["swapped"] else (nu, nv)
du = np.bincount(ucol, minlength=nU)
dv = np.bincount(vcol, minlength=nV)
wed = np.bincount(vcol, weights=du[ucol], minlength=nV)
rank_of = np.empty(nV, np.int64)
rank_of[np.lexsort((np.arange(nV), dv))] = np.arange(nV)
order = np.argsort(-wed, kind="stable")
pick = order[np.linspace(lo, hi - 1, n).astype(int)]
tot = {}
ms = []
g.enumerate(debug=1024)
for vid in pick:
    rk = int(rank_of[vid])
    r = g.enumerate(part=(rk, nV), phases=True, debug=1024)
    ms.append(r.kernel_ms)
    for k, v in r.phase_cycles.items():
        tot[k] = tot.get(k, 0) + v
s = sum(tot.values()) or 1
print("%s issue positions %d-%d, %d roots: |L| median %d, wedges median %d, alone %.3f ms median (kernel incl. launch)" % (
    name, lo, hi, n, np.median(dv[pick]), np.median(wed[pick]), np.median(ms)))
print("   phase cycles per root (k):", {k: round(v / n / 1e3, 1) for k, v in tot.items() if v / s > 0.01})
