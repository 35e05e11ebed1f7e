"""Where root construction time goes: per-root device cycles with subtrees off (debug 1024: roots
only) and on, bucketed by the root's wedge count (the issue order).
    python scripts/root_cost_buckets.py gh_work dblp ..."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

for name in sys.argv[1:]:
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    inf = g.info()
    ue = np.unique(np.asarray(e, np.int64).reshape(-1, 2), axis=0)
    ucol, vcol = (ue[:, 1], ue[:, 0]) if inf["swapped"] else (ue[:, 0], ue[:, 1])
    nU, nV = (nv, nu) if inf["swapped"] else (nu, nv)
    du = np.bincount(ucol, minlength=nU)
    wed = np.bincount(vcol, weights=du[ucol], minlength=nV)
    order = np.argsort(-wed, kind="stable")
    g.enumerate(debug=1024)
    ro = g.enumerate(debug=1024, root_cycles=True)
    fu = g.enumerate(root_cycles=True)
    c_ro = ro.per_root_cycles.astype(np.float64)[order]
    c_fu = fu.per_root_cycles.astype(np.float64)[order]
    print("%s: roots-only kernel %.2f ms, full %.2f ms; root cycles %.2f G (roots only), %.2f G (full, incl. "
          "subtrees walked by the root's warp)" % (name, ro.kernel_ms, fu.kernel_ms, c_ro.sum() / 1e9, c_fu.sum() / 1e9))
    for k in (10, 100, 1000, 10000, 100000):
        if k > len(order):
            break
        print("   top %6d roots (wedges >= %8d): %5.1f%% of root-build cycles, %5.1f%% of full per-root cycles" % (
            k, wed[order[k - 1]], 100 * c_ro[:k].sum() / c_ro.sum(), 100 * c_fu[:k].sum() / c_fu.sum()))
    sys.stdout.flush()
