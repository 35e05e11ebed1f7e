"""Per-root device cycles of one enumeration (opts.per_root_cycles) -> where the time goes.
    python scripts/profile_roots.py gh [--top 20] [extra enumerate kwargs as k=v]"""
import json
import sys
import os
import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
# the phase-profiling build (libgmbe_prof.so, -DGMBE_PROFILE); build it with
#   python -c "import importlib.util as u; ..._build.build(profile=True)"  (see __graft_entry__)
os.environ.setdefault("GMBE_LIB", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                               "paper_conf_sc_panhlzwc23_b200", "libgmbe_prof.so"))
import torch  # noqa: E402,F401
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1]
kw = {}
top = 20
for a in sys.argv[2:]:
    k, v = a.split("=")
    if k == "top":
        top = int(v)
    else:
        kw[k] = int(v)
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
g.enumerate(**kw)
r = g.enumerate(root_cycles=True, per_root=True, phases=True, **kw)
cyc = r.per_root_cycles.astype(np.float64)
deg = np.bincount(e[:, 1].astype(np.int64), minlength=nv) if nu >= nv else np.bincount(e[:, 0].astype(np.int64), minlength=nu)
order = np.argsort(-cyc)
tot = cyc.sum()
print(json.dumps(dict(config=name, kernel_ms=r.kernel_ms, count=r.count, total_cycles=tot,
                      max_root_cycles=float(cyc.max()), ms_at_1965=float(cyc.max()) / 1.965e6,
                      top1pct_share=float(np.sort(cyc)[::-1][: max(1, len(cyc) // 100)].sum() / tot))))
tp = sum(r.phase_cycles.values()) or 1
print("phases:", {k: "%.1f%%" % (100.0 * v / tp) for k, v in r.phase_cycles.items()}, "profiled/total %.2f" % (tp / tot))
print("nodes", r.nodes, "nonmax", r.nonmax, "splits", r.splits, "tasks", r.tasks)
for v in order[:top]:
    print("root %d deg %d cycles %.3g (%.2f ms) bicliques %d" % (v, deg[v], cyc[v], cyc[v] / 1.965e6, r.per_root_count[v]))
