"""Sweep enumerate() options on one config; prints kernel ms per setting (GPU).
    python scripts/sweep.py gh_work "bound_height=20,bound_size=1500" "bound_height=5" ..."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

nu, nv, e = make_config(sys.argv[1])
g = gmbe.load(nu, nv, e)
g.enumerate()
for spec in sys.argv[2:]:
    kw = {}
    for a in filter(None, spec.split(",")):
        k, v = a.split("=")
        kw[k] = int(v) if v.lstrip("-").isdigit() else v
    ts = []
    for _ in range(3):
        r = g.enumerate(**kw)
        ts.append(r.kernel_ms)
    print("%-40s count %d  kernel ms %s  splits %d tasks %d donations %d" % (
        spec, r.count, " ".join("%.1f" % t for t in ts), r.splits, r.tasks, r.donations), flush=True)
