"""Minimal ncu target: build the graph, one warm-up enumeration, one profiled enumeration.
    ncu --set full -k regex:k_enum -s 1 -c 1 python scripts/ncu_target.py gh_work [debug=1024 ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "gh_work"
kw = {k: int(v) for k, v in (a.split("=") for a in sys.argv[2:])}
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
for _ in range(2):
    r = g.enumerate(**kw)
print(name, r.count, hex(r.checksum), "%.2f ms" % r.kernel_ms)
