"""Absolute SM-cycle totals per phase (profiling build) for a full run and one shard.
    python scripts/phase_totals.py gh_work 4/8"""
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
g.enumerate()
runs = [("full", (0, 1))] + [(a, tuple(map(int, a.split("/")))) for a in sys.argv[2:]]
for tag, part in runs:
    r = g.enumerate(part=part, phases=True)
    r = g.enumerate(part=part, phases=True)
    n = part[1]
    print("%-6s kernel %.2f ms  nodes %d tasks %d donations %d" % (tag, r.kernel_ms, r.nodes, r.tasks, r.donations))
    print("   Gcycles x parts:", {k: round(v * n / 1e9, 2) for k, v in r.phase_cycles.items() if v})
