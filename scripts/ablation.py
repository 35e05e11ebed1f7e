"""Design-space ablations on B200 (the paper's Figs 8-11 analogues on synthetic
graphs): GMBE vs W/O_PRUNE (Thm 4.1 off), W/O_SPLIT (no load-aware splitting, Alg 4), warp-centric
search only (thread-level tier off), no dynamic donation, the (bound_height, bound_size) grid (Fig 10),
resident warps per SM (Fig 11) and the active-warp timeline (Fig 9).  Every variant is checked
against the default's count and checksum (the tree is schedule-independent, reading A9).
    python scripts/ablation.py gh_work [--out profiles/r01_ablation_gh_work.json]"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1]
out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else None
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
g.enumerate()
base = None


def run(tag, reps=3, **kw):
    global base
    ts = []
    for _ in range(reps):
        r = g.enumerate(**kw)
        ts.append(r.kernel_ms)
    if base is None:
        base = r
    assert (r.count, r.checksum) == (base.count, base.checksum), (tag, r.count, base.count)
    row = dict(variant=tag, opts=kw, kernel_ms=round(float(np.median(ts)), 3), nodes=r.nodes, nonmax=r.nonmax,
               splits=r.splits, tasks=r.tasks, donations=r.donations)
    print(json.dumps(row), flush=True)
    return row


res = dict(config=name, count=None, variants=[], grid=[], warps_per_sm=[])
res["variants"].append(run("GMBE (default)"))
res["count"] = base.count
res["variants"].append(run("W/O_PRUNE (Thm 4.1 off)", reps=1, prune=False))
res["variants"].append(run("W/O_SPLIT (no Alg 4 splitting)", reps=1, split=False))
res["variants"].append(run("warp-centric only (thread tier off)", debug=16))
res["variants"].append(run("no dynamic donation", debug=4))
res["variants"].append(run("paper thresholds (20, 1500)", bound_height=20, bound_size=1500))
for h in (4, 8, 10, 12, 16, 20):
    for sz in (200, 500, 1000, 1500):
        if sz > h * h:  # A10: bound_size > bound_height^2
            res["grid"].append(run("grid", reps=2, bound_height=h, bound_size=sz))
for w in (8, 16, 24):
    res["warps_per_sm"].append(run("warps_per_sm", reps=2, warps_per_sm=w))
r = g.enumerate(timeline=4_000_000)
t = r.timeline.astype(np.int64)
t0, t1 = t[:, 1], t[:, 2]
b0 = t0.min()
t0, t1 = (t0 - b0) / 1e3, (t1 - b0) / 1e3
edges = np.linspace(0, t1.max(), 21)
res["timeline_busy_warps"] = [round(float(np.clip(np.minimum(t1, b) - np.maximum(t0, a), 0, None).sum() / (b - a)), 1)
                              for a, b in zip(edges[:-1], edges[1:])]
res["timeline_span_us"] = float(t1.max())
if out:
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
