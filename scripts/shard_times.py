"""Projected multi-GPU balance: time each root shard part=(i, N) of a config on one GPU.
    python scripts/shard_times.py gh_work 2 4 8 [mode=cost]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1]
kw = dict(a.split("=") for a in sys.argv[2:] if "=" in a)
mode = kw.pop("mode", "interleave")
kw = {k: int(v) for k, v in kw.items()}
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
full = g.enumerate(**kw)
full = g.enumerate(**kw)
out = {"config": name, "mode": mode, "opts": kw, "n1_ms": full.kernel_ms, "count": full.count}
for n in [int(a) for a in sys.argv[2:] if "=" not in a]:
    ts, cnt = [], 0
    for i in range(n):
        g.enumerate(part=(i, n), part_mode=mode, **kw)
        r = g.enumerate(part=(i, n), part_mode=mode, **kw)
        ts.append(r.kernel_ms)
        cnt += r.count
    assert cnt == full.count
    out["n%d" % n] = {"part_ms": [round(t, 3) for t in ts], "max_ms": max(ts), "mean_ms": sum(ts) / n,
                      "imbalance": max(ts) / (sum(ts) / n), "projected_speedup": full.kernel_ms / max(ts)}
print(json.dumps(out))
