"""Active-warp / active-SM timeline of one enumeration (Fig 4 / Fig 9 analogue).
    python scripts/timeline.py gh_work [k=v ...]  -> utilisation over time, the tail, longest tasks"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1]
kw = {}
for a in sys.argv[2:]:
    k, v = a.split("=")
    kw[k] = tuple(map(int, v.split("/"))) if k == "part" else int(v)
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
g.enumerate(**kw)
r = g.enumerate(timeline=4_000_000, **kw)
t = r.timeline.astype(np.int64)
sm = (t[:, 0] >> 56) & 0xFF
kind = (t[:, 0] >> 48) & 0xFF
t0, t1 = t[:, 1], t[:, 2]
base = t0.min()
t0, t1 = (t0 - base) / 1e3, (t1 - base) / 1e3  # us
end = t1.max()
bins = np.linspace(0, end, 41)
busy = []
for a, b in zip(bins[:-1], bins[1:]):
    ov = np.clip(np.minimum(t1, b) - np.maximum(t0, a), 0, None)
    busy.append(ov.sum() / (b - a))  # average number of busy warps in the bin
dur = t1 - t0
order = np.argsort(-dur)[:10]
out = dict(config=name, kernel_ms=r.kernel_ms, records=len(t), span_us=float(end),
           busy_warps_per_bin=[round(float(x), 1) for x in busy],
           longest=[dict(kind=int(kind[i]), sm=int(sm[i]), root=int(t[i, 0] & 0xFFFFFFFFFFFF),
                         start_us=round(float(t0[i]), 1), dur_us=round(float(dur[i]), 1),
                         nodes=int(t[i, 3] >> 32), l_top=int((t[i, 3] >> 16) & 0xFFFF), c_top=int(t[i, 3] & 0xFFFF))
                    for i in order],
           last_end_by_kind={int(k): round(float(t1[kind == k].max()), 1) for k in np.unique(kind)},
           last_to_end=[dict(kind=int(kind[i]), root=int(t[i, 0] & 0xFFFFFFFFFFFF), start_us=round(float(t0[i]), 1),
                             dur_us=round(float(dur[i]), 1), nodes=int(t[i, 3] >> 32),
                             l_top=int((t[i, 3] >> 16) & 0xFFFF), c_top=int(t[i, 3] & 0xFFFF))
                        for i in np.argsort(-t1)[:8]])
print(json.dumps(out))
