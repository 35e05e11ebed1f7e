"""Active-SM timelines of the three schedulers -- the paper's Fig 9 on synthetic graphs:
GMBE (load-aware task-centric, Alg 4), GMBE-WARP (one warp per Alg 3 task) and GMBE-BLOCK (one block
per task).  Per scheduler: kernel ms, and over 50 time bins of its own span the number of SMs with a
running root / task record and the average number of busy warps (or blocks).
    python scripts/fig9_sched.py bx_work [--out profiles/r02_fig9_bx_work.json]"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1]
out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else None
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
res = {"config": name}
ref = None
for sched in ("task", "warp", "block"):
    g.enumerate(scheduler=sched)
    r = g.enumerate(scheduler=sched, timeline=2_000_000)
    if ref is None:
        ref = (r.count, r.checksum)
    assert (r.count, r.checksum) == ref, sched
    t = r.timeline.astype(np.int64)
    sm = (t[:, 0] >> 56) & 0xFF
    t0, t1 = t[:, 1], t[:, 2]
    base = t0.min()
    t0, t1 = (t0 - base) / 1e3, (t1 - base) / 1e3
    span = float(t1.max())
    bins = np.linspace(0, span, 51)
    act_sm, busy = [], []
    for a, b in zip(bins[:-1], bins[1:]):
        ov = (t1 > a) & (t0 < b)
        act_sm.append(int(len(np.unique(sm[ov]))))
        busy.append(round(float(np.clip(np.minimum(t1, b) - np.maximum(t0, a), 0, None).sum() / (b - a)), 1))
    # time until the number of active SMs first drops below 90% / 50% of the SM count
    nsm = max(act_sm)
    def first_below(f):
        for k, x in enumerate(act_sm):
            if x < f * nsm:
                return round(k / 50, 2)
        return 1.0
    res[sched] = {"kernel_ms": round(r.kernel_ms, 3), "records": int(len(t)), "span_us": round(span, 1),
                  "active_sms": act_sm, "busy_units": busy,
                  "frac_time_all_sms_busy": first_below(0.9), "frac_time_half_sms_busy": first_below(0.5)}
    print(sched, "%.2f ms" % r.kernel_ms, "active SMs", act_sm[::5], flush=True)
g.free()
if out:
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
print(json.dumps({k: (v if not isinstance(v, dict) else {kk: vv for kk, vv in v.items() if kk in ("kernel_ms", "frac_time_all_sms_busy", "frac_time_half_sms_busy")}) for k, v in res.items()}))
