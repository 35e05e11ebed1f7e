"""Cost of the N1 shared root cursor (system-scope atomics) against the local cursor, one process:
kernel ms for local / shared x root_chunk in {1, 16}.
    python scripts/cursor_cost.py dblp gh_work"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

out = {}
for name in sys.argv[1:]:
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    cur = gmbe.SharedCursor.create(0)
    res = {}
    k = 0
    for mode in ("local", "shared"):
        for ch in (1, 16):
            ts = []
            for rep in range(4):
                if mode == "local":
                    r = g.enumerate(root_chunk=ch)
                else:
                    cur.reset(k)
                    r = g.enumerate(root_cursor=cur.slot_ptr(k), root_chunk=ch)
                    k += 1
                ts.append(r.kernel_ms)
            res["%s_chunk%d" % (mode, ch)] = round(min(ts[1:]), 3)
    cur.close()
    g.free()
    out[name] = res
    print(name, res, flush=True)
print(json.dumps(out))
