"""Try planted-block parameters for a work-shaped config and print the biclique counts (GPU).
    python scripts/calibrate.py gh "K,amin,amax,p_in" ..."""
import sys
import os
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config, graph_stats  # noqa: E402

shape = sys.argv[1]
for spec in sys.argv[2:]:
    K, amin, amax, p = spec.split(",")
    cfg = dict(kind="work", shape=shape, seed=0, K=int(K), amin=int(amin), amax=int(amax), p_in=float(p))
    t = time.time()
    nu, nv, e = make_config(cfg)
    tg = time.time() - t
    g = gmbe.load(nu, nv, e)
    r = g.enumerate()
    r = g.enumerate()
    g.free()
    st = graph_stats(nu, nv, e)
    print(spec, "count %d nodes %d nonmax %d kernel %.1f ms gen %.1fs dU %d dV %d" % (
        r.count, r.nodes, r.nonmax, r.kernel_ms, tg, st["delta_u"], st["delta_v"]), flush=True)
