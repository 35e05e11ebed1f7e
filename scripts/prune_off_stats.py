"""Why W/O_PRUNE is so much slower than its node count suggests: the tier mix with and without
Thm 4.1 (GMBE_STATS build: jobs / nodes per tier, warp-level nodes by maximality path).
    GMBE_LIB=build_variants/libgmbe_stats.so python scripts/prune_off_stats.py gh"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

for name in sys.argv[1:]:
    nu, nv, e = make_config(name)
    g = gmbe.load(nu, nv, e)
    for prune in (True, False):
        r = g.enumerate(prune=prune, debug=32, phases=True)
        ph = list(r.phase_cycles.values())
        warp_nodes = r.nodes - ph[1] - ph[3]
        print("%s prune=%s: %.2f ms nodes %d | thread tier %d jobs %d nodes | register tier %d jobs %d nodes | "
              "warp-level nodes %d (%.1f%%)" % (name, prune, r.kernel_ms, r.nodes, ph[0], ph[1], ph[2], ph[3],
                                                warp_nodes, 100.0 * warp_nodes / max(1, r.nodes)), flush=True)
    g.free()
