"""Target of the compute-sanitizer tests (tests/test_sanitizer.py): small graphs through every
kernel path -- graph build, the three root modes, warp / thread / register tiers, forced splits and
donation, streaming output, GMBE-WARP / GMBE-BLOCK -- each result checked against the oracle."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402  (test infrastructure: the expected values)
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import crown_edges, g0_edges, make_config  # noqa: E402


def dense_case():
    rng = np.random.default_rng(2024)
    nu, nv = 90, 60
    a = rng.random((nu, nv)) < 0.12
    a[:24, :20] |= rng.random((24, 20)) < 0.75
    return nu, nv, np.argwhere(a).astype(np.uint32)


def wide_case():
    rng = np.random.default_rng(7)
    nu, nv = 160, 30
    return nu, nv, np.argwhere(rng.random((nu, nv)) < 0.35).astype(np.uint32)


CASES = {"g0": g0_edges(), "er40": make_config("er40"), "crown12": crown_edges(12),
         "dense": dense_case(), "wide": wide_case()}
VARIANTS = [dict(), dict(bound_height=1, bound_size=1), dict(debug=8), dict(thr_min=1),
            dict(thr_min=1, debug=8), dict(debug=128), dict(debug=512), dict(debug=16),
            dict(split_wide=1), dict(scheduler="warp"), dict(scheduler="block"),
            dict(scheduler="block", debug=128)]

fails = 0
for name, (nu, nv, e) in CASES.items():
    o = oracle.oracle_mbe(nu, nv, e)
    g = gmbe.load(nu, nv, e)
    for kw in VARIANTS:
        r = g.enumerate(**kw)
        ok = (r.count, r.checksum, r.nodes, r.nonmax) == (o.count, o.checksum, o.nodes, o.nonmax)
        fails += not ok
        print(name, kw, "ok" if ok else "MISMATCH", flush=True)
    got = []
    r = g.enumerate_stream(lambda w, n: got.extend(gmbe.iter_records(w)), ring_words=1)
    ok = r.count == o.count and len(got) == o.count
    fails += not ok
    print(name, "stream", "ok" if ok else "MISMATCH", flush=True)
    g.free()
print("SANITIZE TARGET", "FAILED %d" % fails if fails else "PASSED")
sys.exit(1 if fails else 0)
