"""Streaming-output throughput: enumerate a config through gmbe_enumerate_stream
with a sink that only counts, and compare with the count-only kernel time.
    python scripts/stream_bench.py gh_work [ring_words]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_panhlzwc23_b200 as gmbe  # noqa: E402
from gmbe_inputs import make_config  # noqa: E402

name = sys.argv[1]
ring = int(sys.argv[2]) if len(sys.argv) > 2 else 0
nu, nv, e = make_config(name)
g = gmbe.load(nu, nv, e)
base = g.enumerate()
tot = {"words": 0, "records": 0, "batches": 0}


def sink(words, n):
    tot["words"] += len(words)
    tot["records"] += n
    tot["batches"] += 1


for rep in range(2):
    for k in tot:
        tot[k] = 0
    t = time.perf_counter()
    r = g.enumerate_stream(sink, ring_words=ring)
    dt = time.perf_counter() - t
assert r.count == base.count == tot["records"] and r.checksum == base.checksum
print("%s: %d bicliques, %.2f GB of records streamed in %.3f s (%.2f GB/s, %.1f M bicliques/s); "
      "count-only kernel %.2f ms; %d batches" % (name, r.count, tot["words"] * 4 / 1e9, dt,
                                                  tot["words"] * 4 / 1e9 / dt, r.count / dt / 1e6,
                                                  base.kernel_ms, tot["batches"]))
