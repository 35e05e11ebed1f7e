"""Write tests/golden/configs_oracle.json: oracle results (count, checksum, canonical-tree counters)
for the named full-size configs.  Calls ONLY oracle/ (and the input generators); the roots are
sharded across host cores (shards partition the output, SURVEY 8(c) ownership invariant).

    python scripts/make_golden.py gh yg dblp [--procs 8]
"""
import argparse
import json
import os
import sys
import time
from multiprocessing import Pool

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from gmbe_inputs import make_config, graph_stats  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "configs_oracle.json")
_G = {}


def _shard(args):
    name, i, n = args
    if name not in _G:
        _G[name] = make_config(name)
    nu, nv, e = _G[name]
    t = time.time()
    r = oracle.oracle_mbe(nu, nv, e, shard=(i, n))
    return r, time.time() - t


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("names", nargs="+")
    ap.add_argument("--procs", type=int, default=os.cpu_count())
    ap.add_argument("--shards", type=int, default=0)
    a = ap.parse_args()
    oracle.build()
    gold = json.load(open(OUT)) if os.path.exists(OUT) else {}
    for name in a.names:
        n = a.shards or a.procs * 4
        t0 = time.time()
        with Pool(a.procs) as pool:
            parts = pool.map(_shard, [(name, i, n) for i in range(n)])
        nu, nv, e = make_config(name)
        st = graph_stats(nu, nv, e)
        tot = dict(count=0, checksum=0, roots_run=0, nodes=0, nonmax=0, algo_bytes=0, algo_bytes_qfull=0,
                   algo_bytes_cand=0)
        for r, _ in parts:
            for k in tot:
                tot[k] += getattr(r, k)
        tot["checksum"] = hex(tot["checksum"] % (1 << 64))
        tot["stats"] = st
        tot["oracle_cpu_seconds"] = round(sum(t for _, t in parts), 1)
        tot["oracle_wall_seconds"] = round(time.time() - t0, 1)
        tot["procs"] = a.procs
        gold[name] = tot
        print(name, tot, flush=True)
        with open(OUT, "w") as f:
            json.dump(gold, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
