"""Full oracle run of one config, sharded over host processes (SURVEY 8(d) "Oracle timing", N cores:
one process per core, root shard i/N each, counts and checksums summed mod 2^64), with per-root
wall times.  Writes profiles/oracle_full_<config>.json (totals, cores, CPU model, wall and CPU
seconds) and profiles/oracle_roots_<config>.npz (per-root ns and counts, internal V ids) -- the data
bench.py's stratified cpu_baseline sample is checked against.

    python scripts/oracle_full.py gh_work [--procs N]
"""
import argparse
import json
import multiprocessing as mp
import os
import platform
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def _cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return platform.processor() or "unknown"


def _work(args):
    name, i, n = args
    import oracle
    from gmbe_inputs import make_config
    nu, nv, e = make_config(name)
    t = time.time()
    c = time.process_time()
    r = oracle.oracle_mbe(nu, nv, e, shard=(i, n), per_root=True, root_times=True)
    return (i, r.count, r.checksum, r.nodes, r.nonmax, r.algo_bytes, time.time() - t,
            time.process_time() - c, r.per_root_ns, r.per_root_count)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--procs", type=int, default=len(os.sched_getaffinity(0)))
    ap.add_argument("--shards", type=int, default=0, help="root shards (default 4 x procs)")
    ap.add_argument("--outdir", default=os.path.join(ROOT, "profiles"))
    ap.add_argument("--tag", default="", help="suffix of the output names (e.g. _box)")
    a = ap.parse_args()
    import oracle
    oracle.build()
    n = a.shards or 4 * a.procs
    t0 = time.time()
    with mp.get_context("spawn").Pool(a.procs) as pool:
        rs = pool.map(_work, [(a.config, i, n) for i in range(n)], chunksize=1)
    wall = time.time() - t0
    count = sum(r[1] for r in rs)
    cks = sum(r[2] for r in rs) % (1 << 64)
    ns = sum(r[8].astype(np.uint64) for r in rs)
    cnt = sum(r[9].astype(np.uint64) for r in rs)
    out = {"config": a.config, "count": count, "checksum": hex(cks), "nodes": sum(r[3] for r in rs),
           "nonmax": sum(r[4] for r in rs), "algo_bytes": sum(r[5] for r in rs),
           "procs": a.procs, "shards": n, "wall_s": round(wall, 1),
           "cpu_s": round(sum(r[7] for r in rs), 1), "root_s": round(float(ns.sum()) * 1e-9, 1),
           "cpu_model": _cpu_model(), "host_cores": os.cpu_count(),
           "rate_per_core": count / (float(ns.sum()) * 1e-9),
           "rate_all_procs": count / wall}
    os.makedirs(a.outdir, exist_ok=True)
    with open(os.path.join(a.outdir, "oracle_full_%s%s.json" % (a.config, a.tag)), "w") as f:
        json.dump(out, f, indent=1)
    np.savez_compressed(os.path.join(a.outdir, "oracle_roots_%s%s.npz" % (a.config, a.tag)), ns=ns, count=cnt)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
