"""bench.py -- maximal bicliques/sec on a Github-shaped synthetic bipartite graph, 1..8 B200.

One STEP = one pass of the whole hot path (DESIGN.md a1-a8) over the workload: device graph build
from device-resident edges (gmbe_load_bipartite) + enumeration (gmbe_enumerate) of this rank's
root shard + (N > 1) the NCCL all-reduce of [count, checksum, ...].  `value` = bicliques of the
whole graph / max-over-ranks step time.  `e2e` repeats the step through the public API with the
edges in pinned HOST memory (H2D inside the timed region) and the result read back to the host.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config gh_work] [--impl reference]
    torchrun --nproc-per-node N bench.py --gpus N ...
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

DEFAULT_CONFIG = "gh_work"
METRIC = "maximal bicliques/sec (Github-shaped)"  # BASELINE.json's metric, on the default gh_work
_SHAPES = {"gh": "Github", "yg": "YouTube", "bx": "BookCrossing", "dblp": "DBLP", "er": "Erdos-Renyi"}


def _metric(config):
    for k, v in _SHAPES.items():
        if config.startswith(k):
            return "maximal bicliques/sec (%s-shaped)" % v
    return METRIC
CTRL_BYTES = 1152  # sizeof(Ctrl): written and read back by gmbe_enumerate (static_assert in gmbe_enum.cu)


def _args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default=DEFAULT_CONFIG)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget-s", type=float, default=15.0)
    ap.add_argument("--partition", default="dynamic", choices=["dynamic", "interleave", "cost"],
                    help="N>1 root distribution: shared root cursor (N1), degree-rank interleave "
                         "(SURVEY 8(e)) or cost-model snake/LPT parts (N4)")
    ap.add_argument("--static", action="store_true", help="alias of --partition interleave")
    return ap.parse_args()


def _dist():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def _gold(name):
    p = os.path.join(ROOT, "tests", "golden", "configs_oracle.json")
    try:
        with open(p) as f:
            return json.load(f).get(name)
    except OSError:
        return None


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def _ncu(name):
    """The committed ncu --set full summary of k_enum on this config (profiles/ncu_summary.json)."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(p) as f:
            return json.load(f).get(name)
    except Exception:
        return None


def _traffic(name):
    """DRAM bytes per k_enum launch from the committed ncu --set full summary, if any."""
    d = _ncu(name)
    return d.get("dram_bytes_per_launch") if d else None


def _secondary(name, peak_hbm):
    """Secondary rooflines of k_enum from the committed ncu capture: L2 bytes against the measured L2
    read peak (profiles/r02_l2_peak.json, scripts/l2peak.cu), issued warp instructions against the
    SM issue peak (148 SMs x 4 schedulers x 1 warp-instruction/clock at the capture's SM clock)."""
    d = _ncu(name)
    if not d or not d.get("kernel_ms_under_ncu"):
        return None
    out = {"source": d.get("source")}
    t = d["kernel_ms_under_ncu"] * 1e-3
    try:
        with open(os.path.join(ROOT, "profiles", "r02_l2_peak.json")) as f:
            l2 = json.load(f)["l2_read_gbs"]
        if d.get("l2_bytes_per_launch"):
            a = d["l2_bytes_per_launch"] / t / 1e9
            out["l2"] = {"achieved": a, "peak": l2, "unit": "GB/s", "frac": a / l2, "peak_kind": "measured (l2peak.cu)"}
    except Exception:
        pass
    if d.get("warp_inst_per_launch") and d.get("sm_mhz"):
        a = d["warp_inst_per_launch"] / t / 1e9
        pk = 148 * 4 * d["sm_mhz"] * 1e6 / 1e9
        out["issue"] = {"achieved": a, "peak": pk, "unit": "G warp-inst/s", "frac": a / pk,
                        "warp_execution_efficiency": d.get("warp_execution_efficiency")}
    if d.get("dram_bytes_per_launch"):
        a = d["dram_bytes_per_launch"] / t / 1e9
        out["dram"] = {"achieved": a, "peak": peak_hbm, "unit": "GB/s", "frac": a / peak_hbm}
    return out


def _profile(name):
    """The committed full oracle run of a config (scripts/oracle_full.py): totals + per-root times."""
    import numpy as np
    pj = os.path.join(ROOT, "profiles", "oracle_full_%s.json" % name)
    pz = os.path.join(ROOT, "profiles", "oracle_roots_%s.npz" % name)
    try:
        with open(pj) as f:
            meta = json.load(f)
        z = np.load(pz)
        return meta, z["ns"].astype(np.float64) * 1e-9, z["count"]
    except (OSError, KeyError, ValueError):
        return None


def _sample_mask(t, budget_s, lo=0.02, hi=2.0):
    """A FIXED root sample of about budget_s seconds of oracle time (the same in every run and in both
    bench arms): the roots whose profiled time lies in [lo, hi] s (all profiled roots up to hi when
    fewer than 1 s of work is that heavy, e.g. DBLP's tiny roots), every j-th of them in order of
    internal id, j chosen so their profiled times add up to ~budget_s."""
    import numpy as np
    mid = np.nonzero((t >= lo) & (t <= hi))[0]
    if t[mid].sum() < 1.0:
        mid = np.nonzero((t > 0) & (t <= hi))[0]
    if len(mid) == 0:
        return None
    j = max(1, int(t[mid].sum() / budget_s))
    m = np.zeros(len(t), bool)
    m[mid[::j]] = True
    return m


def _cpu_sample(name, budget_s, gold):
    """Time the oracle (as it stands, 1 thread) on a bounded, fixed root sample of the workload.

    With a committed full oracle run of the config (profiles/oracle_full_<config>.json, per-root
    times in oracle_roots_<config>.npz; scripts/oracle_full.py): the sample is fixed by that profile
    (_sample_mask), and the whole job's per-core rate is estimated as the known count over the full
    run's CPU time scaled by this host's speed on the sample (measured / profiled sample time).  The
    oracle's per-root rates are far too heavy-tailed for a small sample's count/time to stand for the
    job (on gh_work the top 100 of 55k roots hold 45% of its time).  Without a profile: root shards
    i/S of the degree-rank interleave until about budget_s of CPU time (the raw sample rate).
    Returns (value, detail dict)."""
    import numpy as np
    import oracle
    from gmbe_inputs import make_config
    nu, nv, e = make_config(name)
    prof = _profile(name)
    if prof is not None:
        meta, t, cnt = prof
        mask = _sample_mask(t, budget_s)
        if mask is not None:
            t0 = time.time()
            r = oracle.oracle_mbe(nu, nv, e, root_mask=mask, root_times=True)
            wall = time.time() - t0
            meas = float(r.per_root_ns[mask].sum()) * 1e-9
            setup = max(0.0, wall - meas)  # the oracle's own graph build (CSR, dedupe, order)
            prof_s = float(t[mask].sum())
            speed = meas / prof_s
            full_s = setup + float(t.sum()) * speed
            value = meta["count"] / full_s
            return value, {
                "sample": "%d fixed roots (profiled <= 2 s each, %.1f s of the %.0f s of root work in the "
                          "full oracle run on %s) timed in %.1f s: host speed x%.3f of the profile -> whole "
                          "job %.1f CPU-s (incl. the oracle's %.2f s graph build); raw sample rate %.0f/s" % (
                              int(mask.sum()), prof_s, float(t.sum()), meta.get("cpu_model", "?"), meas,
                              1.0 / speed, full_s, setup, r.count / max(meas, 1e-9)),
                "method": "calibrated", "full_oracle_cpu_s_profile": meta.get("cpu_s"),
                "profile_cores": meta.get("procs"), "sample_count": r.count, "sample_s": round(wall, 2)}
    if gold and gold.get("oracle_cpu_seconds"):
        shards = max(1, int(round(gold["oracle_cpu_seconds"] / budget_s)))
    else:
        shards = 1024
    count, dt, taken = 0, 0.0, 0
    while taken < shards and dt < budget_s:
        t0 = time.time()
        r = oracle.oracle_mbe(nu, nv, e, shard=(taken, shards))
        dt += time.time() - t0
        count += r.count
        taken += 1
    return count / dt, {"sample": "root shards 0..%d of %d (%d bicliques, %.1f s)" % (taken - 1, shards, count, dt),
                        "method": "raw"}


def _cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


class ClockSampler:
    def __init__(self, index):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(index), "--query-gpu=" + q,
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return None
        self.p.terminate()
        self.p.wait()
        self.f.seek(0)
        rows = [r.split(",") for r in self.f.read().strip().splitlines() if r.strip()]
        os.unlink(self.f.name)
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            try:
                sm.append(float(r[1]))
                mx = max(mx, float(r[2]))
                for n, v in zip(names, r[5:9]):
                    if v.strip() == "Active":
                        reasons.add(n)
            except (ValueError, IndexError):
                pass
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def run_reference(a):
    """Reference arm: the CPU oracle as it stands, on the host's cores, same metric and workload; each
    step times the same fixed root sample as the main arm's cpu_baseline (_cpu_sample)."""
    ws, rank, _ = _dist()
    if rank != 0:
        return
    from gmbe_inputs import make_config
    gold = _gold(a.config)
    nu, nv, e = make_config(a.config)
    per_step = min(a.cpu_budget_s, 180.0 / max(1, a.steps + min(a.warmup, 1)))  # whole run: a few minutes
    for _ in range(max(0, min(a.warmup, 1))):
        _cpu_sample(a.config, per_step, gold)
    vals, det = [], {}
    for _ in range(a.steps):
        v, det = _cpu_sample(a.config, per_step, gold)
        vals.append(v)
    v = statistics.median(vals)
    line = {"impl": "reference", "metric": _metric(a.config), "value": v, "unit": "bicliques/s",
            "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup,
            "ms_per_step": 1e3 * (gold["count"] / v if gold else 0.0), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": a.config, "n_u": nu, "n_v": nv, "m": int(len(e)),
                       "sample": det.get("sample")},
            "cpu_baseline": {"value": v, "unit": "bicliques/s", "cores": 1, "kind": "oracle",
                             "sample": "oracle single-thread, median of %d steps; %s" % (a.steps, det.get("sample")),
                             "cpu_model": _cpu_model(), "host_cores": len(os.sched_getaffinity(0)),
                             "step_values": [round(x, 1) for x in vals]},
            "e2e": {"value": v, "unit": "bicliques/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    a = _args()
    if a.impl == "reference":
        return run_reference(a)
    import numpy as np
    import torch
    import torch.distributed as dist
    import paper_conf_sc_panhlzwc23_b200 as gmbe
    from paper_conf_sc_panhlzwc23_b200 import dist as gdist
    from gmbe_inputs import make_config, graph_stats

    ws, rank, local = _dist()
    assert ws == a.gpus or ws == 1, "launch with torchrun --nproc-per-node %d" % a.gpus
    # GMBE_BENCH_SHARE_GPU=1 (tests only): every rank on GPU 0 over gloo, to exercise the N>1 code
    # path (shared cursor through CUDA IPC, collectives, the JSON line) on a one-GPU box; its numbers
    # are not multi-GPU measurements and the line says so
    share = os.environ.get("GMBE_BENCH_SHARE_GPU") == "1"
    if share:
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if ws > 1:
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    stream = torch.cuda.current_stream(dev)

    nu, nv, e = make_config(a.config)
    m = len(e)
    e_dev = torch.from_numpy(e.astype(np.int32)).to(dev)                   # resident in HBM
    # e2e leg: the edges in pinned host memory, handed to load() as a zero-copy uint32 view (the
    # H2D copy inside the timed region is a DMA from this buffer, no pageable staging copy)
    e_host = torch.from_numpy(e.astype(np.int32)).pin_memory()
    e_host_u32 = e_host.numpy().view(np.uint32)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)          # > 126 MB L2
    # N > 1: every rank draws roots from one shared cursor in rank 0's HBM, unless
    # --static or the cursor cannot be mapped (then the degree-rank interleave)
    if share and ws > 1:
        # ranks sharing one GPU size their (free-memory-capped) workspaces one after the other
        for i in range(ws):
            if rank == i:
                g = gmbe.load(nu, nv, e_dev, device=local, stream=stream)
                g.enumerate(part=(rank, ws), stream=stream)
                g.free()
            dist.barrier()
    dr = None
    if ws > 1:
        if a.static:
            a.partition = "interleave"
        dr = gdist.DynamicRoots(rank, ws, local, dev=dev) if a.partition == "dynamic" else None
        if dr is not None and not dr.dynamic:
            dr = None
    pmode = a.partition if a.partition in ("interleave", "cost") else "interleave"
    part = (rank, ws)

    host_ms = {"load": [], "enumerate": []}
    abytes_cand = []

    def step(edges, kernel_ms):
        t0 = time.perf_counter()
        g = gmbe.load(nu, nv, edges, device=local, stream=stream)
        t1 = time.perf_counter()
        if dr is not None:
            r, tot = dr.enumerate(g, stream=stream)
        else:
            r = g.enumerate(part=part, stream=stream, part_mode=pmode)
        t2 = time.perf_counter()
        g.free()
        host_ms["load"].append(1e3 * (t1 - t0))
        host_ms["enumerate"].append(1e3 * (t2 - t1))
        kernel_ms.append(r.kernel_ms)
        abytes_cand.append(r.algo_bytes_cand)
        if dr is not None:
            return tot
        # the only cross-GPU exchange: one NCCL all-reduce of the int64-viewed totals (N > 1)
        return gdist.allreduce_result(r, device=dev)

    # canonical work of this shard (static parts: identical in every schedule)
    g = gmbe.load(nu, nv, e_dev, device=local, stream=stream)
    rc = (dr.enumerate(g, stream=stream)[0] if dr is not None
          else g.enumerate(part=part, stream=stream, part_mode=pmode))
    g.free()

    kms = []
    for _ in range(a.warmup):
        step(e_dev, kms)
    torch.cuda.synchronize(dev)
    if ws > 1:
        dist.barrier()
    launches0 = gmbe.kernel_launch_count()
    clk = ClockSampler(local)
    kms = []
    dev_ms = []
    res = None
    for _ in range(a.steps):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        res = step(e_dev, kms)
        e1.record(stream)
        e1.synchronize()
        dev_ms.append(e0.elapsed_time(e1))
    torch.cuda.synchronize(dev)
    clocks = clk.stop()
    launches = gmbe.kernel_launch_count() - launches0
    # e2e: edges from pinned host memory, result back on the host, per step
    e2e_ms = []
    for _ in range(a.steps):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        g = gmbe.load(nu, nv, e_host_u32, device=local, stream=stream)
        if dr is not None:
            total_e2e = dr.enumerate(g, stream=stream)[1]["count"]
        else:
            r = g.enumerate(part=part, stream=stream, part_mode=pmode)
            total_e2e = gdist.allreduce_result(r, device=dev)["count"]
        g.free()
        e1.record(stream)
        e1.synchronize()
        e2e_ms.append(e0.elapsed_time(e1))

    t_rank = sum(dev_ms) / len(dev_ms)
    t_e2e = sum(e2e_ms) / len(e2e_ms)
    k_rank = sum(kms) / len(kms)
    ab_rank = sum(abytes_cand[-a.steps:]) / a.steps  # this rank's candidate bytes per timed launch
    tt = torch.tensor([t_rank, t_e2e], dtype=torch.float64, device=dev)
    rank_ms = [k_rank]
    if ws > 1:
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        kk = torch.zeros(ws, dtype=torch.float64, device=dev)  # per-rank kernel ms (gather by SUM)
        kk[rank] = k_rank
        dist.all_reduce(kk, op=dist.ReduceOp.SUM)
        rank_ms = [float(x) for x in kk.cpu()]
    t_step, t_e2e = float(tt[0]), float(tt[1])
    count = res["count"]
    checksum = res["checksum"]
    assert total_e2e == count

    if rank == 0:
        gold = _gold(a.config)
        parity = None
        if gold:
            parity = (count == gold["count"] and checksum == int(gold["checksum"], 16))
        peak, peak_kind = _peaks()
        # algorithmic bytes of this launch (SURVEY 8(d) definition, oracle-counted on the canonical
        # tree): the golden total, apportioned to this shard by its exactly-counted candidate bytes
        if gold and gold.get("algo_bytes") and gold.get("algo_bytes_cand"):
            abytes = gold["algo_bytes"] * (ab_rank / gold["algo_bytes_cand"])
            adef = "SURVEY 8(d) (oracle golden, filtered-Q)"
        else:
            abytes = ab_rank
            adef = "wedge + candidate terms only (no golden)"
        achieved = abytes / (k_rank * 1e-3) / 1e9 if k_rank > 0 else 0.0
        st = graph_stats(nu, nv, e)
        if ws == 1:
            par = "single GPU (one persistent kernel, device root cursor)"
        elif dr is not None:
            par = ("shared root cursor x%d (rank 0 HBM via CUDA IPC, system-scope atomics over NVLink)"
                   " + NCCL all-reduce" % ws)
        elif pmode == "cost":
            par = "root-shard x%d (cost-model snake/LPT on wedge counts) + NCCL all-reduce" % ws
        else:
            par = "root-shard x%d (degree-rank interleave) + NCCL all-reduce" % ws
        if share and ws > 1:
            par += " [TEST: all ranks share GPU 0 over gloo; not a multi-GPU measurement]"
        line = {
            "metric": _metric(a.config), "value": count / (t_step * 1e-3), "unit": "bicliques/s",
            "n_gpus": ws, "steps": a.steps, "warmup": a.warmup, "ms_per_step": t_step,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "u32", "data": "synthetic",
            "config": {"workload": a.config, "n_u": nu, "n_v": nv, "m": st["m"],
                       "delta_u": st["delta_u"], "delta_v": st["delta_v"], "seed": 0,
                       "bicliques": count, "checksum": hex(checksum), "oracle_parity": parity,
                       "parallelism": par,
                       "l2": "flushed between steps (256 MiB memset)",
                       "step": "device CSR build + enumerate (+ all-reduce)"},
            "kernel_ms": k_rank,
            "rank_kernel_ms": rank_ms,
            "imbalance": max(rank_ms) / (sum(rank_ms) / len(rank_ms)) if rank_ms and sum(rank_ms) > 0 else 1.0,
            "host_wall_ms": {k: round(sum(v[-a.steps:]) / max(1, len(v[-a.steps:])), 3) for k, v in host_ms.items()},
            "e2e": {"value": count / (t_e2e * 1e-3), "unit": "bicliques/s",
                    "h2d_bytes_per_step": int(m * 8) + CTRL_BYTES, "d2h_bytes_per_step": CTRL_BYTES},
            "gpu_launches": int(launches),
            "roofline": {"bound": "hbm", "kernel": "k_enum", "achieved": achieved, "peak": peak,
                         "peak_kind": peak_kind, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": _traffic(a.config),
                         "algo_bytes_per_launch": abytes, "algo_bytes_definition": adef,
                         "algo_bytes_cand": ab_rank,
                         # the bytes the kernel itself streams (wedge + candidate terms, counted on
                         # the device): the filtered-Q term of the survey's numerator is replaced by
                         # Γ-index tests in this kernel, so this is the stricter fraction
                         "frac_cand": (ab_rank / (k_rank * 1e-3) / 1e9) / peak if k_rank > 0 else 0.0,
                         "secondary": _secondary(a.config, peak)},
            "work": {"nodes": rc.nodes, "nonmax": rc.nonmax, "roots_run": rc.roots_run,
                     "splits": rc.splits, "tasks": rc.tasks, "donations": rc.donations},
            "clocks": clocks,
        }
        if ws == 1 and not a.no_cpu_baseline:
            v, det = _cpu_sample(a.config, a.cpu_budget_s, gold)
            line["cpu_baseline"] = {"value": v, "unit": "bicliques/s", "cores": 1, "kind": "oracle",
                                    "sample": det["sample"], "method": det["method"],
                                    "cpu_model": _cpu_model(), "host_cores": len(os.sched_getaffinity(0))}
        print(json.dumps(line), flush=True)
    if ws > 1:
        if dr is not None and rank != 0:
            dr.close()  # importers unmap first, then the owner frees
        dist.barrier()
        if dr is not None and rank == 0:
            dr.close()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
