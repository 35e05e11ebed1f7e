"""Copy a gpu_evidence2.sh run (gpurun_out/ev_*) into profiles/ (r02_* names) and refresh
profiles/ncu_summary.json, which bench.py reads for the roofline's traffic / secondary fractions."""
import json
import os
import shutil

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
G, PR = os.path.join(ROOT, "gpurun_out"), os.path.join(ROOT, "profiles")
summ = json.load(open(os.path.join(PR, "ncu_summary.json")))
mult = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0}
for c in ["gh_work", "dblp", "bx"]:
    f = os.path.join(G, "ev_ncu_%s.json" % c)
    if not os.path.exists(f):
        continue
    d = json.load(open(f))
    e = dict(d["per_launch"])
    for k, key in (("dram_read_bytes", "dram__bytes_read.sum"), ("dram_write_bytes", "dram__bytes_write.sum")):
        v, u = d[key].split()
        e[k] = int(float(v.replace(",", "")) * mult[u])
    e["lts_hit_rate_pct"] = float(d["lts__t_sector_hit_rate.pct"].split()[0])
    e["source"] = ("profiles/r02_ncu_full_k_enum_%s.json (ncu --set full --clock-control none, k_enum, "
                   "scripts/ncu_target.py %s, 2nd launch; round-2 session-2 kernel)" % (c, c))
    summ[c] = e
    shutil.copy(f, os.path.join(PR, "r02_ncu_full_k_enum_%s.json" % c))
    shutil.copy(os.path.join(G, "ev_ncu_%s.txt" % c), os.path.join(PR, "r02_ncu_full_k_enum_%s.txt" % c))
json.dump(summ, open(os.path.join(PR, "ncu_summary.json"), "w"), indent=1)
for c in ["gh_work", "dblp", "bx", "bx_work", "yg_work", "gh", "yg"]:
    shutil.copy(os.path.join(G, "ev_bench_%s.json" % c), os.path.join(PR, "r02_bench_%s.json" % c))
shutil.copy(os.path.join(G, "ev_bench_ref_gh_work.json"), os.path.join(PR, "r02_bench_ref_gh_work.json"))
for f in ("ev_launches_gh_work.csv", "ev_launches_gh_work.txt"):
    shutil.copy(os.path.join(G, f), os.path.join(PR, f.replace("ev_", "r02_")))
for c in ["gh_work", "bx_work", "dblp"]:
    shutil.copy(os.path.join(G, "ev_shards_%s.json" % c), os.path.join(PR, "r02_shards_%s.json" % c))
for c in ["gh_work", "dblp", "bx", "bx_work", "yg_work", "gh", "yg"]:
    d = json.loads(open(os.path.join(PR, "r02_bench_%s.json" % c)).read().strip().splitlines()[-1])
    print("%-8s value %.4g  step %.2f ms  k_enum %.2f ms  e2e step %.2f ms  frac %.3f  parity %s" % (
        c, d["value"], d["ms_per_step"], d["kernel_ms"], d["config"]["bicliques"] / d["e2e"]["value"] * 1e3,
        d["roofline"]["frac"], d["config"].get("oracle_parity")))
for c in ["gh_work", "bx_work", "dblp"]:
    d = json.loads(open(os.path.join(PR, "r02_shards_%s.json" % c)).read().strip().splitlines()[-1])
    print(c, "n1 %.2f" % d["n1_ms"], " ".join("x%s %.2f ms (%.2fx)" % (k[1:], d[k]["max_ms"], d[k]["projected_speedup"]) for k in ("n2", "n4", "n8")))
