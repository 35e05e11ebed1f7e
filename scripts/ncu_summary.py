"""Summarise an ncu --set full report of k_enum: key metrics, stall mix, top source lines.
    python scripts/ncu_summary.py gpurun_out/prof.ncu-rep [--json out.json] [--src N]"""
import csv
import io
import json
import subprocess
import sys

rep = sys.argv[1]
out_json = sys.argv[sys.argv.index("--json") + 1] if "--json" in sys.argv else None
nsrc = int(sys.argv[sys.argv.index("--src") + 1]) if "--src" in sys.argv else 25


def ncu(*a):
    return subprocess.run(["ncu", "-i", rep] + list(a), capture_output=True, text=True).stdout


rows = list(csv.reader(io.StringIO(ncu("--page", "raw", "--csv"))))
hdr, units, vals = rows[0], rows[1], rows[2]
m = {h: (v, u) for h, v, u in zip(hdr, vals, units)}
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "sm__cycles_active.avg", "sm__cycles_active.max", "sm__cycles_active.min",
        "smsp__thread_inst_executed_per_inst_executed.ratio", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
        "lts__t_sectors.sum", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed"]
summ = {k: m[k][0] + " " + m[k][1] for k in keys if k in m}
try:  # derived: achieved L2 and DRAM bandwidth, warp execution efficiency
    t_s = float(m["gpu__time_duration.sum"][0].replace(",", "")) * {"ms": 1e-3, "us": 1e-6, "s": 1.0}[m["gpu__time_duration.sum"][1].strip()]
    l2 = float(m["lts__t_sectors.sum"][0].replace(",", "")) * 32
    summ["derived_l2_GBps"] = round(l2 / t_s / 1e9, 1)
    mult = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0}
    dr = sum(float(m[k][0].replace(",", "")) * mult[m[k][1].strip()] for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
    summ["derived_dram_GBps"] = round(dr / t_s / 1e9, 1)
    summ["derived_warp_execution_efficiency"] = round(float(m["smsp__thread_inst_executed_per_inst_executed.ratio"][0]) / 32, 3)
    # the per-launch fields bench.py's roofline reads (profiles/ncu_summary.json)
    summ["per_launch"] = {
        "kernel_ms_under_ncu": t_s * 1e3, "dram_bytes_per_launch": int(dr), "l2_bytes_per_launch": int(l2),
        "warp_inst_per_launch": int(float(m["smsp__inst_executed.sum"][0].replace(",", ""))),
        "sm_mhz": round(float(m["sm__cycles_active.avg"][0].replace(",", "")) / t_s / 1e6, 1),
        "warp_execution_efficiency": summ["derived_warp_execution_efficiency"]}
except (KeyError, ValueError):
    pass
st = {h[len("smsp__pcsamp_warps_issue_stalled_"):]: float(v.replace(",", "") or 0) for h, (v, u) in m.items()
      if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued")}
tot = sum(st.values()) or 1
summ["stall_mix_pct"] = {k: round(100 * v / tot, 1) for k, v in sorted(st.items(), key=lambda x: -x[1]) if v / tot > 0.005}
for k, v in summ.items():
    print(k, v)
src = list(csv.reader(io.StringIO(ncu("--page", "source", "--csv", "--print-source", "cuda,sass"))))
h = src[2]
iS = h.index("Warp Stall Sampling (All Samples)")
agg, total = {}, 0
for r in src[3:]:
    if len(r) > iS and r[0] not in ("-", "") and r[2] == "-":
        try:
            n = int(r[iS].replace(",", ""))
        except ValueError:
            continue
        agg[(int(r[0]), r[1].strip())] = n
        total += n
top = sorted(agg.items(), key=lambda x: -x[1])[:nsrc]
print("top source lines by stall samples:")
for (ln, code), n in top:
    print("%5d %5.1f%%  %s" % (ln, 100.0 * n / total, code[:100]))
summ["top_lines"] = [[ln, round(100.0 * n / total, 2), code[:100]] for (ln, code), n in top]
if out_json:
    with open(out_json, "w") as f:
        json.dump(summ, f, indent=1)
