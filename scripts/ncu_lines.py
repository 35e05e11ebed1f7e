"""Per-source-line totals of an ncu --set full capture (--import-source on): warp instructions
executed, thread instructions, stall samples, local-memory traffic.
    python scripts/ncu_lines.py report.ncu-rep [top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = None
lines = []
fname = ""
for r in rows:
    if r and r[0] == "File Path":
        fname = r[1].split("/")[-1]
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or not r or not r[0] or not r[0].isdigit():
        continue
    d = dict(zip(hdr[4:], r[4:]))
    try:
        wi = int(d.get("Instructions Executed", "0") or 0)
        ti = int(d.get("Thread Instructions Executed", "0") or 0)
        ss = int(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
        loc = int(d.get("L2 Theoretical Sectors Local", "0") or 0)
    except ValueError:
        continue
    lines.append((fname, int(r[0]), r[1].strip()[:90], wi, ti, ss, loc))
tw = sum(x[3] for x in lines) or 1
tt = sum(x[4] for x in lines) or 1
ts = sum(x[5] for x in lines) or 1
print("total warp inst %.3fG  thread inst %.3fG  stall samples %d  local sectors %d" % (
    tw / 1e9, tt / 1e9, ts, sum(x[6] for x in lines)))
print("-- by warp instructions")
for f, ln, src, wi, ti, ss, loc in sorted(lines, key=lambda x: -x[3])[:top]:
    print("%s:%-5d %5.1f%% inst %5.1f%% stall  thr/inst %4.1f  loc %8d  %s" % (
        f, ln, 100 * wi / tw, 100 * ss / ts, ti / max(wi, 1), loc, src))
print("-- by local-memory L2 sectors")
tl = sum(x[6] for x in lines) or 1
for f, ln, src, wi, ti, ss, loc in sorted(lines, key=lambda x: -x[6])[:top]:
    if loc == 0:
        break
    print("%s:%-5d %5.1f%% local  %5.1f%% inst  %s" % (f, ln, 100 * loc / tl, 100 * wi / tw, src))
