#!/bin/bash
# round 2: ncu --set full of k_enum on gh_work and dblp (current build), summaries + per-line tables
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
for c in ${CONFIGS:-gh_work dblp}; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_enum$" -s 1 -c 1 -o gpurun_out/r2_$c python scripts/ncu_target.py $c > gpurun_out/ncu_$c.log 2>&1
  python scripts/ncu_summary.py gpurun_out/r2_$c.ncu-rep > gpurun_out/r2_ncu_$c.txt 2>&1
  python scripts/ncu_lines.py gpurun_out/r2_$c.ncu-rep 45 > gpurun_out/r2_lines_$c.txt 2>&1
done
for c in ${CONFIGS:-gh_work dblp}; do cat gpurun_out/r2_ncu_$c.txt; head -50 gpurun_out/r2_lines_$c.txt; done
