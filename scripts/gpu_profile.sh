#!/bin/bash
# Profiling call: phase breakdown, timeline, option sweep, per-config kernel times, ncu --set full of k_enum.
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
CFG=${CFG:-gh_work}
timeout 300 python scripts/profile_roots.py $CFG top=10 > gpurun_out/prof_roots.txt 2>&1
timeout 300 python scripts/timeline.py $CFG > gpurun_out/timeline.json 2>&1
timeout 600 python scripts/sweep.py $CFG "" "warps_per_sm=16" "warps_per_sm=32" "bound_height=6,bound_size=300" "bound_height=12,bound_size=600" > gpurun_out/sweep.txt 2>&1
for c in yg gh bx dblp gh_work_small; do timeout 300 python scripts/sweep.py $c "" >> gpurun_out/configs.txt 2>&1; done
if [ "${NCU:-1}" = 1 ]; then
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_enum -s 1 -c 1 -o gpurun_out/prof python scripts/ncu_target.py $CFG > gpurun_out/ncu.log 2>&1
fi
cat gpurun_out/prof_roots.txt gpurun_out/timeline.json gpurun_out/sweep.txt gpurun_out/configs.txt; tail -3 gpurun_out/ncu.log
