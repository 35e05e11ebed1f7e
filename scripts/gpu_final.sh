#!/bin/bash
# GPU suite + ncu --set full of k_enum on dblp and bx (profiles breadth)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for c in dblp bx; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_enum -s 1 -c 1 -o gpurun_out/prof_$c python scripts/ncu_target.py $c > gpurun_out/ncu_$c.log 2>&1
done
tail -3 gpurun_out/pytest_gpu.log; tail -1 gpurun_out/ncu_*.log
