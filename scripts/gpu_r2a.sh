#!/bin/bash
# round 2, first GPU pass: suite, path statistics, A/B against the round-1 kernel, host CPU info
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
nproc > gpurun_out/host.txt; grep -m1 "model name" /proc/cpuinfo >> gpurun_out/host.txt; python -c "import os; print(len(os.sched_getaffinity(0)))" >> gpurun_out/host.txt
nvidia-smi -L >> gpurun_out/host.txt
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
GMBE_LIB=build_variants/libgmbe_stats.so timeout 600 python scripts/stats_run.py gh_work gh yg_work bx bx_work dblp > gpurun_out/stats.txt 2>&1
: > gpurun_out/ab.txt
for c in gh_work bx dblp yg_work; do
  for v in r1base cur; do
    if [ $v = cur ]; then L=""; else L=build_variants/libgmbe_$v.so; fi
    echo "== $c $v" >> gpurun_out/ab.txt
    GMBE_LIB=$L timeout 300 python scripts/sweep.py $c "" "" >> gpurun_out/ab.txt 2>&1
  done
done
tail -5 gpurun_out/pytest_gpu.log; cat gpurun_out/stats.txt gpurun_out/ab.txt gpurun_out/host.txt
