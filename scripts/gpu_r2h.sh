#!/bin/bash
# round 2: compute-sanitizer suite (logs to gpurun_out) while the full oracle runs on the host cores
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
N=$(python -c "import os; print(max(1, len(os.sched_getaffinity(0)) - 1))")
(python scripts/oracle_full.py gh_work --procs $N --outdir gpurun_out --tag _box > gpurun_out/oracle_full_gh_work_box.log 2>&1) &
OP=$!
GMBE_SANITIZER_LOG_DIR=gpurun_out timeout 3000 python -m pytest tests/test_sanitizer.py -q > gpurun_out/pytest_sanitizer.log 2>&1; echo "sanitizer rc=$?" >> gpurun_out/pytest_sanitizer.log
wait $OP
tail -3 gpurun_out/pytest_sanitizer.log; grep -h "SUMMARY" gpurun_out/r02_sanitizer_*.log; cat gpurun_out/oracle_full_gh_work_box.log | cut -c1-400
