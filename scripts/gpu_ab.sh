#!/bin/bash
# A/B: current build vs named variants on the configs; then a pytest selection
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
: > gpurun_out/ab.txt
for c in ${CONFIGS:-gh_work gh dblp bx bx_work yg_work}; do
  for v in cur ${VARIANTS}; do
    if [ $v = cur ]; then L=""; else L=build_variants/libgmbe_$v.so; fi
    echo "== $c $v" >> gpurun_out/ab.txt
    GMBE_LIB=$L timeout 300 python scripts/sweep.py $c "" ${SWEEP_EXTRA} >> gpurun_out/ab.txt 2>&1
  done
done
sed 's/  splits.*//' gpurun_out/ab.txt
if [ -n "${PYTEST_K}" ]; then
timeout 1500 python -m pytest tests -m gpu -x -q --deselect tests/test_sanitizer.py -k "${PYTEST_K}" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -5 gpurun_out/pytest_gpu.log
fi
