#!/bin/bash
# round 2: witness cache / dense ratio A/B (chunk 1 default)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
: > gpurun_out/ab4.txt
for c in gh_work gh dblp bx bx_work yg_work; do
  for v in cur nowc dr128 dr512 dr2048; do
    if [ $v = cur ]; then L=""; else L=build_variants/libgmbe_$v.so; fi
    echo "== $c $v" >> gpurun_out/ab4.txt
    GMBE_LIB=$L timeout 300 python scripts/sweep.py $c "" "debug=1024" >> gpurun_out/ab4.txt 2>&1
  done
done
cat gpurun_out/ab4.txt | sed 's/  splits.*//'
timeout 1500 python -m pytest tests -m gpu -x -q --deselect tests/test_sanitizer.py -k "thread_tier or donation or full_config_vs or scheduler or stream or suffix or dense or wide or chunk" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -5 gpurun_out/pytest_gpu.log
