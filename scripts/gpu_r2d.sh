#!/bin/bash
# round 2: current kernel (tiny roots, bitmap dense) vs r1 + dense-ratio variants; key parity tests
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
: > gpurun_out/ab3.txt
for c in gh_work dblp gh bx bx_work yg_work; do
  for v in r1base dr128 dr512 dr2048; do
    L=build_variants/libgmbe_$v.so
    echo "== $c $v" >> gpurun_out/ab3.txt
    GMBE_LIB=$L timeout 300 python scripts/sweep.py $c "" >> gpurun_out/ab3.txt 2>&1
  done
  echo "== $c cur" >> gpurun_out/ab3.txt
  timeout 300 python scripts/sweep.py $c "" "root_chunk=1" "root_chunk=4" "debug=4" "debug=2048" "debug=1024" >> gpurun_out/ab3.txt 2>&1
done
cat gpurun_out/ab3.txt
timeout 1500 python -m pytest tests -m gpu -x -q --deselect tests/test_sanitizer.py > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -15 gpurun_out/pytest_gpu.log
