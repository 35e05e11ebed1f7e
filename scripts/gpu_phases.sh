#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
: > gpurun_out/phases.txt
for c in ${CONFIGS:-dblp gh yg}; do
  echo "== $c" >> gpurun_out/phases.txt
  timeout 300 python scripts/profile_roots.py $c top=5 >> gpurun_out/phases.txt 2>&1
  timeout 300 python scripts/timeline.py $c >> gpurun_out/phases.txt 2>&1
done
cat gpurun_out/phases.txt
