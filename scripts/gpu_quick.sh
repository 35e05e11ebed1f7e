#!/bin/bash
# Quick GPU iteration: parity tests + kernel times on every config.
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
: > gpurun_out/configs.txt
for c in ${CONFIGS:-gh_work yg gh bx dblp}; do echo "== $c" >> gpurun_out/configs.txt; timeout 300 python scripts/sweep.py $c "" ${SWEEP} >> gpurun_out/configs.txt 2>&1; done
tail -c 2500 gpurun_out/pytest_gpu.log; cat gpurun_out/configs.txt
