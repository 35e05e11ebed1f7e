#!/bin/bash
# N1/N4 call: GPU tests, projected multi-GPU balance of interleave vs cost parts, default bench,
# ncu --set full of k_enum (gh_work).  Outputs land in gpurun_out/.
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
: > gpurun_out/shards.jsonl
for c in gh_work bx_work bx dblp yg_work; do
  for m in interleave cost; do timeout 300 python scripts/shard_times.py $c 2 4 8 mode=$m >> gpurun_out/shards.jsonl 2>&1; done
done
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_enum -s 1 -c 1 -o gpurun_out/prof python scripts/ncu_target.py gh_work > gpurun_out/ncu.log 2>&1
tail -3 gpurun_out/pytest_gpu.log; cat gpurun_out/shards.jsonl gpurun_out/bench.json; tail -2 gpurun_out/ncu.log
