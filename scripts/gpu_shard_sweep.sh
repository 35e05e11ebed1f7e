#!/bin/bash
# Split-threshold / thread-tier sweep for 1/8 root shards (tail latency), vs the N=1 defaults
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
: > gpurun_out/shard_sweep.jsonl
for c in gh_work bx; do
  for kv in "" "bound_height=8 bound_size=300" "bound_height=6 bound_size=200" "bound_height=10 bound_size=250" "bound_height=4 bound_size=100" "split_wide=16" "thr_min=8"; do
    timeout 200 python scripts/shard_times.py $c 8 $kv | python -c "import sys,json; d=json.load(sys.stdin); print(json.dumps({'config':'$c','opts':'$kv','n1_ms':round(d['n1_ms'],3),'n8_max_ms':round(d['n8']['max_ms'],3),'n8_imb':round(d['n8']['imbalance'],3),'proj':round(d['n8']['projected_speedup'],2)}))" >> gpurun_out/shard_sweep.jsonl 2>&1
  done
done
cat gpurun_out/shard_sweep.jsonl
