#!/bin/bash
# A/B of build variants: kernel ms on the configs and projected x8 balance (cost parts) on gh_work / bx_work
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
: > gpurun_out/ab.txt
for v in ${VARIANTS}; do
  if [ $v = base ]; then L=""; else L=build_variants/libgmbe_$v.so; fi
  for c in ${CONFIGS:-gh_work dblp bx bx_work yg_work}; do
    echo "== $c $v" >> gpurun_out/ab.txt
    GMBE_LIB=$L timeout 300 python scripts/sweep.py $c "" >> gpurun_out/ab.txt 2>&1
  done
  for c in ${SHARD_CONFIGS:-gh_work bx_work}; do
    echo "== shards $c $v" >> gpurun_out/ab.txt
    GMBE_LIB=$L timeout 300 python scripts/shard_times.py $c 8 mode=cost >> gpurun_out/ab.txt 2>&1
  done
done
sed 's/  splits.*//' gpurun_out/ab.txt
