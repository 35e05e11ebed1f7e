#!/bin/bash
# Compare library variants (build_variants/libgmbe_<name>.so) on configs:  VARIANTS="a b" CONFIGS="gh_work dblp"
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
: > gpurun_out/variants.txt
for c in ${CONFIGS:-gh_work dblp}; do
  for v in ${VARIANTS}; do
    echo "== $c $v" >> gpurun_out/variants.txt
    GMBE_LIB=build_variants/libgmbe_$v.so timeout 300 python scripts/sweep.py $c "" ${SWEEP} >> gpurun_out/variants.txt 2>&1
  done
done
for v in ${SHARD_VARIANTS}; do
  GMBE_LIB=build_variants/libgmbe_$v.so timeout 300 python scripts/shard_times.py ${SHARD_CONFIG:-gh_work} 8 | python -c "import sys,json; d=json.load(sys.stdin); print('$v shard8', d['n1_ms'], d['n8']['max_ms'], d['n8']['imbalance'])" >> gpurun_out/variants.txt 2>&1
done
cat gpurun_out/variants.txt
