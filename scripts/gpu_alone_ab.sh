#!/bin/bash
# heavy roots alone + N=1 + projected x8 per variant
cd "${GRAFT_REPO_ROOT:-.}"
for v in ${VARIANTS}; do
  echo "$v alone $(GMBE_LIB=build_variants/libgmbe_$v.so timeout 300 python scripts/roots_alone_times.py gh_work 54177 54411 54955 53998 53460 2>&1 | tail -1)"
done
VARIANTS="$VARIANTS" CONFIGS="gh_work" bash scripts/gpu_ab_shards8.sh
