#!/bin/bash
# repeated A/B of build variants (two processes per variant and config)
cd "${GRAFT_REPO_ROOT:-.}"
for rep in 1 2; do for v in ${VARIANTS}; do for c in ${CONFIGS:-gh_work yg_work bx bx_work dblp}; do
 echo "$rep $v $c $(GMBE_LIB=build_variants/libgmbe_$v.so timeout 120 python scripts/sweep.py $c '' 2>&1 | tail -1 | sed 's/  splits.*//;s/ *count [0-9]* *//')"
done; done; done
