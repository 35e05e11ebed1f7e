#!/bin/bash
# A/B of the dense-table threshold (GMBE_DENSE_RATIO) and no dense tables (debug 256): full and roots-only
cd "${GRAFT_REPO_ROOT:-.}"
for v in ${VARIANTS:-d32 d8 d4 d2 d1}; do for c in ${CONFIGS:-gh_work bx_work yg_work bx dblp}; do
 echo "$v $c $(GMBE_LIB=build_variants/libgmbe_$v.so timeout 120 python scripts/sweep.py $c '' 'debug=1024' 'debug=256' 'debug=1280' 2>&1 | sed 's/  splits.*//;s/ *count [0-9]* *//' | tr '\n' '|')"
done; done
