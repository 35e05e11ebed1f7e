#!/bin/bash
# projected x8 (cost parts) per build variant, twice
cd "${GRAFT_REPO_ROOT:-.}"
for rep in 1 2; do for v in ${VARIANTS}; do for c in ${CONFIGS:-gh_work}; do
 echo "$rep $v $c $(GMBE_LIB=build_variants/libgmbe_$v.so timeout 300 python scripts/shard_times.py $c 8 mode=cost 2>&1 | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print("n1 %.2f  x8 max %.2f mean %.2f -> %.2fx" % (d["n1_ms"], d["n8"]["max_ms"], d["n8"]["mean_ms"], d["n8"]["projected_speedup"]))')"
done; done; done
