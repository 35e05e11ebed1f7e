#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
VARIANTS="prev r1base" PYTEST_K="thread_tier or full_config_vs or g0 or random or er40 or donation or stream" bash scripts/gpu_ab.sh
timeout 300 python scripts/timeline.py gh_work > gpurun_out/tl_gh_work2.json 2>&1
python - <<'PY'
import json
d=json.load(open("gpurun_out/tl_gh_work2.json"))
print("span_us", d["span_us"], "kernel_ms", d["kernel_ms"])
print("busy", d["busy_warps_per_bin"])
print("last_to_end", d["last_to_end"][:5])
print("longest", d["longest"][:5])
PY
