#!/bin/bash
# round 2 (session 2): heavy-root phases on bx_work, projected shard balance, dblp phase totals and
# root-construction-only timing
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python scripts/root_phases.py bx_work 6 > gpurun_out/rp_bx_work.txt 2>&1
timeout 300 python scripts/shard_times.py bx_work 8 mode=cost > gpurun_out/shards_bx_work.json 2>&1
timeout 300 python scripts/shard_times.py gh_work 8 mode=cost > gpurun_out/shards_gh_work.json 2>&1
timeout 300 python scripts/phase_totals.py dblp > gpurun_out/pt_dblp.txt 2>&1
timeout 300 python scripts/phase_totals.py gh_work > gpurun_out/pt_gh_work.txt 2>&1
timeout 300 python scripts/sweep.py dblp "" "debug=1024" "root_chunk=16" > gpurun_out/dblp_roots_only.txt 2>&1
cat gpurun_out/rp_bx_work.txt gpurun_out/shards_*.json gpurun_out/pt_*.txt gpurun_out/dblp_roots_only.txt
