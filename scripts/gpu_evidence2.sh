#!/bin/bash
# round 2 (session 2) evidence: GPU suite, bench lines (all shapes), reference arm, launch list,
# ncu full of k_enum on gh_work / dblp / bx, projected shard balance
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/ev_bench_gh_work.json 2> gpurun_out/ev_bench_gh_work.err
for c in dblp bx bx_work yg_work gh yg; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/ev_bench_$c.json 2> gpurun_out/ev_bench_$c.err
done
timeout 900 python bench.py --impl reference > gpurun_out/ev_bench_ref_gh_work.json 2> gpurun_out/ev_bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_launches_gh_work.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ev_bench_under_ncu.log 2>&1
python scripts/launch_summary.py gpurun_out/ev_launches_gh_work.csv > gpurun_out/ev_launches_gh_work.txt 2>&1
for c in gh_work dblp bx; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_enum$" -s 1 -c 1 -o gpurun_out/ev_$c python scripts/ncu_target.py $c > gpurun_out/ev_ncu_$c.log 2>&1
  python scripts/ncu_summary.py gpurun_out/ev_$c.ncu-rep --json gpurun_out/ev_ncu_$c.json > gpurun_out/ev_ncu_$c.txt 2>&1
done
for c in gh_work bx_work dblp; do timeout 900 python scripts/shard_times.py $c 2 4 8 mode=cost > gpurun_out/ev_shards_$c.json 2>&1; done
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log
for f in gpurun_out/ev_bench_*.json; do echo "== $f"; cat $f | cut -c1-300; done
head -8 gpurun_out/ev_launches_gh_work.txt; for c in gh_work dblp bx; do head -3 gpurun_out/ev_ncu_$c.txt; done
cat gpurun_out/ev_shards_*.json | cut -c1-400
